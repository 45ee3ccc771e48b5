#!/bin/bash
# C5's per-GPU shard sizes on one GPU (256/G images for G = 1, 2, 4, 8): the work one rank does
# in the strong-scaling run (no collective in the timed loop) -- a proxy for the 1/2/4/8 curve
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
python paper_conf_icpp_hanhyylhgwwlq20_b200/_build.py > /dev/null 2>&1
for b in 4 8; do for n in 256 128 64 32; do
  timeout 600 python bench.py --bits $b --batch $n --steps 30 --warmup 5 --no-cpu-baseline --no-e2e > gpurun_out/shard_a${b}_b$n.json 2>/dev/null
  python -c "import json;d=json.load(open('gpurun_out/shard_a${b}_b$n.json'));print('A${b}W${b} shard', $n, 'images/GPU:', round(d['value']), 'img/s', round(d['ms_per_step'],4), 'ms/step', d['parity']['bit_exact'], d['config']['plans'][:40])"
done; done
