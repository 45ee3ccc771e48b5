#!/bin/bash
# profile-run tile tables for C5's per-GPU shard sizes (256/G images, G = 2, 4, 8), then the
# shard timings with them (bench.py loads plans/resnet50_trunk_a<bits>_b<per_gpu>.json by default)
cd "$(dirname "$0")/.."
mkdir -p gpurun_out plans
python paper_conf_icpp_hanhyylhgwwlq20_b200/_build.py > /dev/null 2>&1
for b in 4 8; do for n in 128 64 32; do
  timeout 900 python bench.py --bits $b --batch $n --steps 20 --warmup 5 --no-cpu-baseline --no-e2e --tune --save-plans plans/resnet50_trunk_a${b}_b$n.json > /dev/null 2>&1
  cp plans/resnet50_trunk_a${b}_b$n.json gpurun_out/
  timeout 600 python bench.py --bits $b --batch $n --steps 30 --warmup 5 --no-cpu-baseline --no-e2e > gpurun_out/shardt_a${b}_b$n.json 2>/dev/null
  python -c "import json;d=json.load(open('gpurun_out/shardt_a${b}_b$n.json'));print('A${b}W${b} shard', $n, round(d['value']), 'img/s', round(d['ms_per_step'],4), 'ms', d['parity']['bit_exact'], d['config']['plans'][:48])"
done; done
