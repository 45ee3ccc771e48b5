#!/bin/bash
# re-tune the trunk plan tables on the current build, then time the default bench (tables
# copied back through gpurun_out/): bash scripts/retune_bench.sh <tag>
TAG=${1:-rt}
cd "$(dirname "$0")/.."
mkdir -p gpurun_out plans
python paper_conf_icpp_hanhyylhgwwlq20_b200/_build.py > /dev/null 2>&1
for b in 4 8; do
  timeout 900 python bench.py --bits $b --steps 20 --warmup 5 --no-cpu-baseline --no-e2e --tune --save-plans plans/resnet50_trunk_a${b}_b256.json > gpurun_out/${TAG}_tuned_a$b.json 2>/dev/null
  cp plans/resnet50_trunk_a${b}_b256.json gpurun_out/${TAG}_plans_a$b.json
  timeout 600 python bench.py --bits $b --steps 20 --warmup 5 --no-cpu-baseline --no-e2e --layers-json gpurun_out/${TAG}_layers_a$b.json > gpurun_out/${TAG}_bench_a$b.json 2>/dev/null
  python -c "import json;d=json.load(open('gpurun_out/${TAG}_bench_a$b.json'));print('bench', $b, round(d['ms_per_step'],4), d['parity']['bit_exact'], {k:round(v['us']) for k,v in d['roofline']['families'].items()})"
done
