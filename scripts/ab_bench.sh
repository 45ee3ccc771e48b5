#!/bin/bash
# A/B of compile-time variants on the full bench step: bash scripts/ab_bench.sh "<flags1>" ...
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
i=0
for flags in "$@"; do
  python paper_conf_icpp_hanhyylhgwwlq20_b200/_build.py $flags > /dev/null 2>&1 || { echo "build failed: $flags"; continue; }
  for b in 4 8; do
    timeout 300 python bench.py --bits $b --steps 20 --warmup 5 --no-cpu-baseline --no-e2e --no-verify --layers-json gpurun_out/ab_${i}_layers_a$b.json > gpurun_out/ab_${i}_a$b.json 2>/dev/null
    python -c "import json;d=json.load(open('gpurun_out/ab_${i}_a$b.json'));print('$flags'.ljust(40), $b, round(d['ms_per_step'],4), {k:round(v['us']) for k,v in d['roofline']['families'].items()})"
  done
  i=$((i+1))
done
