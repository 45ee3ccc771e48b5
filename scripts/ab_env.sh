#!/bin/bash
# A/B of environment switches on the full bench step: bash scripts/ab_env.sh "" "QC_X=1" ...
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
python paper_conf_icpp_hanhyylhgwwlq20_b200/_build.py > /dev/null 2>&1
i=0
for envs in "$@"; do
  for b in 4 8; do
    env $envs timeout 300 python bench.py --bits $b --steps 20 --warmup 5 --no-cpu-baseline --no-e2e --no-verify --layers-json gpurun_out/abe_$b.json > gpurun_out/abe_${i}_a$b.json 2>/dev/null
    python -c "import json;d=json.load(open('gpurun_out/abe_${i}_a$b.json'));print('$envs'.ljust(30), $b, round(d['ms_per_step'],4), {k:round(v['us']) for k,v in d['roofline']['families'].items()})"
  done
  i=$((i+1))
done
