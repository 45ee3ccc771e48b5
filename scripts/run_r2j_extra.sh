#!/bin/bash
# C3 (batch 32, every layer) and f4 (bs1/bs16 + DenseNet-121) lines and the Fig.11/12 ablations on the current code
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
python paper_conf_icpp_hanhyylhgwwlq20_b200/_build.py > /dev/null 2>&1
timeout 900 python scripts/fig11_fig12.py gpurun_out/r2j_fig11_fig12.json 2>&1 | tail -4
for b in 4 8; do
  timeout 600 python bench.py --workload f4 --bits $b --steps 20 --warmup 3 --layers-json gpurun_out/r2j_f4_a$b.json > /dev/null 2>gpurun_out/r2j_f4_a$b.err
  timeout 900 python bench.py --workload f4 --bits $b --steps 20 --warmup 3 --tune --save-plans gpurun_out/r2j_plans_f4_a$b.json --layers-json gpurun_out/r2j_f4_tuned_a$b.json > /dev/null 2>gpurun_out/r2j_f4t_a$b.err
  timeout 600 python bench.py --workload c3 --bits $b --steps 20 --warmup 3 --layers-json gpurun_out/r2j_c3_a$b.json > /dev/null 2>gpurun_out/r2j_c3_a$b.err
  python -c "
import json
for n in ['f4','f4_tuned','c3']:
    d=json.load(open('gpurun_out/r2j_'+n+'_a$b.json')); print(n, $b, round(d['value'],1), d['unit'], round(d['roofline']['frac'],3), d['parity']['bit_exact'])"
done
