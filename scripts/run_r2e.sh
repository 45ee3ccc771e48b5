#!/bin/bash
# tests after the channel-kernel restore; f2/f4 workloads; fig11/12 ablations; tuned trunk
cd "$(dirname "$0")/.."
mkdir -p gpurun_out plans
timeout 900 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/r2e_tests.log 2>&1; tail -2 gpurun_out/r2e_tests.log
timeout 900 python scripts/fig11_fig12.py gpurun_out/r2e_fig11_fig12.json 2>&1 | tail -4
for b in 4 8; do
  timeout 600 python bench.py --workload f4 --bits $b --steps 20 --warmup 3 --layers-json gpurun_out/r2e_f4_a$b.json > /dev/null 2>gpurun_out/r2e_f4_a$b.err
  timeout 900 python bench.py --workload f4 --bits $b --steps 20 --warmup 3 --tune --save-plans gpurun_out/r2e_plans_f4_a$b.json --layers-json gpurun_out/r2e_f4_tuned_a$b.json > /dev/null 2>gpurun_out/r2e_f4t_a$b.err
  timeout 600 python bench.py --workload c3 --bits $b --steps 20 --warmup 3 --layers-json gpurun_out/r2e_c3_a$b.json > /dev/null 2>gpurun_out/r2e_c3_a$b.err
  python -c "
import json
for n in ['f4','f4_tuned','c3']:
    d=json.load(open('gpurun_out/r2e_'+n+'_a$b.json')); print(n, $b, round(d['value'],1), d['unit'], round(d['roofline']['frac'],3), d['parity']['bit_exact'])"
  timeout 900 python bench.py --bits $b --steps 20 --warmup 5 --no-cpu-baseline --no-e2e --tune --save-plans plans/resnet50_trunk_a${b}_b256.json > gpurun_out/r2e_trunk_tuned_a$b.json 2> gpurun_out/r2e_trunk_tuned_a$b.err
  python -c "import json;d=json.load(open('gpurun_out/r2e_trunk_tuned_a$b.json'));print('trunk tuned', $b, d['ms_per_step'], d['parity']['bit_exact'], {k:round(v['us']) for k,v in d['roofline']['families'].items()})"; tail -2 gpurun_out/r2e_trunk_tuned_a$b.err
  cp plans/resnet50_trunk_a${b}_b256.json gpurun_out/ 2>/dev/null
done
