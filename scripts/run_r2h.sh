#!/bin/bash
# Round-2 (continued) evidence: re-tuned plans, GPU tests, default bench lines (A4W4 / A8W8),
# C1/C2/C4 lines, ncu launch lists + full captures of the channel-major kernel and the stem.
TAG=${1:-r2h}
cd "$(dirname "$0")/.."
mkdir -p gpurun_out plans
python paper_conf_icpp_hanhyylhgwwlq20_b200/_build.py > /dev/null 2>&1
for b in 4 8; do
  timeout 900 python bench.py --bits $b --steps 20 --warmup 5 --no-cpu-baseline --no-e2e --tune --save-plans plans/resnet50_trunk_a${b}_b256.json > gpurun_out/${TAG}_trunk_tuned_a$b.json 2> gpurun_out/${TAG}_trunk_tuned_a$b.err
  python -c "import json;d=json.load(open('gpurun_out/${TAG}_trunk_tuned_a$b.json'));print('trunk tuned', $b, d['ms_per_step'], d['parity']['bit_exact'])"
  cp plans/resnet50_trunk_a${b}_b256.json gpurun_out/${TAG}_plans_a$b.json
done
timeout 900 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/${TAG}_tests.log 2>&1; tail -2 gpurun_out/${TAG}_tests.log
for b in 4 8; do
  timeout 900 python bench.py --bits $b --layers-json gpurun_out/${TAG}_layers_a$b.json > gpurun_out/${TAG}_bench_a$b.json 2> gpurun_out/${TAG}_bench_a$b.err
  python -c "import json;d=json.load(open('gpurun_out/${TAG}_bench_a$b.json'));print('bench', $b, d['value'], d['ms_per_step'], d['e2e']['value'], d['roofline']['frac'], d['parity']['bit_exact'], d['clocks'])"
done
for w in c1 c2 c4; do
  timeout 600 python bench.py --workload $w --steps 20 --warmup 3 --layers-json gpurun_out/${TAG}_${w}_layers.json > gpurun_out/${TAG}_$w.json 2> gpurun_out/${TAG}_$w.err
  python -c "import json;d=json.load(open('gpurun_out/${TAG}_$w.json'));print('$w', d['value'], d['unit'], d['roofline']['frac'], d['parity']['bit_exact'])"
done
timeout 1500 bash scripts/prof_r2.sh ${TAG}
