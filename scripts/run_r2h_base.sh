#!/bin/bash
cd "$(dirname "$0")/.." 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
python paper_conf_icpp_hanhyylhgwwlq20_b200/_build.py > /dev/null 2>&1
timeout 900 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/r2h_tests.log 2>&1; tail -2 gpurun_out/r2h_tests.log
for b in 4 8; do
  timeout 600 python bench.py --bits $b --steps 20 --warmup 5 --no-cpu-baseline --no-e2e --layers-json gpurun_out/r2h_layers_a$b.json > gpurun_out/r2h_bench_a$b.json 2> gpurun_out/r2h_bench_a$b.err
  python -c "import json;d=json.load(open('gpurun_out/r2h_bench_a$b.json'));print('bench', $b, d['value'], d['ms_per_step'], d['roofline']['frac'], d['parity']['bit_exact'], d['clocks'], {k:round(v['us']) for k,v in d['roofline']['families'].items()})"
done
