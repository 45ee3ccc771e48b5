#!/bin/bash
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
for b in 4 8; do
timeout 600 python bench.py --bits $b --steps 20 --warmup 5 --no-cpu-baseline --no-e2e --layers-json gpurun_out/r2b_layers_a$b.json > gpurun_out/r2b_bench_a$b.json 2> gpurun_out/r2b_bench_a$b.err
python -c "import json;d=json.load(open('gpurun_out/r2b_bench_a$b.json'));print($b, d['ms_per_step'], d['value'], d['parity']['bit_exact'], d['roofline']['frac_of_roofline_time'])"; tail -3 gpurun_out/r2b_bench_a$b.err
done
