#!/bin/bash
# round-2 check: bench-size parity tests, default bench, per-layer workloads
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_bench.py -m gpu -q --timeout 800 -p no:cacheprovider > gpurun_out/r2a_tests_bench.log 2>&1
tail -5 gpurun_out/r2a_tests_bench.log
timeout 600 python bench.py --steps 20 --warmup 5 --layers-json gpurun_out/r2a_layers_a4.json > gpurun_out/r2a_bench_a4.json 2> gpurun_out/r2a_bench_a4.err
tail -c 3000 gpurun_out/r2a_bench_a4.json; tail -5 gpurun_out/r2a_bench_a4.err
for w in c1 c2 c4; do
  timeout 600 python bench.py --workload $w --steps 20 --warmup 3 > gpurun_out/r2a_bench_$w.json 2> gpurun_out/r2a_bench_$w.err
  python -c "import json;d=json.load(open('gpurun_out/r2a_bench_$w.json'));print('$w', d['value'], d['unit'], d['roofline']['frac'], d['parity'])" ; tail -3 gpurun_out/r2a_bench_$w.err
done
