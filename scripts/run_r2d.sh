#!/bin/bash
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_round2.py tests/test_gpu_kernel_paths.py -m gpu -q -x --timeout 800 -p no:cacheprovider > gpurun_out/r2d_tests.log 2>&1; tail -3 gpurun_out/r2d_tests.log
for b in 4 8; do
timeout 600 python bench.py --bits $b --steps 20 --warmup 5 --no-cpu-baseline --no-e2e --no-verify --layers-json gpurun_out/r2d_layers_a$b.json > gpurun_out/r2d_bench_a$b.json 2> gpurun_out/r2d_bench_a$b.err
python -c "import json;d=json.load(open('gpurun_out/r2d_bench_a$b.json'));print($b, d['ms_per_step'], d['value'], {k:round(v['us']) for k,v in d['roofline']['families'].items()})"; tail -3 gpurun_out/r2d_bench_a$b.err
done
exit 0
for b in 4 8; do
timeout 600 python bench.py --bits $b --steps 20 --warmup 5 --no-cpu-baseline --no-e2e --no-verify --layers-json gpurun_out/r2d_layers_sleep_a$b.json > gpurun_out/r2d_bench_sleep_a$b.json 2> gpurun_out/r2d_bench_sleep_a$b.err
python -c "import json;d=json.load(open('gpurun_out/r2d_bench_sleep_a$b.json'));print('sleep', $b, d['ms_per_step'], d['value'], {k:round(v['us']) for k,v in d['roofline']['families'].items()})"; tail -3 gpurun_out/r2d_bench_sleep_a$b.err
done
