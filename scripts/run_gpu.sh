#!/bin/bash
# usage: scripts/run_gpu.sh TAG [tests|bench|ncu|all]
TAG=${1:-r1}; WHAT=${2:-all}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1
if [[ $WHAT == tests || $WHAT == all ]]; then
  timeout 1200 python -m pytest tests -m gpu -q --timeout 300 > gpurun_out/tests_$TAG.log 2>&1
fi
if [[ $WHAT == bench || $WHAT == all || $WHAT == ncu ]]; then
  timeout 900 python bench.py --steps 30 --warmup 5 --layers-json gpurun_out/layers_a4_$TAG.json > gpurun_out/bench_a4_$TAG.json 2> gpurun_out/bench_a4_$TAG.err
  timeout 600 python bench.py --bits 8 --steps 30 --warmup 5 --no-cpu-baseline --no-e2e --layers-json gpurun_out/layers_a8_$TAG.json > gpurun_out/bench_a8_$TAG.json 2> gpurun_out/bench_a8_$TAG.err
fi
if [[ $WHAT == ncu || $WHAT == all ]]; then
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$TAG.csv python bench.py --profile-steps 1 --warmup 1 > gpurun_out/ncu_launch_$TAG.log 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:qconv_fwd -s 53 -c 12 -o gpurun_out/prof_$TAG python bench.py --profile-steps 1 --warmup 1 > gpurun_out/ncu_full_$TAG.log 2>&1
fi
tail -3 gpurun_out/tests_$TAG.log 2>/dev/null
head -c 600 gpurun_out/bench_a4_$TAG.json 2>/dev/null
