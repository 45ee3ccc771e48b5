#!/bin/bash
# round-1 GPU session: bench (4-bit, 8-bit), ncu launch list, ncu full on 12 conv launches
set -x
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1
timeout 600 python bench.py --steps 30 --warmup 5 --layers-json gpurun_out/layers_a4_r1.json > gpurun_out/bench_a4_r1.json 2> gpurun_out/bench_a4_r1.err
timeout 600 python bench.py --bits 8 --steps 30 --warmup 5 --no-cpu-baseline --layers-json gpurun_out/layers_a8_r1.json > gpurun_out/bench_a8_r1.json 2> gpurun_out/bench_a8_r1.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_r1.csv python bench.py --profile-steps 1 --warmup 1 > gpurun_out/ncu_launch.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:qconv_fwd -s 53 -c 12 -o gpurun_out/prof_r1 python bench.py --profile-steps 1 --warmup 1 > gpurun_out/ncu_full.log 2>&1
ls -la gpurun_out
