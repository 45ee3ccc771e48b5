#!/bin/bash
# Round-end evidence: benches (A4W4 default + A8W8), ncu launch list with DRAM bytes over one
# bench step, ncu --set full of representative kernels (CSV export; reports are too big to ship).
TAG=${1:-r1j}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1
timeout 900 python bench.py --steps 30 --warmup 5 --layers-json gpurun_out/layers_a4_$TAG.json > gpurun_out/bench_a4_$TAG.json 2> gpurun_out/bench_a4_$TAG.err
timeout 600 python bench.py --bits 8 --steps 30 --warmup 5 --no-cpu-baseline --layers-json gpurun_out/layers_a8_$TAG.json > gpurun_out/bench_a8_$TAG.json 2> gpurun_out/bench_a8_$TAG.err
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/launches_$TAG.csv python bench.py --profile-steps 1 --warmup 1 > gpurun_out/ncu_launch_$TAG.log 2>&1
for spec in "conv1:halo_stem" "res2a_branch2b:halo_3x3" "res2a_branch2c:t_1x1" "res4b_branch2b:fwd_3x3"; do
  L=${spec%%:*}; N=${spec##*:}
  R=gpurun_out/full_${TAG}_$N
  timeout 600 ncu --set full --clock-control none -k regex:qconv -s 3 -c 1 -o $R python scripts/time_trunk.py 4 $L > gpurun_out/ncu_full_${TAG}_$N.log 2>&1
  ncu -i $R.ncu-rep --page raw --csv > ${R}_raw.csv 2>/dev/null
  rm -f $R.ncu-rep
done
ls -la gpurun_out | tail -20
