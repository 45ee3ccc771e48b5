#!/bin/bash
# sanitizers + ncu captures of the dominant kernels
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
python scripts/sanitize_cases.py > gpurun_out/r2c_plain.log 2>&1; tail -2 gpurun_out/r2c_plain.log
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 50 python scripts/sanitize_cases.py > gpurun_out/r2c_san_$tool.log 2>&1
  echo "$tool rc=$?"; tail -4 gpurun_out/r2c_san_$tool.log
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:qconv_t_kernel -s 1 -c 1 -o gpurun_out/r2c_trans python bench.py --profile-steps 1 --warmup 0 > gpurun_out/r2c_ncu_trans.log 2>&1; tail -2 gpurun_out/r2c_ncu_trans.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:qconv_halo_kernel -s 0 -c 1 -o gpurun_out/r2c_stem python bench.py --profile-steps 1 --warmup 0 > gpurun_out/r2c_ncu_stem.log 2>&1; tail -2 gpurun_out/r2c_ncu_stem.log
