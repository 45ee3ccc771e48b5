#!/bin/bash
# launch lists (time + DRAM bytes) of one bench step at 4 and 8 bits, and full captures of the
# dominant kernel (channel-major res2a_branch2c) and the stem, exported to CSV (reports stay small)
TAG=${1:-r2f}
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
for b in 4 8; do
  timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
    -k regex:"qconv" -s 53 -c 53 --csv --log-file gpurun_out/${TAG}_launches_a$b.csv \
    python bench.py --bits $b --profile-steps 1 --warmup 1 > gpurun_out/${TAG}_ncu_launch_a$b.log 2>&1
  python scripts/prof_launches.py gpurun_out/${TAG}_launches_a$b.csv ${TAG}_a$b $b 256
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:qconv_t_kernel -s 28 -c 1 \
  -o gpurun_out/${TAG}_full_trans python bench.py --bits 4 --profile-steps 1 --warmup 1 > gpurun_out/${TAG}_ncu_full.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:qconv_halo_kernel -s 4 -c 1 \
  -o gpurun_out/${TAG}_full_stem python bench.py --bits 4 --profile-steps 1 --warmup 1 >> gpurun_out/${TAG}_ncu_full.log 2>&1
cp profiles/${TAG}_* gpurun_out/ 2>/dev/null
ls -la gpurun_out | grep $TAG
