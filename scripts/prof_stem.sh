#!/bin/bash
# ncu --set full capture of the fused stem kernel alone: bash scripts/prof_stem.sh
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
python paper_conf_icpp_hanhyylhgwwlq20_b200/_build.py > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:qconv_halo_kernel -s 1 -c 1 \
  -o gpurun_out/stem_v3 python scripts/run_layer.py 4 0 3 > gpurun_out/stem_v3.log 2>&1
tail -2 gpurun_out/stem_v3.log
