#!/bin/bash
# ncu --set full (with source) of one trunk layer: bash scripts/prof_layer.sh <bits> <layer> <tag>
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
python paper_conf_icpp_hanhyylhgwwlq20_b200/_build.py > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:qconv -s 1 -c 1 \
  -o gpurun_out/$3 python scripts/run_layer.py $1 $2 3 > gpurun_out/$3.log 2>&1
tail -2 gpurun_out/$3.log
