#!/bin/bash
# bench A/B of the current build + a QC_DEBUG trace of one layer: bash scripts/ab_trace.sh layer:bits
cd "$(dirname "$0")/.."
bash scripts/ab_bench.sh ""
python paper_conf_icpp_hanhyylhgwwlq20_b200/_build.py -DQC_DEBUG > /dev/null 2>&1
python scripts/trace_tiles.py "$@" 2>&1 | tee gpurun_out/trace_last.txt
python paper_conf_icpp_hanhyylhgwwlq20_b200/_build.py > /dev/null 2>&1
