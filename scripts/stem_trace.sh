#!/bin/bash
# cycle-stamped per-role timeline of the fused stem (QC_DEBUG build): bash scripts/stem_trace.sh
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
python paper_conf_icpp_hanhyylhgwwlq20_b200/_build.py -DQC_DEBUG > /dev/null 2>&1 || echo buildfail
timeout 120 python scripts/trace_stem.py /tmp/tr.bin 4 0 2>&1 | tail -14
