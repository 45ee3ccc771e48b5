#!/bin/bash
# usage: scripts/run_trace.sh TAG BITS "layers"
TAG=$1; BITS=$2; L=$3
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_$TAG.log 2>&1
QC_TRACE=/tmp/qc_trace.bin python scripts/trace_trunk.py $BITS /tmp/qc_trace.bin $L > gpurun_out/trace_$TAG.txt 2>&1
cat gpurun_out/trace_$TAG.txt | tail -60
