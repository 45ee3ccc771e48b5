#!/bin/bash
mkdir -p gpurun_out
python scripts/time_quant.py > gpurun_out/exp5.txt 2>&1
for E in 0 128 32 160; do
QC_EXPERIMENT=$E python scripts/time_layer.py res2a_branch2c:8 res2a_branch2c:4 res3a_branch2c:8 res4b_branch2c:8 res2b_branch2a:4 >> gpurun_out/exp5.txt 2>&1
done
