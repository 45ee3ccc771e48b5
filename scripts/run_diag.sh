#!/bin/bash
mkdir -p gpurun_out
L="res2a_branch2b:8 res2a_branch2b:4 res2a_branch2c:8 res2a_branch2c:4 res3a_branch2b:8 res4a_branch2b:8 res4b_branch2c:8"
for E in 0 3 4 7 8 16 20; do
QC_EXPERIMENT=$E python scripts/time_layer.py $L >> gpurun_out/exp2.txt 2>&1
done
