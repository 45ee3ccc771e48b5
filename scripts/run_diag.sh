#!/bin/bash
mkdir -p gpurun_out
./scripts/micro/cvt_bench > gpurun_out/cvt_bench.txt 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q --timeout 300 -x > gpurun_out/tests_t1.log 2>&1
tail -3 gpurun_out/tests_t1.log
L="res2a_branch2c:8 res2a_branch2c:4 res2a_branch2a:4 res3a_branch1:4 res4b_branch2c:8 res4b_branch2a:4 res5a_branch2c:4 res2a_branch2b:4 res3b_branch2b:4 res4b_branch2b:4"
python scripts/time_layer.py $L > gpurun_out/time_t1.txt 2>&1
QC_NO_TRANS=1 python scripts/time_layer.py $L >> gpurun_out/time_t1.txt 2>&1
