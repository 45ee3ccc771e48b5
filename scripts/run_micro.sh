#!/bin/bash
mkdir -p gpurun_out
timeout 120 ./scripts/micro/cvt_bench > gpurun_out/cvt_bench.txt 2>&1
