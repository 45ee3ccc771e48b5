#!/bin/bash
mkdir -p gpurun_out
./scripts/micro/tma_bench > gpurun_out/tma_bench3.txt 2>&1
