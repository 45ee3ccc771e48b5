#!/bin/bash
mkdir -p gpurun_out
./scripts/micro/mma_bench > gpurun_out/mma_bench.txt 2>&1
