#!/bin/bash
# A/B of compile-time variants (last one stays built), then the GPU tests on the last variant:
# bash scripts/ab_test.sh "<flags1>" ... "<flagsN>"
cd "$(dirname "$0")/.."
bash scripts/ab_bench.sh "$@"
timeout 900 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/ab_tests.log 2>&1; tail -3 gpurun_out/ab_tests.log
