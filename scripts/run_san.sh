#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck over scripts/sanitize_cases.py: bash scripts/run_san.sh <tag>
TAG=${1:-r2i}
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
python paper_conf_icpp_hanhyylhgwwlq20_b200/_build.py > /dev/null 2>&1
python scripts/sanitize_cases.py > gpurun_out/${TAG}_sanitize_cases_plain.log 2>&1; tail -2 gpurun_out/${TAG}_sanitize_cases_plain.log
for tool in memcheck racecheck synccheck; do
  timeout 1200 compute-sanitizer --tool $tool --print-limit 50 python scripts/sanitize_cases.py > gpurun_out/${TAG}_san_$tool.log 2>&1
  echo "$tool rc=$?"; tail -3 gpurun_out/${TAG}_san_$tool.log
done
