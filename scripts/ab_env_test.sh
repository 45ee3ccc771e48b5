bash scripts/ab_env.sh "QC_T_BNP=256" "QC_T_BNP=128"
timeout 900 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/ab_tests.log 2>&1; tail -3 gpurun_out/ab_tests.log
