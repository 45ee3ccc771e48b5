#!/bin/bash
# usage: scripts/run_prof.sh TAG "layer:bits ..." [tests]  -- (tests) + microbenchmarks + single-layer
# timings + ncu --set full of single layers, exported to CSV on the box (reports are too big to ship)
TAG=${1:-p}; L=${2:-"res2a_branch2c:4 res2a_branch2b:4 res4b_branch2b:4 res4b_branch2b:8"}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_$TAG.log 2>&1
if [[ "$3" == tests ]]; then timeout 900 python -m pytest tests -m gpu -q -x --timeout 300 > gpurun_out/tests_$TAG.log 2>&1; tail -3 gpurun_out/tests_$TAG.log; fi
for m in tmem_bench mma_bench cvt_bench; do [ -x scripts/micro/$m ] && timeout 120 ./scripts/micro/$m > gpurun_out/micro_${m}_$TAG.txt 2>&1; done
python scripts/time_layer.py $L > gpurun_out/time_$TAG.txt 2>&1
exp() {  # report -> csv (raw metrics + source-line hot spots), then drop the report
  ncu -i $1.ncu-rep --page raw --csv > $1_raw.csv 2>/dev/null
  ncu -i $1.ncu-rep --page details --csv > $1_details.csv 2>/dev/null
  rm -f $1.ncu-rep
}
timeout 600 ncu --set full --clock-control none -k regex:qconv_halo -c 1 -o gpurun_out/prof_${TAG}_stem python bench.py --profile-steps 1 --warmup 1 > gpurun_out/ncu_stem_$TAG.log 2>&1
exp gpurun_out/prof_${TAG}_stem
for l in $L; do
  n=${l/:/_}
  timeout 300 ncu --set full --clock-control none -k regex:qconv -s 2 -c 1 -o gpurun_out/prof_${TAG}_$n python scripts/time_layer.py $l > gpurun_out/ncu_${n}_$TAG.log 2>&1
  exp gpurun_out/prof_${TAG}_$n
done
du -sh gpurun_out; ls gpurun_out
