for m in 0 1; do
  R=gpurun_out/prof_c2_$m
  if [ $m = 1 ]; then export QC_CTA2=1; fi
  timeout 300 ncu --set full --clock-control none -k regex:qconv -s 3 -c 1 -o $R python scripts/time_trunk.py 8 res4b_branch2b > gpurun_out/ncu_c2_$m.log 2>&1
  ncu -i $R.ncu-rep --page raw --csv > ${R}_raw.csv 2>/dev/null
  rm -f $R.ncu-rep
done
