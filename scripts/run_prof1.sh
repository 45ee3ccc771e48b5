#!/bin/bash
# usage: scripts/run_prof1.sh TAG BITS layer -- ncu --set full of one trunk layer, exported to CSV
TAG=$1; BITS=$2; L=$3
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
R=gpurun_out/prof_${TAG}
timeout 600 ncu --set full --import-source on --clock-control none -k regex:qconv -s 3 -c 1 -o $R python scripts/time_trunk.py $BITS $L > gpurun_out/ncu_$TAG.log 2>&1
ncu -i $R.ncu-rep --page raw --csv > ${R}_raw.csv 2>/dev/null
ncu -i $R.ncu-rep --page source --csv --print-source sass > ${R}_sass.csv 2>/dev/null
ncu -i $R.ncu-rep --page details --csv > ${R}_details.csv 2>/dev/null
rm -f $R.ncu-rep
ls -la gpurun_out | tail -5
