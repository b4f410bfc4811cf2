#!/bin/bash
# Full ncu captures of single launches (run under gpurun):
#   bash tools/ncu_cap.sh name "prof_one args" kernel-regex [name args regex ...]
mkdir -p gpurun_out/ncu
while [ $# -ge 3 ]; do
  timeout 300 ncu --set full --import-source on --clock-control none -k regex:"$3" -s 2 -c 1 \
    -o gpurun_out/ncu/$1 python tools/prof_one.py $2 > gpurun_out/ncu/$1.log 2>&1
  echo "$1 rc=$?"
  ncu -i gpurun_out/ncu/$1.ncu-rep --page raw --csv > gpurun_out/ncu/$1.raw.csv 2>/dev/null
  ncu -i gpurun_out/ncu/$1.ncu-rep --page details --csv > gpurun_out/ncu/$1.details.csv 2>/dev/null
  shift 3
done
