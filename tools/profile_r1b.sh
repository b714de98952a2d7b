#!/bin/bash
# ncu evidence for the kernels changed after the first profile pass:
# HotSpot temporal block (hotspot_tb<8>) and Nbody (f32x2).  Launch list of a
# short bench + one --set full capture of the dominant kernel.
set -u
B="python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-strategies --no-e2e"
mkdir -p gpurun_out
for spec in "hotspot:hotspot_tb" "nbody:nbody_rows"; do
  app=${spec%%:*}; k=${spec##*:}
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$app.csv $B --app $app > gpurun_out/ncu_l_$app.log 2>&1
  echo "$app launches rc=$?"
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:$k -s 2 -c 1 -o gpurun_out/prof_$app $B --app $app > gpurun_out/ncu_f_$app.log 2>&1
  echo "$app full rc=$?"
done
