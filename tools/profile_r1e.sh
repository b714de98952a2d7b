#!/bin/bash
# ncu evidence after the round-1 HotSpot wave fix: launch list of the bench's
# HotSpot step and a --set full capture of hotspot_tb<8>.
set -u
B="python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-strategies --no-e2e --no-profile --app hotspot"
mkdir -p gpurun_out
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_hotspot_tb8e.csv $B > gpurun_out/ncu_l_hot.log 2>&1
echo "launches rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:hotspot_tb -s 3 -c 1 -o gpurun_out/prof_hotspot_tb8e $B > gpurun_out/ncu_f_hot.log 2>&1
echo "full rc=$?"
