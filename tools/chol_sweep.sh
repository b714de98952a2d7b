#!/bin/bash
# Sweep Cholesky launch knobs (env) on the GPU box: one bench line per setting.
# usage: tools/chol_sweep.sh "G1 G2 ..." [extra bench args]  (G = MM_POTRF_GRID, 0 = default)
mkdir -p gpurun_out
for g in $1; do
  out=$(MM_POTRF_GRID=$g timeout 200 python bench.py --app cholesky --steps 5 --no-strategies --no-e2e --no-cpu-baseline --no-profile ${@:2} 2>&1 | tail -n 1)
  echo "G=$g $(echo "$out" | grep -o '"ms_per_step": [0-9.]*') $(echo "$out" | grep -o '"sm_mhz": [0-9.]*')"
done
