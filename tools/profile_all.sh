#!/bin/bash
# ncu evidence for every app's dominant kernel (run under gpurun, one GPU).
# Launch lists: per-launch device time (cold-cache, serialised) of a short bench.
# Full captures: --set full of 2 launches of the dominant kernel.
set -u
B="python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-strategies --no-e2e"
mkdir -p gpurun_out
for spec in "hotspot:hotspot_vec" "stencil:residual_rows" "blackscholes:bs_vec" "sgemm:gemm_tf32x3" "cholesky:gemm_tf32x3"; do
  app=${spec%%:*}; k=${spec##*:}
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$app.csv $B --app $app > gpurun_out/ncu_l_$app.log 2>&1
  echo "$app launches rc=$?"
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:$k -s 8 -c 2 -o gpurun_out/prof_$app $B --app $app > gpurun_out/ncu_f_$app.log 2>&1
  echo "$app full rc=$?"
done
