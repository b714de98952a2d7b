#!/bin/bash
# ncu --set full of the dominant kernel of each app, taken from the bench's
# own warm-up step (equal profile => no profiling launches precede it).
set -u
B="python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-strategies --no-e2e --no-profile"
mkdir -p gpurun_out
for spec in "hotspot:hotspot_vec:5" "stencil:residual_rows:5" "blackscholes:bs_vec:0" "sgemm:gemm_tf32x3:0" "cholesky:gemm_tf32x3:4" "cholesky:trsm_rows:3"; do
  IFS=: read app k skip <<< "$spec"
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:$k -s $skip -c 1 -o gpurun_out/prof_${app}_$k $B --app $app > gpurun_out/ncu_f_${app}_$k.log 2>&1
  echo "$app $k full rc=$?"
done
