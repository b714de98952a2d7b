#!/bin/bash
# ncu evidence for the final round-1 GEMM / Cholesky kernels (2-SM pair GEMM,
# dataflow POTRF, TRSM leaf): launch lists + per-launch metrics of one
# Cholesky step's GEMMs + --set full captures.
set -u
B="python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-strategies --no-e2e --no-profile"
mkdir -p gpurun_out
for app in cholesky sgemm matmul1k; do
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$app.csv $B --app $app > gpurun_out/ncu_l_$app.log 2>&1
  echo "$app launches rc=$?"
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:gemm_tf32x3 -s 10 -c 1 -o gpurun_out/prof_chol_gemm $B --app cholesky > gpurun_out/ncu_f1.log 2>&1; echo "chol gemm full rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:potrf_df -s 4 -c 1 -o gpurun_out/prof_chol_potrf $B --app cholesky > gpurun_out/ncu_f2.log 2>&1; echo "potrf full rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:trsm_leaf -s 8 -c 1 -o gpurun_out/prof_chol_leaf $B --app cholesky > gpurun_out/ncu_f3.log 2>&1; echo "leaf full rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:gemm_tf32x3 -s 1 -c 1 -o gpurun_out/prof_sgemm $B --app sgemm > gpurun_out/ncu_f4.log 2>&1; echo "sgemm full rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:gemm_tf32x3 -s 1 -c 1 -o gpurun_out/prof_matmul1k $B --app matmul1k > gpurun_out/ncu_f5.log 2>&1; echo "matmul1k full rc=$?"
