#!/bin/bash
# ncu evidence for the round-1 Cholesky / GEMM rework: launch lists of the
# Cholesky and SGEMM benches, per-launch metrics of every gemm_tf32x3 launch
# of one Cholesky step, and --set full captures of the largest bulk GEMM
# launch, the dataflow POTRF, the TRSM leaf and the SGEMM / MatrixMul GEMMs.
set -u
B="python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-strategies --no-e2e --no-profile"
mkdir -p gpurun_out
for app in cholesky sgemm matmul1k; do
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$app.csv $B --app $app > gpurun_out/ncu_l_$app.log 2>&1
  echo "$app launches rc=$?"
done
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active,launch__grid_size
timeout 900 ncu --metrics $M --clock-control none --csv -k regex:gemm_tf32x3 --log-file gpurun_out/chol_gemms.csv $B --app cholesky > gpurun_out/ncu_g_chol.log 2>&1
echo "cholesky gemm metrics rc=$?"
# index (among gemm_tf32x3 launches) of the largest grid
IDX=$(python - << 'PY'
import csv, io
rows = [l for l in open("gpurun_out/chol_gemms.csv") if not l.startswith("==")]
best, bi, ids = -1, 0, {}
for r in csv.DictReader(io.StringIO("".join(rows))):
    if r["Metric Name"] == "launch__grid_size":
        i = int(r["ID"]); g = float(r["Metric Value"].replace(",", ""))
        ids.setdefault(i, len(ids))
        if g > best: best, bi = g, ids[i]
print(bi)
PY
)
echo "largest gemm launch index $IDX"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:gemm_tf32x3 -s $IDX -c 1 -o gpurun_out/prof_chol_gemm $B --app cholesky > gpurun_out/ncu_f1.log 2>&1; echo "chol gemm full rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:potrf_df -s 4 -c 1 -o gpurun_out/prof_chol_potrf $B --app cholesky > gpurun_out/ncu_f2.log 2>&1; echo "potrf full rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:trsm_leaf -s 8 -c 1 -o gpurun_out/prof_chol_leaf $B --app cholesky > gpurun_out/ncu_f3.log 2>&1; echo "leaf full rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:gemm_tf32x3 -s 1 -c 1 -o gpurun_out/prof_sgemm $B --app sgemm > gpurun_out/ncu_f4.log 2>&1; echo "sgemm full rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:gemm_tf32x3 -s 1 -c 1 -o gpurun_out/prof_matmul1k $B --app matmul1k > gpurun_out/ncu_f5.log 2>&1; echo "matmul1k full rc=$?"
