#!/bin/bash
# One bench line per BASELINE config / paper app (1 GPU) into gpurun_out/bench_<app>.json
# (copied to profiles/bench_<round>/ after review).  Default K/W per app.
mkdir -p gpurun_out
for app in stream stream-loop hotspot stencil blackscholes matmul1k sgemm cholesky nbody; do
  case $app in
    cholesky|nbody) extra="--steps 5 --warmup 3";;
    hotspot|stencil) extra="--steps 5 --warmup 3";;
    *) extra="--steps 20 --warmup 5";;
  esac
  timeout 900 python bench.py --app $app $extra > gpurun_out/bench_$app.log 2>&1
  rc=$?
  grep '^{' gpurun_out/bench_$app.log | tail -n 1 > gpurun_out/bench_$app.json
  echo "$app rc=$rc"
done
