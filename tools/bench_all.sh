#!/bin/bash
# One bench line per BASELINE config / paper app (1 GPU) into gpurun_out/bench_<app>.json.
mkdir -p gpurun_out
for app in stream stream-loop hotspot stencil blackscholes matmul1k sgemm cholesky nbody; do
  case $app in
    cholesky|nbody) extra="--steps 5";;
    hotspot|stencil) extra="--steps 5";;
    *) extra="";;
  esac
  timeout 600 python bench.py --app $app $extra > gpurun_out/bench_$app.log 2>&1
  tail -n 1 gpurun_out/bench_$app.log > gpurun_out/bench_$app.json
  echo "$app rc=$?"
done
