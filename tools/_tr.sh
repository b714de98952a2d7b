cd /root/repo
rm -f gpurun_out/chol_trace.csv
MM_TRACE=gpurun_out/chol_trace.csv timeout 300 python bench.py --app cholesky --steps 1 --warmup 3 --kernel-timing all --no-cpu-baseline --no-e2e > gpurun_out/ct.log 2>&1
python tools/chol_trace.py gpurun_out/chol_trace.csv > gpurun_out/chol_trace_summary.txt 2>&1
