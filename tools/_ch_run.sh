for ov in 1 0; do
MM_TRSM_OVERLAP=$ov MM_TRACE=gpurun_out/chol_trace_ov$ov.txt timeout 300 python bench.py --app cholesky --steps 1 --warmup 1 --no-strategies --no-e2e --no-cpu-baseline --no-profile --kernel-timing all > /dev/null 2>&1
echo "overlap=$ov"; python tools/chol_trace.py gpurun_out/chol_trace_ov$ov.txt | sed -n '1,2p;25,35p'
done
