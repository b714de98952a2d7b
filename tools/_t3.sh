cd /root/repo
timeout 900 python -m pytest tests -m gpu -x -q -k "cholesky or chol or sgemm or matmul" --timeout 300 2>&1 | tail -3 > gpurun_out/t3.txt
for i in 1 2; do
timeout 300 python bench.py --app cholesky --steps 3 --warmup 3 --kernel-timing none --no-cpu-baseline --no-e2e --no-strategies > gpurun_out/cb.log 2>&1
echo "$(grep -o '"ms_per_step": [0-9.]*' gpurun_out/cb.log | head -1) $(grep -o '"sm_mhz": [0-9.]*' gpurun_out/cb.log)" >> gpurun_out/t3.txt
done
