cd /root/repo
for r in 1 2 3; do
for cfg in "MM_POTRF_PART=3" "MM_POTRF_PART=2" "MM_TRSM_OVERLAP=0"; do
env $cfg timeout 300 python bench.py --app cholesky --steps 3 --warmup 2 --kernel-timing none --no-cpu-baseline --no-e2e --no-strategies > gpurun_out/ab.log 2>&1
echo "$cfg $(grep -o '"ms_per_step": [0-9.]*' gpurun_out/ab.log | head -1) $(grep -o '"sm_mhz": [0-9.]*' gpurun_out/ab.log)" >> gpurun_out/ab.txt
done; done
