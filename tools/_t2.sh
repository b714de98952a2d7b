cd /root/repo
timeout 300 python tools/trsm_stamps.py > gpurun_out/stamps.txt 2>&1
timeout 600 python -m pytest tests -m gpu -x -q -k "cholesky" --timeout 300 2>&1 | tail -3 >> gpurun_out/stamps.txt
for col in 1; do
MM_TRSM_COL=$col timeout 300 python bench.py --app cholesky --steps 3 --warmup 3 --kernel-timing none > gpurun_out/cb_$col.log 2>&1
echo "col=$col $(grep -o '"ms_per_step": [0-9.]*' gpurun_out/cb_$col.log) $(grep -o '"sm_mhz": [0-9.]*' gpurun_out/cb_$col.log)" >> gpurun_out/stamps.txt
done
