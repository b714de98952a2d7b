cd /root/repo
B="python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-strategies --no-e2e --no-profile"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:gemm_tf32x3_pair -s 5 -c 1 -o gpurun_out/prof_chol_bulk $B --app cholesky > gpurun_out/ncu_bulk.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum,launch__grid_size --clock-control none -k regex:gemm_tf32x3_pair -c 12 --csv --log-file gpurun_out/bulk_list.csv $B --app cholesky > /dev/null 2>&1
