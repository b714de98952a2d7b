cd /root/repo
B="python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-strategies --no-e2e --no-profile"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sgemm_fused -s 1 -c 1 -o gpurun_out/prof_fused_g2 $B --app matmul1k > gpurun_out/ncu_fused.log 2>&1
