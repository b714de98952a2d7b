B="python bench.py --app matmul1k --steps 20 --warmup 5 --no-cpu-baseline --no-strategies --no-e2e --no-profile"
for extra in "" "--no-graph" "--kernel-timing none" "--no-graph --kernel-timing none"; do timeout 300 $B $extra 2>&1 | tail -1 | python -c "import sys,json; d=json.loads(sys.stdin.read()); print('[$extra]', round(d['ms_per_step']*1000,2), 'us', d['kernel_ms_per_step'])"; done
