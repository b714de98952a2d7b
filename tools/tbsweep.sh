# HotSpot temporal-block sweep: parity of the tb kernels, then bench per tb
timeout 600 python -m pytest tests/test_gpu_parity.py -q -m gpu -x -k "temporal" 2>&1 | tail -2
for tb in ${TBS:-2 4 8}; do
  timeout 300 python bench.py --app hotspot --tb $tb --steps 3 --warmup 3 --no-cpu-baseline --no-strategies --no-e2e --no-profile 2>&1 | tail -1 | python -c "import sys,json; d=json.loads(sys.stdin.read()); r=d['roofline']; print('TB', $tb, round(d['ms_per_step'],2), 'ms', r['bound'], round(r['frac'],3), '%.3e upd/s' % r.get('cell_updates_per_s', 0))"
done
