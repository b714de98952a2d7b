cd /root/repo
timeout 600 python -m pytest tests -m gpu -q -x -k "sgemm or matmul" --timeout 300 2>&1 | tail -2 >> gpurun_out/ab.txt
timeout 300 python tools/_st.py >> gpurun_out/ab.txt 2>&1
for r in 1 2; do
timeout 600 python bench.py --app matmul1k --steps 20 --warmup 5 --no-strategies --no-cpu-baseline --no-e2e > gpurun_out/ab.log 2>&1
python3 -c "
import json
d=[json.loads(l) for l in open('gpurun_out/ab.log') if l.startswith('{')][-1]
print('mm1k', round(d['ms_per_step'],4), round(d['value'],2), d['unit'], round(d['roofline']['frac'],3), d['roofline'].get('avg_launch_ms'), d['clocks']['sm_mhz'])" >> gpurun_out/ab.txt
done
