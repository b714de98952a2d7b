cd /root/repo
for app in matmul1k stream; do
for f in "--kernel-timing none" "--kernel-timing none --no-repeat" "--kernel-timing last" "--kernel-timing last --no-repeat"; do
timeout 600 python bench.py --app $app --steps 20 --warmup 5 --no-strategies --no-cpu-baseline --no-e2e $f > gpurun_out/ab.log 2>&1
python3 -c "
import json
d=[json.loads(l) for l in open('gpurun_out/ab.log') if l.startswith('{')][-1]
print('$app', '$f', round(d['ms_per_step'],4), round(d['value'],2), d['unit'], d['gpu_launches'], d['clocks']['sm_mhz'])" >> gpurun_out/ab.txt
done; done
