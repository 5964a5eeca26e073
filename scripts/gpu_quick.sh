mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest rc=$?
tail -3 gpurun_out/pytest_gpu.log
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --out gpurun_out/bench_quick.json > gpurun_out/bench_quick.log 2>&1; echo bench rc=$?
python - <<'PY'
import json
d=json.load(open('gpurun_out/bench_quick.json'))
print('value',d['value'],'pct',d['pct_fp32_peak_eff'],'clocks',d['clocks'])
for k,v in d['layers'].items(): print(k, {a:round(b,2) for a,b in v.items()})
print('roofline',d['roofline']['frac'],'e2e',d.get('e2e',{}).get('value'))
PY
