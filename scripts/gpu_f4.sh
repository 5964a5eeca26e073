mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_f4.py -x -q > gpurun_out/pytest_f4.log 2>&1; echo pytest_f4 rc=$?
tail -15 gpurun_out/pytest_f4.log
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --out gpurun_out/bench_f4.json > gpurun_out/bench_f4.log 2>&1; echo bench rc=$?
tail -5 gpurun_out/bench_f4.log
python - <<'PY'
import json
d=json.load(open('gpurun_out/bench_f4.json'))
print('fp32', d['value'], {k: round(v['conv_tflops_eff'] if 'conv_tflops_eff' in v else -1, 1) for k, v in d['layers'].items()})
for k,v in d.get('variants',{}).items(): print(k, round(v['value'],1), {a: round(b,1) for a,b in v['layers_eff_tflops'].items()})
PY
