# NEXT row N4 (FP16 / BF16 on tcgen05 kind::f16): parity tests, then a bench run with all variants.
mkdir -p gpurun_out
TAG=${1:-half}
timeout 600 python -m pytest tests/test_gpu_half.py -x -q > gpurun_out/pytest_$TAG.log 2>&1; echo pytest rc=$?; tail -30 gpurun_out/pytest_$TAG.log
timeout 600 python bench.py --no-e2e --no-cpu-baseline --out gpurun_out/bench_$TAG.json > gpurun_out/bench_$TAG.log 2>&1; echo bench rc=$?
python - <<'PY'
import json,sys
try:
    d=json.load(open('gpurun_out/bench_'+sys.argv[1] if len(sys.argv)>1 else 'gpurun_out/bench_half.json'))
except Exception as e:
    print(e); sys.exit()
print(d['value'])
for k,v in d.get('variants',{}).items(): print(k, round(v['value'],1), {a:round(b,1) for a,b in v['layers_eff_tflops'].items()}, v.get('roofline',{}).get('frac'))
PY
