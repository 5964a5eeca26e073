# A/B of FP32 builds in build_ab/*.so: bench step (no variants), twice each
for rep in 1 2; do
for lib in build_ab/*.so; do
  n=$(basename $lib .so)
  WINO_LIB_PATH=$PWD/$lib timeout 600 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-e2e --no-variants --out gpurun_out/ab_$n.json > /dev/null 2>&1
  python -c "
import json; d=json.load(open('gpurun_out/ab_$n.json'))
print('$n', round(d['value'],2), {k: round(v['eff_tflops'],1) for k,v in d['layers'].items()})"
done
done
