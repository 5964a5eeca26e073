# A/B: bench + ncu of the conv3 fused kernel for every lib in build_ab/
mkdir -p gpurun_out
for lib in build_ab/*.so; do
  n=$(basename $lib .so)
  WINO_LIB_PATH=$PWD/$lib timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --out gpurun_out/ab_$n.json > /dev/null 2>&1
  python -c "
import json; d=json.load(open('gpurun_out/ab_$n.json'))
print('$n', round(d['value'],2), {k: round(v['eff_tflops'],1) for k,v in d['layers'].items()})"
  if [ "${PROF:-0}" = "1" ]; then
    WINO_LIB_PATH=$PWD/$lib timeout 600 ncu --set full --clock-control none --import-source on -k regex:fused_fp32 -s 2 -c 1 -o gpurun_out/ab_$n python bench.py --workload conv3_x --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1
  fi
done
