mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "tc_" > gpurun_out/pytest_tc.log 2>&1; echo pytest-tc rc=$?; tail -2 gpurun_out/pytest_tc.log
WINO_LIB_PATH=$PWD/build_ab/libwino_mm64all.so timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "tc_" > gpurun_out/pytest_tc_mm64.log 2>&1; echo pytest-tc-mm64 rc=$?; tail -2 gpurun_out/pytest_tc_mm64.log
for lib in build_ab/*.so; do
  n=$(basename $lib .so)
  for v in tf32 3xtf32; do
  WINO_LIB_PATH=$PWD/$lib timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --no-variants --variant $v --out gpurun_out/ab_$n_$v.json > /dev/null 2>&1
  python -c "
import json; d=json.load(open('gpurun_out/ab_$n_$v.json'))
print('$n $v', round(d['value'],2), {k: round(v['eff_tflops'],1) for k,v in d['layers'].items()})"
  done
done
