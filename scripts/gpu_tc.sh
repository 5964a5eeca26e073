mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "tc_" > gpurun_out/pytest_tc.log 2>&1; echo pytest-tc rc=$?
tail -15 gpurun_out/pytest_tc.log
for v in tf32 3xtf32; do
timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --variant $v --out gpurun_out/bench_$v.json > gpurun_out/bench_$v.log 2>&1; echo bench-$v rc=$?
python -c "
import json; d=json.load(open('gpurun_out/bench_$v.json'))
print('$v', round(d['value'],2), {k: (round(v['eff_tflops'],1), round(v['conv_us'],1)) for k,v in d['layers'].items()})" 2>&1 | tail -2
done
