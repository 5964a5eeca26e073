# Evidence after NEXT row N4: smoke, full GPU tests, default bench (all variants), reference arm,
# ncu --set full of the 16-bit tcgen05 kernel (fp16, 4 layers), launch list of the fp16 step.
mkdir -p gpurun_out
TAG=${1:-r01d}
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1; echo smoke rc=$?
timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu_$TAG.log 2>&1; echo pytest rc=$?; tail -2 gpurun_out/pytest_gpu_$TAG.log
timeout 900 python bench.py --out gpurun_out/bench_$TAG.json > gpurun_out/bench_$TAG.log 2>&1; echo bench rc=$?
timeout 900 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_ref_$TAG.json 2>gpurun_out/bench_ref_$TAG.log; echo ref rc=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:fused_tc16 -s 0 -c 4 -o gpurun_out/full_fp16_$TAG python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-variants --variant fp16 > /dev/null 2>&1; echo ncu-fp16 rc=$?
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/launches_fp16_$TAG.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-variants --variant fp16 > /dev/null 2>&1; echo ncu-launch rc=$?
