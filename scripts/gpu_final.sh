# Final evidence of the session: smoke, full GPU tests, default bench, reference arm, launch list.
mkdir -p gpurun_out
TAG=${1:-r01g}
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1; echo smoke rc=$?
timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu_$TAG.log 2>&1; echo pytest rc=$?; tail -1 gpurun_out/pytest_gpu_$TAG.log
timeout 900 python bench.py --out gpurun_out/bench_$TAG.json > gpurun_out/bench_$TAG.log 2>&1; echo bench rc=$?
timeout 900 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_ref_$TAG.json 2>gpurun_out/bench_ref_$TAG.log; echo ref rc=$?
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-variants > /dev/null 2>&1; echo ncu-launch rc=$?
