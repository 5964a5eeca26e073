mkdir -p gpurun_out
TAG=r01c
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1; echo smoke rc=$?
timeout 1200 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu_$TAG.log 2>&1; echo pytest rc=$?; tail -3 gpurun_out/pytest_gpu_$TAG.log
timeout 900 python bench.py --out gpurun_out/bench_$TAG.json > gpurun_out/bench_$TAG.log 2>&1; echo bench rc=$?; tail -c 600 gpurun_out/bench_$TAG.log
