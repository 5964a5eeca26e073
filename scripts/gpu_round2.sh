# Round evidence after split-C / small-N / NCHW work: smoke, full GPU tests, default bench,
# reference arm, ncu launch list, ncu --set full of the FP32 fused kernels (P=1 step and the
# P=8 split shards) and of the TF32 kernel.
mkdir -p gpurun_out
TAG=${1:-r01b}
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1; echo smoke rc=$?
timeout 900 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu_$TAG.log 2>&1; echo pytest rc=$?; tail -1 gpurun_out/pytest_gpu_$TAG.log
timeout 900 python bench.py --out gpurun_out/bench_$TAG.json > gpurun_out/bench_$TAG.log 2>&1; echo bench rc=$?
timeout 900 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_ref_$TAG.json 2>gpurun_out/bench_ref_$TAG.log; echo ref rc=$?
timeout 900 python scripts/shard_sweep.py --variants fp32,tf32 --out gpurun_out/shard_$TAG.json > gpurun_out/shard_$TAG.log 2>&1; echo sweep rc=$?
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-variants > /dev/null 2>&1; echo ncu-launch rc=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:fused_fp32_ws -s 0 -c 4 -o gpurun_out/full_fp32_$TAG python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-variants > /dev/null 2>&1; echo ncu-fp32 rc=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:fused_fp32_ws -s 0 -c 4 -o gpurun_out/full_fp32_p8_$TAG python scripts/shard_sweep.py --variants fp32 --worlds 8 --reps 1 > /dev/null 2>&1; echo ncu-fp32-p8 rc=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:fused_tc -s 0 -c 4 -o gpurun_out/full_tf32_$TAG python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-variants --variant tf32 > /dev/null 2>&1; echo ncu-tf32 rc=$?
ls -la gpurun_out
