mkdir -p gpurun_out
TAG=${1:-r01}
timeout 900 ncu --set full --clock-control none --import-source on -k regex:fused_fp32 -s 0 -c 4 -o gpurun_out/prof_${TAG} python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_full_${TAG}.log 2>&1; echo ncu-full rc=$?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_${TAG}.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_launch_${TAG}.log 2>&1; echo ncu-launch rc=$?
