# FP32 step evidence (current planner incl. stream-K): ncu --set full of every conv-path kernel of one
# bench step, and the launch list of 2 steps.
mkdir -p gpurun_out
TAG=${1:-r01e}
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"fused_fp32_ws|sk_fixup" -s 0 -c 6 -o gpurun_out/full_fp32_$TAG python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-variants > /dev/null 2>&1; echo ncu-full rc=$?
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/launches_fp32_$TAG.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-variants > /dev/null 2>&1; echo ncu-launch rc=$?
