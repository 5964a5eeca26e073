mkdir -p gpurun_out
V=${1:-fp16}
timeout 900 ncu --set full --clock-control none --import-source on -k regex:fused_tc16 -s 0 -c 4 -o gpurun_out/prof_half_$V python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-variants --variant $V > gpurun_out/ncu_half_$V.log 2>&1; echo ncu rc=$?
