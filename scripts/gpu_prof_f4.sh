mkdir -p gpurun_out
TAG=${1:-f4}; WL=${2:-conv3_x}
timeout 900 ncu --set full --clock-control none --import-source on -k regex:fused_f4 -c 1 -o gpurun_out/prof_$TAG python bench.py --workload $WL --variant f4_fp32 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-variants > gpurun_out/ncu_$TAG.log 2>&1; echo ncu rc=$?
tail -3 gpurun_out/ncu_$TAG.log
