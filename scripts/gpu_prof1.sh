mkdir -p gpurun_out
TAG=$1; shift
timeout 900 ncu --set full --clock-control none --import-source on "$@" -o gpurun_out/prof_$TAG python bench.py --workload conv3_x --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-variants > gpurun_out/ncu_$TAG.log 2>&1; echo ncu rc=$?
