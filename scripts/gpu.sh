#!/usr/bin/env bash
# Every GPU recipe of this repo in one place (replaces round 1's 30 one-off gpu_*.sh lease scripts).
# Run on a B200 box from the repo root, e.g.
#   /usr/local/graft/bin/gpurun --timeout 1800 -- 'bash scripts/gpu.sh tests bench'
# Outputs go to gpurun_out/<TAG>_* (TAG defaults to "run"; set TAG=... to name a session).
#
#   tests        smoke() + the full GPU test suite (pytest -m gpu)
#   bench        the default bench line (all variants, e2e, cpu_baseline) + the reference arm
#   shards       bench --shard-of P for P = 1 2 4 8 (rank 0's batch shard through the step graph)
#   launches     ncu launch list (gpu__time_duration, dram bytes) of 2 bench steps (not a bench value)
#   profile V R  ncu --set full of the kernels matching regex R in one step of variant V
#                (e.g. "profile fp32 fused_fp32_ws", "profile tf32 fused_tc_kernel")
#   sanitize     compute-sanitizer memcheck + synccheck over every variant, racecheck of the
#                tcgen05 kernels (scripts/sanitize.py)
#   racerepro    racecheck on scripts/microbench/racecheck_mbar_repro.cu (both hand-off patterns)
#   stress       repeated-run exactness (tests/test_gpu_stress.py + scripts/stress_{fp32,tc}.py)
#   ab           bench + optional ncu of every A/B library in build_ab/*.so (PROF=1 for ncu)
set -u
mkdir -p gpurun_out
TAG=${TAG:-run}
O=gpurun_out/$TAG
step() { echo "== $1: rc=$2"; }

while [ $# -gt 0 ]; do
  case "$1" in
    tests)
      python -c "import __graft_entry__ as g; g.smoke()" > ${O}_smoke.log 2>&1; step smoke $?
      timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider > ${O}_pytest_gpu.log 2>&1; step pytest $?
      tail -3 ${O}_pytest_gpu.log ;;
    bench)
      timeout 900 python bench.py --out ${O}_bench.json > ${O}_bench.log 2>&1; step bench $?
      timeout 900 python bench.py --impl reference --steps 3 --warmup 1 > ${O}_bench_ref.json 2> ${O}_bench_ref.log; step reference $? ;;
    shards)
      for P in 1 2 4 8; do
        timeout 600 python bench.py --shard-of $P --no-e2e --no-cpu-baseline --no-check --out ${O}_shard$P.json > ${O}_shard$P.log 2>&1
        step shard$P $?
      done ;;
    launches)
      timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
        --csv --log-file ${O}_launches.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline \
        --no-variants --no-check > /dev/null 2>&1; step launches $? ;;
    profile)
      # the .ncu-rep stays in /tmp (gpurun copies back at most 64 MiB); summaries come back
      V=$2; R=$3; shift 2
      REP=/tmp/${TAG}_prof_$V
      timeout 900 ncu --set full --clock-control none --import-source on -k regex:"$R" -s 0 -c 8 -o $REP \
        python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-check --no-variants --variant $V \
        > ${O}_prof_$V.log 2>&1; step profile-$V $?
      python scripts/ncu_summary.py $REP.ncu-rep --json ${O}_prof_$V.json > ${O}_prof_$V.txt 2>&1
      for L in 0 1 2 3; do python scripts/ncu_line_stalls.py $REP.ncu-rep $L > ${O}_prof_${V}_lines$L.txt 2>&1; done
      [ "${KEEP_REP:-0}" = "1" ] && cp $REP.ncu-rep ${O}_prof_$V.ncu-rep ;;
    sanitize)
      for tool in memcheck synccheck; do
        timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 python scripts/sanitize.py > ${O}_$tool.log 2>&1
        step $tool $?; tail -1 ${O}_$tool.log
      done
      for part in tc half; do
        timeout 900 compute-sanitizer --tool racecheck --racecheck-report hazard --error-exitcode 9 \
          python scripts/sanitize.py $part > ${O}_racecheck_$part.log 2>&1
        step racecheck-$part $?; tail -1 ${O}_racecheck_$part.log
      done ;;
    racerepro)
      for p in 0 1; do
        nvcc -gencode arch=compute_100a,code=sm_100a -DPER_LANE=$p scripts/microbench/racecheck_mbar_repro.cu \
          -o /tmp/rc_repro$p && compute-sanitizer --tool racecheck /tmp/rc_repro$p > ${O}_racerepro$p.log 2>&1
        step racerepro$p $?; tail -1 ${O}_racerepro$p.log
      done ;;
    stress)
      timeout 1200 python -m pytest tests/test_gpu_stress.py -q -p no:cacheprovider > ${O}_stress.log 2>&1; step stress $?
      timeout 1200 python scripts/stress_fp32.py 10 > ${O}_stress_fp32.log 2>&1; step stress_fp32 $?
      timeout 1200 python scripts/stress_tc.py 10 > ${O}_stress_tc.log 2>&1; step stress_tc $? ;;
    ab)
      for lib in build_ab/*.so; do
        n=$(basename $lib .so)
        WINO_LIB_PATH=$PWD/$lib timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e \
          --no-check --out ${O}_ab_$n.json > /dev/null 2>&1; step ab-$n $?
        if [ "${PROF:-0}" = "1" ]; then
          WINO_LIB_PATH=$PWD/$lib timeout 600 ncu --set full --clock-control none --import-source on \
            -k regex:fused_fp32 -s 2 -c 1 -o ${O}_ab_$n python bench.py --workload conv3_x --steps 1 --warmup 3 \
            --no-e2e --no-cpu-baseline --no-check > /dev/null 2>&1
        fi
      done ;;
    *) echo "unknown recipe $1"; exit 2 ;;
  esac
  shift
done
