mkdir -p gpurun_out
timeout 600 ncu --metrics gpu__time_duration.sum,sm__cycles_active.avg,smsp__inst_executed.sum --clock-control none --csv --log-file gpurun_out/sk_launches.csv python scripts/shard_sweep.py --sk on --worlds 1,8 --layers conv5_x --reps 1 > /dev/null 2>&1; echo rc=$?
timeout 600 ncu --metrics gpu__time_duration.sum,sm__cycles_active.avg,smsp__inst_executed.sum --clock-control none --csv --log-file gpurun_out/nosk_launches.csv python scripts/shard_sweep.py --worlds 1,8 --layers conv5_x --reps 1 > /dev/null 2>&1; echo rc=$?
