mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none -k regex:sk_fixup -s 0 -c 2 -o gpurun_out/sk_fixup python scripts/shard_sweep.py --sk on --worlds 1,8 --layers conv5_x --reps 1 > /dev/null 2>&1; echo rc=$?
timeout 600 python -m pytest tests/test_gpu_streamk.py -q -x 2>&1 | tail -2
