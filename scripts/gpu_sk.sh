mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_streamk.py -q -x > gpurun_out/pytest_sk.log 2>&1; echo pytest rc=$?; tail -3 gpurun_out/pytest_sk.log
for m in none auto on; do
  timeout 600 python scripts/shard_sweep.py --sk $m --reps 30 --out gpurun_out/shard_sk_$m.json 2>&1 | grep -v Warn
done
