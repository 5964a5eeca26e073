# split-C / small-N parity + per-rank shard sweep + A/B of build_ab/*.so at P=1
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_split.py -x -q > gpurun_out/pytest_split.log 2>&1; echo split-tests rc=$?
tail -3 gpurun_out/pytest_split.log
python scripts/ws_trace.py conv2_x 1 2 2>&1 | head -8
python scripts/ws_trace.py conv5_x 8 4 2>&1 | head -8
timeout 600 python scripts/shard_sweep.py --variants fp32 --out gpurun_out/shard_split.json 2>&1 | tail -4
for s in 1 2 4 8; do echo "forced split $s"; timeout 300 python scripts/shard_sweep.py --variants fp32 --worlds 1,2,4,8 --split $s 2>&1 | tail -4; done
