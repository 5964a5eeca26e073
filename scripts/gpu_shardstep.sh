# Per-rank step (rank 0's shard through the bench step graph) for P = 1, 2, 4, 8 on one GPU.
mkdir -p gpurun_out
TAG=${1:-final}
for P in 1 2 4 8; do
  timeout 600 python bench.py --shard-of $P --no-e2e --no-cpu-baseline --out gpurun_out/shardstep_${TAG}_$P.json > /dev/null 2>&1; echo shard $P rc=$?
done
