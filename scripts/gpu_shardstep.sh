# Per-rank bench step (the real step graph) for rank 0's shard of P = 1, 2, 4, 8 on one GPU.
mkdir -p gpurun_out
for P in 1 2 4 8; do
  timeout 600 python bench.py --shard-of $P --no-e2e --no-cpu-baseline --out gpurun_out/shardstep_$P.json > /dev/null 2>&1
  python -c "
import json; d=json.load(open('gpurun_out/shardstep_$P.json')); print($P, round(d['ms_per_step']*1e3,1), round(d['projected_value_if_all_ranks_equal'],1), {k: round(v*1e3,1) for k,v in d['variants_ms_per_step'].items()})"
done
