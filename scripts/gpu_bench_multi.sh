mkdir -p gpurun_out
# multi-rank bench logic on ONE GPU (gloo, 2 ranks sharing cuda:0) -- correctness of the dp path only
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29511 bench.py --gpus 2 --steps 3 --warmup 3 --dist-backend gloo --no-cpu-baseline --no-variants > gpurun_out/bench_dp2_gloo.log 2>&1; echo dp2 rc=$?
tail -c 600 gpurun_out/bench_dp2_gloo.log
timeout 600 python bench.py --steps 10 --warmup 3 --out gpurun_out/bench_full.json > gpurun_out/bench_full.log 2>&1; echo bench rc=$?
python -c "
import json; d=json.load(open('gpurun_out/bench_full.json'))
print('value', round(d['value'],2), 'pct', round(d['pct_fp32_peak_eff'],1), 'e2e', round(d['e2e']['value'],2), 'cpu', d['cpu_baseline']['value'], d['cpu_baseline']['cores'])
print({k: (round(v['value'],1), v.get('roofline',{}).get('frac')) for k,v in d.get('variants',{}).items()})
print(d['clocks'])"
