timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k multi 2>&1 | tail -2
timeout 600 python bench.py --no-e2e --no-cpu-baseline --no-variants --out gpurun_out/bm.json > /dev/null 2>&1; python -c "
import json; d=json.load(open('gpurun_out/bm.json')); print('P1', d['value'], d['ms_per_step'], d['gpu_launches'])"
for P in 1 8; do timeout 600 python bench.py --shard-of $P --no-e2e --no-cpu-baseline --no-variants --out gpurun_out/ss_$P.json > /dev/null 2>&1; python -c "
import json; d=json.load(open('gpurun_out/ss_$P.json')); print($P, round(d['ms_per_step']*1e3,1))"; done
