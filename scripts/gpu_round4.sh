# Round evidence (session 3): smoke, full GPU tests, default bench, reference arm, per-rank step
# of P = 1/2/4/8 (rank 0's shard through the bench step graph), ncu launch list, ncu --set full of
# the FP32 / TF32 / FP16 fused kernels.
mkdir -p gpurun_out
TAG=${1:-r01f}
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1; echo smoke rc=$?
timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu_$TAG.log 2>&1; echo pytest rc=$?; tail -1 gpurun_out/pytest_gpu_$TAG.log
timeout 900 python bench.py --out gpurun_out/bench_$TAG.json > gpurun_out/bench_$TAG.log 2>&1; echo bench rc=$?
timeout 900 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_ref_$TAG.json 2>gpurun_out/bench_ref_$TAG.log; echo ref rc=$?
for P in 1 2 4 8; do timeout 600 python bench.py --shard-of $P --no-e2e --no-cpu-baseline --out gpurun_out/shardstep_${TAG}_$P.json > /dev/null 2>&1; echo shard $P rc=$?; done
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-variants > /dev/null 2>&1; echo ncu-launch rc=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"fused_fp32_ws|sk_fixup" -s 0 -c 6 -o gpurun_out/full_fp32_$TAG python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-variants > /dev/null 2>&1; echo ncu-fp32 rc=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"fused_tc_kernel|tc_fixup" -s 0 -c 5 -o gpurun_out/full_tf32_$TAG python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-variants --variant tf32 > /dev/null 2>&1; echo ncu-tf32 rc=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"fused_tc16|tc16_fixup" -s 0 -c 5 -o gpurun_out/full_fp16_$TAG python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-variants --variant fp16 > /dev/null 2>&1; echo ncu-fp16 rc=$?
# summarise on the box (the .ncu-rep files would exceed gpurun's 64 MiB copy-back limit)
for k in fp32 tf32 fp16; do
  python scripts/ncu_summary.py gpurun_out/full_${k}_$TAG.ncu-rep --json gpurun_out/ncu_${k}_$TAG.json > /dev/null 2>&1
  python scripts/ncu_line_stalls.py gpurun_out/full_${k}_$TAG.ncu-rep 2 40 > gpurun_out/stalls_${k}_$TAG.txt 2>&1
done
ls -la gpurun_out/*.ncu-rep; rm -f gpurun_out/full_tf32_$TAG.ncu-rep gpurun_out/full_fp16_$TAG.ncu-rep
du -sh gpurun_out
