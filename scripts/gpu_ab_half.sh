# A/B of 16-bit tcgen05 kernel builds in build_ab/*.so (per-layer device time)
for lib in build_ab/*.so; do
  n=$(basename $lib .so)
  echo -n "$n "; WINO_LIB_PATH=$PWD/$lib PYTHONPATH=$PWD timeout 300 python scripts/half_time.py fp16 2>&1 | tail -1
done
