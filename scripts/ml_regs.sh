#!/bin/bash
# Register-split grid of the multi-layer kernel (fused_fp32_ml.cuh, TEPI): compiles the kernel alone
# for each (compute, producer, epilogue) setmaxnreg budget and prints the FFMA register-bank read
# cycles (scripts/sass_bank.py) and the spills per setmaxnreg region.  CPU only (nvcc + cuobjdump).
#   bash scripts/ml_regs.sh "200 64 48" "208 56 40" ...
R=$(cd "$(dirname "$0")/.." && pwd)
T=$(mktemp -d)
echo '#include "fused_fp32_ml.cuh"' > $T/t.cu
for a in "$@"; do
  set -- $a
  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -cubin -DML_RC=$1 -DML_RP=$2 -DML_RE=$3 $EXTRA \
    -I$R/paper_conf_ppopp_yanwc20_b200/csrc -I$R/include -o $T/t.cubin $T/t.cu 2>/dev/null || { echo "$a: compile failed"; continue; }
  cuobjdump -sass $T/t.cubin | awk '/Function : _ZN4wino6fp32ml20fused_fp32_ml_kernel/{f=1} /Function : _ZN4wino6fp32ml13ml_itf/{f=0} f' > $T/t.sass
  bank=$(python $R/scripts/sass_bank.py $T/t.sass | tail -1 | grep -o '([0-9.]*/FFMA)')
  spills=$(python - $T/t.sass <<'PY'
import re, sys
cur = "prologue"; cnt = {}
for l in open(sys.argv[1]):
    m = re.search(r"USETMAXREG\.(\w+)\.CTAPOOL\s+(?:UP0, )?(0x[0-9a-f]+)", l)
    if m:
        cur = f"{m.group(1).lower()} {int(m.group(2), 16)}"
        continue
    if re.search(r"\s(STL|LDL)", l):
        cnt[cur] = cnt.get(cur, 0) + 1
print(cnt or "no spills")
PY
)
  echo "compute $1 producer $2 epilogue $3: $bank $spills"
done
rm -rf $T
