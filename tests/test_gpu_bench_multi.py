"""bench.py's multi-rank path on one GPU: `bench.py --gpus 2 --dist-backend gloo` launches two ranks
itself (torch.distributed.run), each takes a contiguous batch shard, and rank 0 prints
one JSON line.  Checked: n_gpus == 2, the per-rank step times and ms_per_step == their max, the
element-wise oracle comparison the bench itself reports, the broadcast u bit-identical on both ranks,
and the two ranks' dumped outputs reassembled along N equal to the fp64 oracle (Eq. 4) of the whole
batch within the FP32 bar."""
import json
import os
import subprocess
import sys

import numpy as np
import pytest
import torch

import oracle
from synth_inputs import CONFIGS, make_inputs

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.mark.skipif(not torch.cuda.is_available(), reason="no CUDA device")
def test_bench_launches_two_ranks(tmp_path):
    dump = str(tmp_path / "y")
    cmd = [sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2", "--dist-backend", "gloo",
           "--workload", "conv3_x", "--steps", "3", "--warmup", "3", "--no-e2e", "--no-variants",
           "--no-cpu-baseline", "--dump-outputs", dump]
    env = dict(os.environ, MASTER_ADDR="127.0.0.1")
    env.pop("WORLD_SIZE", None)
    res = subprocess.run(cmd, capture_output=True, text=True, timeout=900, env=env, cwd=ROOT)
    assert res.returncode == 0, res.stderr[-3000:]
    lines = [ln for ln in res.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, res.stdout[-2000:]
    line = json.loads(lines[0])
    assert line["n_gpus"] == 2
    ranks = line["ms_per_step_ranks"]
    assert len(ranks) == 2 and line["ms_per_step"] == pytest.approx(max(ranks))
    assert line["parity"]["pass"] and line["max_rel_err"] <= 1e-4
    assert line["u_broadcast_bit_identical"] is True
    cfg = CONFIGS["conv3_x"]
    x, w = make_inputs(cfg)
    parts = [torch.load(f"{dump}.rank{r}.pt")["conv3_x"] for r in range(2)]
    y = torch.cat(parts, dim=-1).double().numpy()
    assert y.shape == (cfg.K, cfg.H, cfg.W, cfg.N)
    assert oracle.max_rel_err(y, oracle.direct_conv(x, w)) <= 1e-4
