#!/usr/bin/env python
"""Per-rank shard timing on ONE GPU: what each rank of a P-GPU batch-sharded run
executes (rank 0's contiguous N/P shard of every ResNet layer), timed alone with
CUDA events over CUDA-graph replays, L2 flushed before each replay.

Diagnostic for the strong-scaling behaviour of bench.py --gpus P:
predicted step time at P = sum over layers of the shard's FTF + conv time, and the
implied scaling efficiency t_1 / (P * t_P).  Not a bench number.

  python scripts/shard_sweep.py [--variants fp32,tf32] [--split S] [--out f.json]
"""
from __future__ import annotations

import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_ppopp_yanwc20_b200 as wino  # noqa: E402
from paper_conf_ppopp_yanwc20_b200.dist import shard_range  # noqa: E402
from synth_inputs import CONFIGS, make_inputs  # noqa: E402


def time_graph(fn, reps, flush):
    fn()
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        fn()
    ts = []
    for i in range(reps + 2):
        flush.fill_(float(i))
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        g.replay()
        b.record()
        torch.cuda.synchronize()
        if i >= 2:
            ts.append(a.elapsed_time(b))
    ts.sort()
    ts = ts[: max(1, len(ts) - len(ts) // 5)]  # drop the slowest fifth, average the rest
    return sum(ts) / len(ts)  # (event timestamps are ~2 us granular: a mean resolves more)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--variants", default="fp32")
    ap.add_argument("--worlds", default="1,2,4,8")
    ap.add_argument("--layers", default="conv5_x,conv4_x,conv3_x,conv2_x")
    ap.add_argument("--reps", type=int, default=10)
    ap.add_argument("--split", type=int, default=0, help="force split_c (fp32 only; 0 = planner)")
    ap.add_argument("--sk", default="none", choices=["none", "auto", "on", "off"],
                    help="fp32: pass a stream-K workspace (wino_conv2d_f2x3_fwd_ws) with this mode")
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    dev = torch.device("cuda:0")
    flush = torch.empty(512 << 18, dtype=torch.float32, device=dev)
    res = {}
    for var in a.variants.split(","):
        res[var] = {}
        for P in [int(p) for p in a.worlds.split(",")]:
            tot, rows = 0.0, {}
            for name in a.layers.split(","):
                cfg = CONFIGS[name]
                lo, hi = shard_range(cfg.N, 0, P)
                x, w = make_inputs(cfg)
                xs = x[..., lo:hi].contiguous().to(dev)
                wd = w.to(dev)
                y = torch.empty((cfg.K, cfg.H, cfg.W, hi - lo), device=dev)
                if var == "fp32":
                    u = wino.filter_transform(wd)
                    if a.sk != "none":
                        wsb = torch.zeros(wino.conv_workspace_bytes(hi - lo, cfg.C, cfg.H, cfg.W, cfg.K),
                                          dtype=torch.uint8, device=dev)
                        conv = lambda: wino.conv2d(xs, u, out=y, ws=wsb, stream_k=a.sk)  # noqa: E731
                    elif a.split:
                        conv = lambda: wino.conv2d(xs, u, out=y, split_c=a.split)  # noqa: E731
                    else:
                        conv = lambda: wino.conv2d(xs, u, out=y)  # noqa: E731
                    ftf = lambda: wino.filter_transform(wd, out=u)  # noqa: E731
                    pl = wino.plan(hi - lo, cfg.C, cfg.H, cfg.W, cfg.K, 0)
                else:
                    u = wino.filter_transform_tc(wd, var)
                    conv = lambda: wino.conv2d_tc(xs, u, out=y)  # noqa: E731
                    ftf = lambda: wino.filter_transform_tc(wd, var, out=u)  # noqa: E731
                    pl = wino.plan(hi - lo, cfg.C, cfg.H, cfg.W, cfg.K, 1 if var == "tf32" else 2)
                tc = time_graph(conv, a.reps, flush)
                tf = time_graph(ftf, a.reps, flush)
                eff = 18 * (hi - lo) * cfg.K * cfg.C * cfg.H * cfg.W / (tc * 1e-3) / 1e12
                split = a.split if (var == "fp32" and a.split) else pl.split_c
                rows[name] = {"n": hi - lo, "conv_us": tc * 1e3, "ftf_us": tf * 1e3, "eff_tflops_rank": eff,
                              "plan": {"ctas": pl.ctas // pl.split_c * split, "split_c": split,
                                       "load_x": pl.load_x}}
                tot += tc + tf
            res[var][P] = {"step_us": tot * 1e3, "layers": rows}
        t1 = res[var].get(1, {}).get("step_us")
        for P, r in res[var].items():
            if t1:
                r["scaling_eff"] = t1 / (P * r["step_us"])
            print(var, "P=%d" % P, "step %.1f us" % r["step_us"], "eff %.3f" % r.get("scaling_eff", 0),
                  {k: (v["n"], round(v["conv_us"], 1), v["plan"]["ctas"], v["plan"]["split_c"])
                   for k, v in r["layers"].items()}, flush=True)
    if a.out:
        with open(a.out, "w") as f:
            json.dump(res, f, indent=1)


if __name__ == "__main__":
    main()
