#!/usr/bin/env python
"""bench.py -- effective TFLOPS of the fused Winograd F(2x2,3x3) path on B200.

Metric (BASELINE.json): effective TFLOPS = 2*N*K*C*H*W*9 / t (direct-conv
equivalent) and % of FP32 peak, per ResNet 3x3 layer, at 1/2/4/8 GPUs.

One *step* = one pass of the whole hot path (FTF kernel + fused
ITF/GEMM/OTF kernel) over every layer of the workload.  The default workload is
all four ResNet 3x3 layers (BASELINE configs[1..4]: conv5_x N=32, conv4_x N=64,
conv3_x N=128, conv2_x N=256) at their global batch.  With --gpus P the script
launches P ranks itself (torch.distributed.run, one process per GPU, NCCL) unless
it already runs under torchrun; rank r takes a contiguous N/P batch shard of every
layer (strong scaling: total work fixed).  Every rank holds the (replicated) filter
w and runs the FTF (a1) of it inside every step; at setup rank 0's transformed
filter is broadcast once with NCCL and each rank checks its own FTF output against
it bit for bit.  There is no collective on the conv path.

Timing: the step is captured in one CUDA graph.  Headline (cold L2): L2 flushed
(512 MiB write + 256 MiB read) before every timed step, outside the events; CUDA
events on the launching stream; max over ranks.  Paper protocol (hot L2, L863):
5 repeats of 20 back-to-back replays, median of the means.  Per-kernel durations
come from timing events recorded inside a second, instrumented capture of the same
step (event nodes between kernels cost ~10 us each, so `value` replays the bare graph).
After timing, every variant's outputs are compared element by element with the
fp64 oracle (Eq. 4) on this rank's full shard: measured max_rel_err per layer.

Prints ONE JSON line (rank 0).  `--impl reference` times the CPU fp64 oracle
(test infrastructure) on the same workload instead.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import torch  # noqa: E402
import torch.distributed as dist  # noqa: E402

from paper_conf_ppopp_yanwc20_b200.dist import shard_range  # noqa: E402
from synth_inputs import CONFIGS, RESNET_LAYERS, SEED_W, SEED_X, make_inputs  # noqa: E402

FP32_PEAK_NOTE = "derived: 148 SMs x 128 FP32 lanes x 2 flop x sm_max_mhz (B200_PROFILING.md SM count, clocks.max.sm)"
L2_FLUSH_BYTES = 512 << 20
METRIC = "effective TFLOPS & % of FP32 peak per ResNet 3x3 layer at 1/2/4/8 B200"


def _peaks():
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    sm_mhz, src = 1965.0, "fallback clocks.max.sm 1965 MHz (B200_PROFILING.md)"
    hbm = 6650.0
    if os.path.exists(path):
        with open(path) as f:
            mp = json.load(f)
        sm_mhz = float(mp.get("sm_max_mhz", sm_mhz))
        hbm = float(mp.get("hbm_gbs", hbm))
        src = "MEASURED_PEAKS.json sm_max_mhz"
    fp32_tflops = 148 * 128 * 2 * sm_mhz * 1e6 / 1e12
    return fp32_tflops, hbm, src


def _bf16_peak():
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(path):
        with open(path) as f:
            return float(json.load(f).get("bf16_tflops", 1590.0))
    return 1590.0


def _tf32_peak():
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    bf16 = 1590.0
    if os.path.exists(path):
        with open(path) as f:
            bf16 = float(json.load(f).get("bf16_tflops", bf16))
    return 0.5 * bf16


def _workload(name):
    if name == "resnet_3x3":
        return [CONFIGS[n] for n in ("conv5_x", "conv4_x", "conv3_x", "conv2_x")]
    return [CONFIGS[name]]


class ClockSampler:
    """nvidia-smi sampling of SM clock and throttle reasons DURING the timed region."""

    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")

    def __init__(self, device_index: int):
        self.dev = device_index
        self.proc = None
        self.lines = []
        self._t = None

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", f"--id={self.dev}", f"--query-gpu={self.FIELDS}", "--format=csv,noheader,nounits",
                 "-lms", "100"], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except (FileNotFoundError, OSError):
            self.proc = None
            return
        self._t = threading.Thread(target=self._read, daemon=True)
        self._t.start()

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"], "samples": 0}
        time.sleep(0.15)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=2)
        except subprocess.TimeoutExpired:
            self.proc.kill()
        if self._t:
            self._t.join(timeout=1)
        sm, smax, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            parts = [p.strip() for p in ln.split(",")]
            if len(parts) < 7:
                continue
            try:
                sm.append(float(parts[0]))
                smax.append(float(parts[1]))
            except ValueError:
                continue
            for nm, v in zip(names, parts[3:7]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        sm.sort()
        return {"sm_mhz": sm[len(sm) // 2] if sm else None, "sm_max_mhz": max(smax) if smax else None,
                "reasons": sorted(reasons), "samples": len(sm)}


def _free_port() -> int:
    import socket
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _spawn_ranks(args) -> int:
    """--gpus P > 1 outside torchrun: launch this script as P ranks on this node (one process per
    GPU, the driver's own launch form) and return their exit status."""
    if args.dist_backend == "nccl":
        n = torch.cuda.device_count()
        if n < args.gpus:
            print(f"bench.py --gpus {args.gpus}: only {n} CUDA device(s) visible (one rank per GPU over NCCL)",
                  file=sys.stderr)
            return 2
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes", "1", "--nproc-per-node", str(args.gpus),
           "--master-addr", "127.0.0.1", "--master-port", str(_free_port()), os.path.abspath(__file__),
           *sys.argv[1:]]
    return subprocess.call(cmd)


def _init_dist(backend="nccl"):
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world > 1 and torch.cuda.is_available():
        if backend == "nccl" and torch.cuda.device_count() < int(os.environ.get("LOCAL_WORLD_SIZE", world)):
            raise SystemExit(f"bench.py: {world} NCCL ranks but only {torch.cuda.device_count()} GPUs visible")
        # one process per GPU; with --dist-backend gloo several ranks may share a GPU (tests)
        local = local % torch.cuda.device_count()
    if world > 1 and not dist.is_initialized():
        if not torch.cuda.is_available():
            backend = "gloo"
        if torch.cuda.is_available():
            torch.cuda.set_device(local)
        dist.init_process_group(backend=backend)
    return rank, world, local


def _ewmm_flops(c, variant):
    """Algorithmic multiply-add flops of the Winograd-domain GEMMs (Eq. 7): 2 x alpha^2 x
    K x C x N x tiles; alpha = 4 for F(2x2,3x3), 6 for F(4x4,3x3)."""
    if variant == "f4_fp32":
        return 2 * 36 * c.K * c.C * c.N * ((c.H + 3) // 4) * ((c.W + 3) // 4)
    return 32 * c.K * c.C * c.N * c.tiles


def _nonfused_bytes(c, n, planes):
    """Bytes the non-fused method must move for one layer of batch n (Sec. 9): x read, the
    Winograd-domain input V = 16 x C x NV written by the ITF and read by the GEMMs, U (16 x K x C) read,
    the Winograd-domain output M = 16 x K x NV written by the GEMMs and read by the OTF, y written."""
    nv = n * ((c.H + 1) // 2) * ((c.W + 1) // 2)
    c4 = (c.C + 3) // 4 * 4
    x = c.C * c.H * c.W * n * 4
    y = c.K * c.H * c.W * n * 4
    v = planes * 16 * c4 * nv * 4
    u = planes * 16 * c.K * c4 * 4
    m_ = 16 * c.K * nv * 4
    return x + 2 * v + u + 2 * m_ + y


def _coll_device(device):
    """Scalars for the timing / error reductions live on the GPU for NCCL, on the host for gloo."""
    return device if dist.get_backend() == "nccl" else torch.device("cpu")


def _reduce(v: float, world: int, device, op=None) -> float:
    if world == 1:
        return v
    t = torch.tensor([v], dtype=torch.float64, device=_coll_device(device))
    dist.all_reduce(t, op=op or dist.ReduceOp.MAX)
    return float(t.item())


def _gather_scalar(v: float, world: int, device) -> list:
    """Every rank's value (for the line: the max over ranks is what `value` uses)."""
    if world == 1:
        return [v]
    t = torch.tensor([v], dtype=torch.float64, device=_coll_device(device))
    out = [torch.empty_like(t) for _ in range(world)]
    dist.all_gather(out, t)
    return [float(o.item()) for o in out]


def _max_over_ranks(v: float, world: int, device) -> float:
    return _reduce(v, world, device)


def _median(xs):
    xs = sorted(xs)
    n = len(xs)
    return xs[n // 2] if n % 2 else 0.5 * (xs[n // 2 - 1] + xs[n // 2])


TOL = {"fp32": 1e-4, "tf32": 5e-3, "3xtf32": 1e-4, "f4_fp32": 1e-4, "fp32_nchw": 1e-4,
       "nonfused_fp32": 1e-4, "nonfused_tf32": 5e-3, "fp16": 5e-3, "bf16": 3e-2}
VARIANTS = ("fp32", "tf32", "3xtf32", "f4_fp32", "fp32_nchw", "nonfused_fp32", "nonfused_tf32", "fp16", "bf16")


def _oracle_step(layers, ks=None):
    """One pass of the fp64 oracle's direct conv (Eq. 4) over the workload (or over K-slices
    k < ks[i] of each layer); returns (flops, seconds)."""
    import oracle
    flops, sec = 0, 0.0
    for i, (cfg, x, w) in enumerate(layers):
        wk = w if ks is None else w[..., :ks[i]].contiguous()
        t0 = time.perf_counter()
        oracle.direct_conv(x, wk)
        sec += time.perf_counter() - t0
        flops += 18 * cfg.N * cfg.C * cfg.H * cfg.W * wk.shape[3]
    return flops, sec


def run_reference(args, layers, rank, world):
    """--impl reference: the CPU fp64 oracle (Eq. 4), as it stands, on all host cores.  A step is the
    whole workload when (warmup + steps) full passes fit the time budget, else the same K-slice of
    every layer sized to fit (the sample is stated in the line)."""
    if rank != 0:
        return None
    import oracle
    # every host core (under torchrun OMP_NUM_THREADS is 1; only rank 0 works here)
    oracle.set_num_threads(len(os.sched_getaffinity(0)))
    cores = oracle.num_threads()
    data = [(cfg, *make_inputs(cfg)) for cfg in layers]
    # calibrate with one output channel per layer
    f1, t1 = _oracle_step(data, ks=[1] * len(data))
    per_k = [18 * c.N * c.C * c.H * c.W for c, _, _ in data]
    full_flops = sum(pk * c.K for pk, (c, _, _) in zip(per_k, data))
    est_full = t1 / f1 * full_flops
    n_runs = args.steps + args.warmup
    frac = min(1.0, args.ref_budget_s / max(est_full * n_runs, 1e-9))
    ks = None if frac >= 1.0 else [max(1, min(c.K, int(c.K * frac))) for c, _, _ in data]
    for _ in range(args.warmup):
        _oracle_step(data, ks)
    tot_f, tot_s = 0, 0.0
    for _ in range(args.steps):
        f, s_ = _oracle_step(data, ks)
        tot_f += f
        tot_s += s_
    value = tot_f / tot_s / 1e12
    if ks is None:
        sample = "whole workload every step (direct fp64, Eq. 4): " + ", ".join(c.name for c, _, _ in data)
    else:
        sample = "; ".join(f"{c.name}: k 0..{k - 1} of {c.K}" for (c, _, _), k in zip(data, ks)) + \
            " (direct fp64, Eq. 4; K-slice sized to the time budget)"
    return {
        "impl": "reference", "metric": METRIC, "value": value, "unit": "TFLOPS", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": tot_s / args.steps * 1e3,
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f64",
        "data": "synthetic", "config": _config(args, layers, world),
        "cpu_baseline": {"value": value, "unit": "TFLOPS", "cores": cores, "kind": "oracle", "sample": sample},
        "e2e": {"value": value, "unit": "TFLOPS", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }


def _config(args, layers, world):
    return {
        "workload": args.workload if args.workload != "resnet_3x3" else "resnet_3x3 (conv5_x,conv4_x,conv3_x,conv2_x)",
        "layers": {c.name: {"N": c.N, "C": c.C, "K": c.K, "H": c.H, "W": c.W, "pad": 1, "stride": 1} for c in layers},
        "global_batch": {c.name: c.N for c in layers},
        "parallelism": f"dp{world} (batch-sharded, strong scaling)",
        "variant": args.variant,
        "inputs": f"uniform[-1,1) fp32, torch seeds x={SEED_X} w={SEED_W}",
        "l2": "headline: flushed before every timed step by a 512 MiB write + 256 MiB read (outside the events); "
              "hot_l2: the paper's protocol (L863), 5 repeats x 20 back-to-back replays, median of the means",
        "step": ("fp32: all layers' FTFs in one wino_filter_transform_multi launch, then every conv through "
                 "ONE wino_conv2d_f2x3_fwd_multi call (layers with < 64 tiles per SM share one persistent "
                 "stream-K launch, larger ones run alone through the planner); "
                 if args.variant == "fp32" and not args.per_layer_launches else
                 "per layer: FTF + fused ITF/16xGEMM/OTF kernel (FTFs on a side stream, each conv waits for "
                 "its own FTF; fp32: all layers' FTFs in one wino_filter_transform_multi launch, convs through "
                 "wino_conv2d_f2x3_fwd_ws with a stream-K workspace, the planner picks regular / split-C / "
                 "stream-K per layer); " + ("each layer's conv on its own stream (the layers are independent "
                 "problems), " if args.concurrent_layers else "convs in sequence on one stream, ")) +
                "the whole step replayed from one CUDA graph",
        "filter": "w replicated on every rank; each rank runs the FTF inside every step; rank 0's u broadcast "
                  "once over NCCL at setup and checked bit-identical to every rank's own FTF output",
    }


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--workload", default="resnet_3x3", choices=["resnet_3x3", *RESNET_LAYERS, "tiny"])
    ap.add_argument("--variant", default="fp32", choices=list(VARIANTS))
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-variants", action="store_true", help="skip timing the other kernel variants")
    ap.add_argument("--no-check", action="store_true", help="skip the element-wise oracle comparison")
    ap.add_argument("--per-layer-launches", action="store_true",
                    help="fp32: one conv launch per layer (wino_conv2d_f2x3_fwd_ws) instead of one "
                         "wino_conv2d_f2x3_fwd_multi call for all layers (shared persistent stream-K launch)")
    ap.add_argument("--concurrent-layers", action="store_true",
                    help="issue each layer's convolution on its own stream (the BASELINE layers are independent "
                         "problems); default: in sequence on one stream, as a network would")
    ap.add_argument("--dist-backend", default="nccl", choices=["nccl", "gloo"],
                    help="gloo only to exercise the multi-rank logic with several ranks on one GPU")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--ref-budget-s", type=float, default=120.0,
                    help="--impl reference: oracle seconds for the whole warmup + steps run")
    ap.add_argument("--out", default=None)
    ap.add_argument("--dump-outputs", default=None,
                    help="test hook: save this rank's shard outputs of the main variant to <path>.rank<r>.pt")
    ap.add_argument("--shard-of", type=int, default=0,
                    help="diagnostic: on one process / GPU, run rank 0's batch shard of a P-rank job (the per-rank "
                         "step of --gpus P); not a bench line (the JSON is marked 'diagnostic')")
    args = ap.parse_args()
    if args.warmup < 3 and args.impl == "ours":
        print("warning: --warmup < 3 violates the timing rules; using 3", file=sys.stderr)
        args.warmup = 3
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        sys.exit(_spawn_ranks(args))

    rank, world, local = _init_dist(args.dist_backend)
    if world != args.gpus:
        raise SystemExit(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={world}")
    layers = _workload(args.workload)

    if args.impl == "reference":
        res = run_reference(args, layers, rank, world)
        if rank == 0:
            print(json.dumps(res), flush=True)
        if world > 1 and dist.is_initialized():
            dist.destroy_process_group()
        return

    import paper_conf_ppopp_yanwc20_b200 as wino

    dev = torch.device(f"cuda:{local}")
    torch.cuda.set_device(dev)
    stream = torch.cuda.current_stream(dev)
    fp32_peak, hbm_peak, peak_src = _peaks()

    # ---- setup: inputs (host, full N, seeded) -> this rank's shard on device ----
    per = []
    for cfg in layers:
        lo, hi = shard_range(cfg.N, rank, world) if not args.shard_of else shard_range(cfg.N, 0, args.shard_of)
        x, w = make_inputs(cfg)
        xs = x[..., lo:hi].contiguous()
        n_loc = hi - lo
        d = {"cfg": cfg, "n": n_loc, "x_cpu": xs, "w_cpu": w, "x": xs.to(dev), "w": w.to(dev),
             "y": torch.empty((cfg.K, cfg.H, cfg.W, max(n_loc, 1)), dtype=torch.float32, device=dev)}
        if not args.no_e2e:
            d["x_h"] = xs.pin_memory()
            d["w_h"] = w.pin_memory()
            d["y_h"] = torch.empty((cfg.K, cfg.H, cfg.W, max(n_loc, 1)), dtype=torch.float32).pin_memory()
        per.append(d)
    live = [d for d in per if d["n"] > 0]

    # ---- the transformed filter: rank 0's u, broadcast once over NCCL, vs every rank's own FTF ----
    u_bcast_ok = None
    if world > 1:
        ok = True
        for d in per:
            c = d["cfg"]
            u_own = wino.filter_transform(d["w"])
            cd = _coll_device(dev)  # NCCL: over NVLink; gloo (tests): through the host
            u0 = u_own.to(cd) if rank == 0 else torch.empty(u_own.shape, dtype=u_own.dtype, device=cd)
            dist.broadcast(u0, src=0)
            ok = ok and bool(torch.equal(u0.to(dev), u_own))
        u_bcast_ok = _reduce(0.0 if ok else 1.0, world, dev) == 0.0
        if not u_bcast_ok:
            raise SystemExit("bench.py: a rank's FTF output differs from rank 0's broadcast u")

    flush = torch.empty(L2_FLUSH_BYTES // 4, dtype=torch.float32, device=dev)
    flush_rd = torch.ones(L2_FLUSH_BYTES // 8, dtype=torch.float32, device=dev)

    def flush_l2(v):
        # write > L2 (126 MB), then read another 256 MiB so the dirty lines are written
        # back here, outside the timed events, instead of inside the first timed kernel
        flush.fill_(v)
        flush_rd.sum()
    mk = lambda: torch.cuda.Event(enable_timing=True)  # noqa: E731
    mk_in_graph = lambda: torch.cuda.Event(enable_timing=True, external=True)  # noqa: E731

    def measure(variant, sample_clocks):
        """Warm up, capture the step in a CUDA graph, time args.steps replays (L2 flushed
        before each, outside the events), the per-kernel breakdown from timing events inside
        the same graph, and the paper's hot-L2 protocol.  Max over ranks."""
        f4 = variant == "f4_fp32"  # NEXT row N1: fused F(4x4,3x3), FTF4 + one fused launch per layer
        tc = variant in ("tf32", "3xtf32")
        nchw = variant == "fp32_nchw"  # NEXT row N2: NCHW / KCRS front end (Sec. 8.4)
        nonfused = variant in ("nonfused_fp32", "nonfused_tf32")  # NEXT row N3: ITF -> 16 GEMMs -> OTF
        half = variant in ("fp16", "bf16")  # NEXT row N4: 16-bit x, w, y on tcgen05 kind::f16 (Sec. 8.3)
        # fp32: every layer through one wino_conv2d_f2x3_fwd_multi call (shared persistent launch)
        multi = variant == "fp32" and not args.per_layer_launches
        if f4:  # FTF4 + conv (+ a stream-K fixup where the planner takes it: counted as taken)
            launches = sum(3 for d in live)
        elif half:  # FTF + conv (+ stream-K fixup with the workspace, variant 5 plans it)
            launches = sum(1 + wino.plan(d["n"], d["cfg"].C, d["cfg"].H, d["cfg"].W, d["cfg"].K, variant=5).launches
                           for d in live)
        elif nchw:  # FTF, transpose, conv (+ stream-K fixup), transpose
            launches = sum(3 + wino.plan(d["n"], d["cfg"].C, d["cfg"].H, d["cfg"].W, d["cfg"].K, variant=4).launches
                           for d in live)
        elif nonfused:
            launches = sum(1 + wino.nonfused_launches() for d in live)  # FTF + u arrangement, ITF, GEMM, OTF
        elif multi:  # one batched FTF + the conv launches of wino_conv2d_f2x3_fwd_multi
            launches = 1 + wino.conv_multi_launches([(d["n"], d["cfg"].C, d["cfg"].H, d["cfg"].W, d["cfg"].K)
                                                     for d in live])
        else:
            # fp32 per layer: the stream-K workspace plan (variant 4) is one launch; tf32: + a fixup launch
            vid = {"fp32": 4, "tf32": 6, "3xtf32": 7}[variant]  # plans with the stream-K workspaces
            launches = sum((1 if variant != "fp32" else 0) +
                           wino.plan(d["n"], d["cfg"].C, d["cfg"].H, d["cfg"].W, d["cfg"].K, variant=vid).launches
                           for d in live) + (1 if variant == "fp32" else 0)  # fp32: one batched FTF
        for d in per:
            c = d["cfg"]
            n1 = max(d["n"], 1)
            if f4:
                d["u"] = torch.empty((c.C, 6, 6, c.K), dtype=torch.float32, device=dev)
                d["ws_f4"] = torch.empty(max(wino.f4_workspace_bytes(n1, c.C, c.H, c.W, c.K), 16),
                                         dtype=torch.uint8, device=dev)
            elif tc:
                d["u"] = wino.filter_transform_tc(d["w"], variant)
                d["ws_tc"] = torch.empty(max(wino.tc_workspace_bytes(n1, c.C, c.H, c.W, c.K), 16),
                                         dtype=torch.uint8, device=dev)
            elif half:
                # the synthetic fp32 inputs stored in the 16-bit type at setup (outside the timed region)
                dt16 = torch.float16 if variant == "fp16" else torch.bfloat16
                d["x16"], d["w16"] = d["x"].to(dt16), d["w"].to(dt16)
                d["y16"] = torch.empty(d["y"].shape, dtype=dt16, device=dev)
                d["u"] = wino.filter_transform_half(d["w16"])
                d["ws16"] = torch.empty(max(wino.half_workspace_bytes(n1, c.C, c.H, c.W, c.K), 16),
                                        dtype=torch.uint8, device=dev)
            elif nonfused:
                d["u"] = torch.empty((c.C, 4, 4, c.K), dtype=torch.float32, device=dev)
                d["ws_nf"] = torch.empty(wino.nonfused_workspace_bytes(n1, c.C, c.H, c.W, c.K),
                                         dtype=torch.uint8, device=dev)
            elif nchw:
                # layout change of the synthetic inputs at setup (outside the timed region)
                d["x_nchw"] = d["x"].permute(3, 0, 1, 2).contiguous()
                d["w_kcrs"] = d["w"].permute(3, 0, 1, 2).contiguous()
                d["y_nchw"] = torch.empty((n1, c.K, c.H, c.W), dtype=torch.float32, device=dev)
                d["u"] = torch.empty((c.C, 4, 4, c.K), dtype=torch.float32, device=dev)
                # workspace of the transpose -> CHWN fused kernel -> transpose path (DESIGN 7.8)
                d["ws_nchw"] = torch.zeros(wino.nchw_workspace_bytes(n1, c.C, c.H, c.W, c.K),
                                           dtype=torch.uint8, device=dev)
            else:
                d["u"] = torch.empty((c.C, 4, 4, c.K), dtype=torch.float32, device=dev)
                # device workspace of the stream-K plan (wino_conv2d_f2x3_fwd_ws; the planner decides)
                d["ws_sk"] = torch.zeros(max(wino.conv_workspace_bytes(n1, c.C, c.H, c.W, c.K), 16),
                                         dtype=torch.uint8, device=dev)

        def run_layer(d, ftf=True, conv=True, ftf_stream=None):
            if d["n"] == 0:
                return
            if ftf:
                if f4:
                    wino.filter_transform_f4(d["w"], out=d["u"], stream=ftf_stream)
                elif tc:
                    wino.filter_transform_tc(d["w"], variant, out=d["u"], stream=ftf_stream)
                elif nchw:
                    wino.filter_transform_kcrs(d["w_kcrs"], out=d["u"], stream=ftf_stream)
                elif half:
                    wino.filter_transform_half(d["w16"], out=d["u"], stream=ftf_stream)
                else:
                    wino.filter_transform(d["w"], out=d["u"], stream=ftf_stream)
            if conv:
                if f4:
                    wino.conv2d_f4(d["x"], d["u"], out=d["y"], ws=d["ws_f4"])
                elif tc:
                    wino.conv2d_tc(d["x"], d["u"], out=d["y"], ws=d["ws_tc"])
                elif nchw:
                    wino.conv2d_nchw(d["x_nchw"], d["u"], out=d["y_nchw"], ws=d["ws_nchw"])
                elif half:
                    wino.conv2d_half(d["x16"], d["u"], out=d["y16"], ws=d["ws16"])
                elif nonfused:
                    wino.conv2d_nonfused(d["x"], d["u"], d["ws_nf"], out=d["y"], tf32=variant == "nonfused_tf32")
                else:
                    wino.conv2d(d["x"], d["u"], out=d["y"], ws=d["ws_sk"])

        if multi:
            ws_ml = torch.zeros(max(wino.conv_multi_workspace_bytes(
                [(d["n"], d["cfg"].C, d["cfg"].H, d["cfg"].W, d["cfg"].K) for d in live]), 16),
                dtype=torch.uint8, device=dev)
        side = torch.cuda.Stream(dev)
        lstreams = [torch.cuda.Stream(dev) for _ in per]  # one stream per (independent) layer
        # timing events recorded inside the step graph (event-record nodes): per-kernel durations
        # of the very step `value` times
        conv_ev = [(mk_in_graph(), mk_in_graph()) for _ in per]
        multi_ev = (mk_in_graph(), mk_in_graph())
        ftf_ev = (mk_in_graph(), mk_in_graph())

        def step(timed=False, concurrent=None):
            # concurrent: the layers are independent problems (BASELINE configs), so each layer's
            # conv goes on its own stream -- a layer's persistent grid starts on the SMs the previous
            # one frees in its tail instead of after its last CTA (no data dependence between them)
            concurrent = args.concurrent_layers if concurrent is None else concurrent
            # The layers' filter transforms (a1) do not depend on the convolutions, so they run
            # on a side stream: FTF of layer l+1 overlaps conv l (the persistent conv grids
            # leave SMs free at small per-rank batches).  conv l waits for its own FTF only.
            # the stream this step is issued on: inside torch.cuda.graph() that is the capture
            # stream, so the side stream joins the capture through the fork event
            cur = torch.cuda.current_stream(dev)
            fork = torch.cuda.Event()
            fork.record(cur)
            side.wait_event(fork)
            if timed:
                ftf_ev[0].record(side)
            ready = []
            if variant == "fp32":
                # every layer's FTF in one launch (wino_filter_transform_multi): one launch latency
                wino.filter_transform_multi([(d["w"], d["u"]) for d in live], stream=side)
                ev = torch.cuda.Event()
                ev.record(side)
                ready = [ev] * len(per)
            else:
                for d in per:
                    run_layer(d, conv=False, ftf_stream=side)
                    ev = torch.cuda.Event()
                    ev.record(side)
                    ready.append(ev)
            if timed:
                ftf_ev[1].record(side)
            done = []
            if multi:  # all layers' convolutions through one call; its x-only input transforms (N = 4 / 8
                # shards) are queued before its wait for the FTF event, so they overlap the FTF
                if timed:
                    multi_ev[0].record(cur)
                wino.conv2d_multi([(d["x"], d["u"], d["y"]) for d in live], ws_ml, u_ready=ready[0])
                if timed:
                    multi_ev[1].record(cur)
            for d, ev, (ea, eb), ls in zip(per, ready if not multi else [], conv_ev, lstreams):
                st = ls if concurrent else cur
                if concurrent:
                    st.wait_event(fork)
                st.wait_event(ev)
                with torch.cuda.stream(st):
                    if timed:
                        ea.record(st)
                    run_layer(d, ftf=False)
                    if timed:
                        eb.record(st)
                if concurrent:
                    e = torch.cuda.Event()
                    e.record(st)
                    done.append(e)
            for e in done:
                cur.wait_event(e)
            join = torch.cuda.Event()
            join.record(side)
            cur.wait_event(join)

        for _ in range(args.warmup):
            flush_l2(1.0)
            step()
        torch.cuda.synchronize()
        # The timed step is replayed from a CUDA graph (captured once, after warm-up):
        # host launch latency stays out of the device timeline, as in a serving loop.
        # `value` replays an uninstrumented graph: timing-event nodes between the kernels of a graph
        # were measured to add ~10 us each to the step (round 2); the per-kernel breakdown replays
        # a second, instrumented capture of the same step (layers in sequence)
        g_step = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g_step):
            step()
        g_timed = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g_timed):
            step(timed=True, concurrent=False)
        g_conv = []
        for d in per:
            gc = torch.cuda.CUDAGraph()
            with torch.cuda.graph(gc):
                run_layer(d, ftf=False)
            g_conv.append(gc)
        for _ in range(2):
            flush_l2(2.0)
            g_step.replay()
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()

        sampler = ClockSampler(local) if (rank == 0 and sample_clocks) else None
        if sampler:
            sampler.start()
            time.sleep(0.3)
        step_ev = [(mk(), mk()) for _ in range(args.steps)]
        t_wall0 = time.perf_counter()
        for s in range(args.steps):
            flush_l2(float(s))
            step_ev[s][0].record(stream)
            g_step.replay()
            step_ev[s][1].record(stream)
        torch.cuda.synchronize()
        wall = time.perf_counter() - t_wall0
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        clocks = sampler.stop() if sampler else None
        ms_step = sum(a.elapsed_time(b) for a, b in step_ev) / args.steps

        # per-kernel breakdown: the instrumented capture of the same step, the same flush
        conv_ms, ftf_ms_step, timed_ms, multi_ms = [0.0] * len(per), 0.0, 0.0, 0.0
        for s in range(args.steps):
            flush_l2(float(s))
            a, b = mk(), mk()
            a.record(stream)
            g_timed.replay()
            b.record(stream)
            torch.cuda.synchronize()
            if multi:
                multi_ms += multi_ev[0].elapsed_time(multi_ev[1]) / args.steps
            for i, d in enumerate(per):
                if d["n"] and not multi:
                    conv_ms[i] += conv_ev[i][0].elapsed_time(conv_ev[i][1]) / args.steps
            ftf_ms_step += ftf_ev[0].elapsed_time(ftf_ev[1]) / args.steps
            timed_ms += a.elapsed_time(b) / args.steps

        # the paper's protocol (L863): hot L2, 20 back-to-back launches, mean; 5 repeats, median
        def hot(g, reps=5, n=20):
            means = []
            for _ in range(reps):
                a, b = mk(), mk()
                a.record(stream)
                for _ in range(n):
                    g.replay()
                b.record(stream)
                torch.cuda.synchronize()
                means.append(a.elapsed_time(b) / n)
            return _median(means)
        hot_step = hot(g_step)
        hot_conv = [hot(gc) if d["n"] else 0.0 for gc, d in zip(g_conv, per)]
        if multi:  # per-layer breakdown: each layer alone through wino_conv2d_f2x3_fwd_ws, L2 flushed
            for s in range(args.steps):
                for i, (gc, d) in enumerate(zip(g_conv, per)):
                    if not d["n"]:
                        continue
                    flush_l2(float(s))
                    a, b = mk(), mk()
                    a.record(stream)
                    gc.replay()
                    b.record(stream)
                    torch.cuda.synchronize()
                    conv_ms[i] += a.elapsed_time(b) / args.steps
        torch.cuda.synchronize()

        # outputs of the last replay (deterministic) vs the fp64 oracle, element by element
        outs = []
        for d in per:
            if not d["n"]:
                outs.append(None)
            elif nchw:
                outs.append(d["y_nchw"].permute(1, 2, 3, 0))
            elif half:
                outs.append(d["y16"])
            else:
                outs.append(d["y"])
        return {"ms_step": _max_over_ranks(ms_step, world, dev),
                "ms_step_ranks": _gather_scalar(ms_step, world, dev),
                "conv_ms": [_max_over_ranks(v, world, dev) for v in conv_ms],
                "ftf_ms_step": _max_over_ranks(ftf_ms_step, world, dev),
                "hot_ms_step": _max_over_ranks(hot_step, world, dev),
                "hot_conv_ms": [_max_over_ranks(v, world, dev) for v in hot_conv],
                "launches": launches, "wall": wall, "clocks": clocks, "outs": outs,
                "timed_ms": _max_over_ranks(timed_ms, world, dev),
                "multi_ms": _max_over_ranks(multi_ms, world, dev) if multi else None}

    # ---- the fp64 oracle's outputs on this rank's shard (computed once per input rounding) ----
    refs, ref_time = {}, {}

    def oracle_ref(kind):
        import oracle
        if kind not in refs:
            if world > 1:
                oracle.set_num_threads(max(1, (os.cpu_count() or 1) // world))
            r, t = [], 0.0
            for d in per:
                if not d["n"]:
                    r.append(None)
                    continue
                x, w = d["x_cpu"], d["w_cpu"]
                if kind != "f32":  # R18: the oracle runs on the stored 16-bit values
                    dt16 = torch.float16 if kind == "fp16" else torch.bfloat16
                    x, w = x.to(dt16).float(), w.to(dt16).float()
                t0 = time.perf_counter()
                r.append(oracle.direct_conv(x, w))
                t += time.perf_counter() - t0
            refs[kind], ref_time[kind] = r, t
        return refs[kind]

    def errors(variant, outs):
        """max|y - y_ref| / max|y_ref| per layer, this rank's whole shard; max over ranks."""
        import numpy as np
        kind = variant if variant in ("fp16", "bf16") else "f32"
        ref = oracle_ref(kind)
        errs = {}
        for d, y, r in zip(per, outs, ref):
            if y is None:
                e = 0.0
            else:
                yd = y.double().cpu().numpy()
                den = float(np.max(np.abs(r)))
                num = float(np.max(np.abs(yd - r)))
                e = num / den if den > 0 else (0.0 if num == 0 else float("inf"))
            errs[d["cfg"].name] = _max_over_ranks(e, world, dev)
        return errs

    main_m = measure(args.variant, sample_clocks=True)
    errs_main = None if args.no_check else errors(args.variant, main_m["outs"])
    if args.dump_outputs:
        torch.save({d["cfg"].name: (o.cpu() if o is not None else None) for d, o in zip(per, main_m["outs"])},
                   f"{args.dump_outputs}.rank{rank}.pt")
    main_m["outs"] = None
    others = {}
    if not args.no_variants:
        for v in VARIANTS:
            if v == args.variant:
                continue
            m = measure(v, sample_clocks=False)
            m["errs"] = None if args.no_check else errors(v, m["outs"])
            m["outs"] = None
            others[v] = m
    ms_step, conv_ms = main_m["ms_step"], main_m["conv_ms"]
    launches_per_step, wall, clocks = main_m["launches"], main_m["wall"], main_m["clocks"]

    # ---- e2e: the public C-ABI host entry point, host buffers, copies in the timed region ----
    e2e = None
    if not args.no_e2e:
        # layers are independent: order them so the largest transfer is neither first nor last
        # (copy-in of layer l+1 and copy-out of layer l-1 then overlap its compute on PCIe)
        order = sorted(live, key=lambda d: d["x_h"].numel())
        if len(order) > 2:
            order = [order[0], order[-1]] + order[1:-1]
        hl = [(d["x_h"], d["w_h"], d["y_h"]) for d in order]
        ws = torch.empty(wino.host_multi_workspace_bytes(hl), dtype=torch.uint8, device=dev)
        for _ in range(2):
            wino.conv2d_host_multi(hl, ws)
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        e_steps = max(1, min(args.steps, 5))
        e0, e1 = mk(), mk()
        e0.record(stream)
        for _ in range(e_steps):
            wino.conv2d_host_multi(hl, ws)
        e1.record(stream)
        torch.cuda.synchronize()
        e_ms = _max_over_ranks(e0.elapsed_time(e1) / e_steps, world, dev)
        h2d = sum(d["x_h"].numel() * 4 + d["w_h"].numel() * 4 for d in live) * world
        d2h = sum(d["y_h"].numel() * 4 for d in live) * world
        total_flops = sum(c.eff_flops for c in layers)
        e2e = {"value": total_flops / (e_ms * 1e-3) / 1e12, "unit": "TFLOPS", "ms_per_step": e_ms,
               "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h,
               "api": "wino_conv2d_f2x3_fwd_host_multi (pinned host x,w -> H2D | FTF+fused FP32 conv | D2H, "
                      "copy/compute overlapped on library streams)"}

    # the oracle's full-workload time (rank 0, one rank only): the cpu_baseline
    cpu_base = None
    if world == 1 and not args.no_cpu_baseline and not args.shard_of:
        import oracle
        oracle_ref("f32")
        cpu_base = {"value": sum(c.eff_flops for c in layers) / ref_time["f32"] / 1e12, "unit": "TFLOPS",
                    "cores": oracle.num_threads(), "kind": "oracle",
                    "sample": f"the whole workload once: direct fp64 conv (Eq. 4) of every layer at its full batch "
                              f"({ref_time['f32']:.2f} s); the same run gives the reference outputs of the parity check"}

    if rank != 0:
        if world > 1:
            dist.destroy_process_group()
        return

    total_eff = sum(c.eff_flops for c in layers)
    value = total_eff / (ms_step * 1e-3) / 1e12
    layer_rep = {}
    ewmm_flops, conv_total_ms = 0, 0.0
    for i, d in enumerate(per):
        c = d["cfg"]
        if not d["n"]:
            continue
        eff = c.eff_flops / (conv_ms[i] * 1e-3) / 1e12
        eff_hot = c.eff_flops / (main_m["hot_conv_ms"][i] * 1e-3) / 1e12
        ew = _ewmm_flops(c, args.variant)
        ewmm_flops += ew
        conv_total_ms += conv_ms[i]
        layer_rep[c.name] = {
            "conv_us": conv_ms[i] * 1e3, "eff_tflops": eff, "pct_fp32_peak_eff": 100 * eff / fp32_peak,
            "ffma_pipe_pct": 100 * ew / (conv_ms[i] * 1e-3) / 1e12 / fp32_peak,
            "conv_us_hot_l2": main_m["hot_conv_ms"][i] * 1e3, "eff_tflops_hot_l2": eff_hot,
            "pct_fp32_peak_eff_hot_l2": 100 * eff_hot / fp32_peak,
        }
        if errs_main is not None:
            layer_rep[c.name]["max_rel_err"] = errs_main[c.name]
    multi_ms = main_m.get("multi_ms")
    # the dominant kernel's duration inside the step: the multi-layer launch (fp32 default) or the
    # summed per-layer conv launches
    conv_step_ms = multi_ms if multi_ms else conv_total_ms
    achieved = ewmm_flops / (conv_step_ms * 1e-3) / 1e12
    traffic = None
    tpath = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(tpath):
        try:
            with open(tpath) as f:
                tj = json.load(f)
            key = f"{args.workload}:{args.variant}:dp{world}"
            traffic = tj.get(key)
        except (OSError, ValueError):
            traffic = None

    res = {
        "metric": METRIC, "value": value, "unit": "TFLOPS", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms_step, "higher_is_better": True, "scaling": "strong",
        "vs_baseline": None, "dtype": "f32", "data": "synthetic", "config": _config(args, layers, world),
        "pct_fp32_peak_eff": 100 * value / fp32_peak,
        "fp32_peak_tflops": fp32_peak, "fp32_peak_source": f"{FP32_PEAK_NOTE}; {peak_src}",
        "hot_l2": {"value": total_eff / (main_m["hot_ms_step"] * 1e-3) / 1e12, "ms_per_step": main_m["hot_ms_step"],
                   "protocol": "L863: 20 back-to-back graph replays of the step, mean; 5 repeats, median"},
        "ftf_us_step": main_m["ftf_ms_step"] * 1e3,
        "conv_launch": ("all layers through one wino_conv2d_f2x3_fwd_multi call: " + f"{multi_ms * 1e3:.1f} us in "
                        "the instrumented step; layers.*.conv_us time each layer alone (wino_conv2d_f2x3_fwd_ws, "
                        "L2 flushed)") if multi_ms else "one launch per layer (layers.*.conv_us from the step)",
        "layers_in_step": ("concurrent: one stream per layer (independent problems), each conv waits only for "
                           "its FTF" if args.concurrent_layers else "in sequence on one stream"),
        "layers": layer_rep,
        "roofline": {"bound": "alu", "kernel": f"wino fused_{args.variant}", "achieved": achieved,
                     "peak": fp32_peak, "unit": "TFLOP/s", "frac": achieved / fp32_peak, "traffic": traffic,
                     "traffic_source": "stored, not measured in this run: ncu dram__bytes_read.sum + "
                                       "dram__bytes_write.sum of the conv launches of one step "
                                       "(profiles/traffic.json)",
                     "achieved_def": ("EWMM flops 32*K*C*N*ceil(H/2)*ceil(W/2) summed over layers / the duration of "
                                      "the wino_conv2d_f2x3_fwd_multi call (input transforms of N = 4 / 8 shards, the wait for the FTF, "
                                      "the shared persistent stream-K launch, any layer run alone) "
                                      if multi_ms else
                                      "EWMM flops 32*K*C*N*ceil(H/2)*ceil(W/2) per launch summed over layers / "
                                      "summed conv durations") +
                                     " from timing events inside an instrumented capture of the same step graph "
                                     "(L2 flushed as for value)",
                     "peak_def": FP32_PEAK_NOTE},
        "ms_per_step_ranks": main_m["ms_step_ranks"],
        "gpu_launches": launches_per_step * args.steps,
        "clocks": clocks, "wall_s_timed_region": wall,
    }
    if errs_main is not None:
        res["max_rel_err"] = max(errs_main.values()) if errs_main else 0.0
        res["parity"] = {"vs": "fp64 oracle direct conv (Eq. 4), every output element of every rank's shard",
                         "tolerance": TOL[args.variant], "pass": res["max_rel_err"] <= TOL[args.variant]}
    res["instrumented_step"] = {"ms_per_step": main_m["timed_ms"],
                                "note": "the step graph with timing-event nodes around every kernel (the source "
                                        "of the per-layer conv_us and of roofline.achieved); value uses the "
                                        "uninstrumented graph"}
    if u_bcast_ok is not None:
        res["u_broadcast_bit_identical"] = u_bcast_ok
    if e2e:
        res["e2e"] = e2e
    tf32_peak = _tf32_peak()
    vrep = {}
    for v, m in others.items():
        val = total_eff / (m["ms_step"] * 1e-3) / 1e12
        vrep[v] = {"value": val, "ms_per_step": m["ms_step"],
                   "pct_fp32_peak_eff": 100 * val / fp32_peak,
                   "hot_l2_value": total_eff / (m["hot_ms_step"] * 1e-3) / 1e12,
                   "layers_eff_tflops": {d["cfg"].name: d["cfg"].eff_flops / (m["conv_ms"][i] * 1e-3) / 1e12
                                         for i, d in enumerate(per) if d["n"]},
                   "tolerance": TOL[v]}
        if m.get("errs") is not None:
            vrep[v]["max_rel_err"] = m["errs"]
            vrep[v]["pass"] = max(m["errs"].values()) <= TOL[v]
        if v == "nonfused_tf32":
            vrep[v]["note"] = ("NEXT row N3 ablation: ITF kernel -> V workspace, 16 batched tcgen05 TF32 GEMMs "
                               "-> M workspace, OTF kernel")
        if v == "nonfused_fp32":
            vrep[v]["note"] = ("NEXT row N3 ablation: ITF kernel -> V workspace, 16 batched tcgen05 3xTF32 GEMMs "
                               "(FP32-level accuracy) -> M workspace, OTF kernel")
        if v in ("fp32_nchw", "f4_fp32", "fp32"):
            ach = sum(_ewmm_flops(d["cfg"], v) for d in live) / (sum(m["conv_ms"]) * 1e-3) / 1e12
            vrep[v]["roofline"] = {"bound": "alu", "achieved": ach, "peak": fp32_peak, "unit": "TFLOP/s",
                                   "frac": ach / fp32_peak,
                                   "achieved_def": ("F(4x4) EWMM flops 72*K*C*N*ceil(H/4)*ceil(W/4)" if v == "f4_fp32"
                                                    else "EWMM flops 32*K*C*N*ceil(H/2)*ceil(W/2)") + " / conv time"}
        if v in ("nonfused_tf32", "nonfused_fp32"):
            # the non-fused method moves its Winograd-domain operands through HBM (Sec. 9, Sec. 8.1
            # cost model): its roofline is the bytes it must move, not the tensor pipe (its GEMM runs at
            # the HBM rate, profiles/r02_nonfused_launches.csv)
            pp = 2 if v == "nonfused_fp32" else 1  # 3xTF32: big + small planes of V and U
            byt = sum(_nonfused_bytes(d["cfg"], d["n"], pp) for d in live)
            ach_b = byt / (sum(m["conv_ms"]) * 1e-3) / 1e9
            ach = sum(_ewmm_flops(d["cfg"], v) for d in live) / (sum(m["conv_ms"]) * 1e-3) / 1e12
            vrep[v]["roofline"] = {"bound": "hbm", "achieved": ach_b, "peak": hbm_peak, "unit": "GB/s",
                                   "frac": ach_b / hbm_peak,
                                   "achieved_def": "algorithmic bytes of the non-fused method per step: x read, V "
                                                   "written and read, U read, M written and read, y written "
                                                   "(V, U with 2 planes for 3xTF32) / conv time (ITF + GEMM + OTF)",
                                   "peak_def": "MEASURED_PEAKS hbm_gbs",
                                   "tensor_frac": ach * (3 if pp == 2 else 1) / tf32_peak}
        if v in ("tf32", "3xtf32"):
            ach = sum(_ewmm_flops(d["cfg"], v) for d in live) / (sum(m["conv_ms"]) * 1e-3) / 1e12
            mult = 3 if v in ("3xtf32", "nonfused_fp32") else 1
            vrep[v]["roofline"] = {"bound": "tensor", "achieved": ach * mult, "peak": tf32_peak,
                                   "unit": "TFLOP/s", "frac": ach * mult / tf32_peak,
                                   "achieved_def": f"{mult} x EWMM flops (tcgen05 kind::tf32 work) / conv time"
                                                   + (" (ITF + GEMM + OTF)" if v.startswith("nonfused") else ""),
                                   "peak_def": "MEASURED_PEAKS bf16_tflops x 0.5 (nominal tf32:bf16 dense ratio)"}
        if v in ("fp16", "bf16"):
            ach = sum(_ewmm_flops(d["cfg"], v) for d in live) / (sum(m["conv_ms"]) * 1e-3) / 1e12
            vrep[v]["note"] = ("NEXT row N4: x, w, y stored in " + v + "; FP32 transforms and accumulation, "
                               "tcgen05 kind::f16 Winograd-domain GEMM")
            vrep[v]["roofline"] = {"bound": "tensor", "achieved": ach, "peak": _bf16_peak(), "unit": "TFLOP/s",
                                   "frac": ach / _bf16_peak(),
                                   "achieved_def": "EWMM flops 32*K*C*N*ceil(H/2)*ceil(W/2) (kind::f16 work) / "
                                                   "conv time",
                                   "peak_def": "MEASURED_PEAKS bf16_tflops (fp16 and bf16 share the dense rate)"}
    if vrep:
        res["variants"] = vrep
    if cpu_base:
        res["cpu_baseline"] = cpu_base
    if args.shard_of:
        res = {"diagnostic": f"rank 0 shard of a {args.shard_of}-rank job timed alone on one GPU", "ms_per_step": ms_step,
               "instrumented_ms_per_step": main_m["timed_ms"],
               "multi_conv_us": main_m["multi_ms"] * 1e3 if main_m.get("multi_ms") else None,
               "projected_value_if_all_ranks_equal": total_eff / (ms_step * 1e-3) / 1e12,
               "layers_us": {k: {"conv_us": v["conv_us"]} for k, v in layer_rep.items()},
               "variants_ms_per_step": {k: v["ms_per_step"] for k, v in vrep.items()}}
    line = json.dumps(res)
    print(line, flush=True)
    if args.out:
        with open(args.out, "w") as f:
            f.write(line + "\n")
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
