#!/usr/bin/env python
"""bench.py -- effective TFLOPS of the fused Winograd F(2x2,3x3) path on B200.

Metric (BASELINE.json): effective TFLOPS = 2*N*K*C*H*W*9 / t (direct-conv
equivalent) and % of FP32 peak, per ResNet 3x3 layer, at 1/2/4/8 GPUs.

One *step* = one pass of the whole hot path (FTF kernel + fused
ITF/GEMM/OTF kernel) over every layer of the workload.  The default workload is
all four ResNet 3x3 layers (BASELINE configs[1..4]: conv5_x N=32, conv4_x N=64,
conv3_x N=128, conv2_x N=256) at their global batch; with --gpus P each rank
takes a contiguous N/P batch shard of every layer (strong scaling: total work
fixed), the transformed filter is broadcast once from rank 0 with NCCL at setup,
and there is no collective on the conv path.  Time = max over ranks of CUDA-event
device time; L2 is flushed (512 MiB write) before every timed step, outside the
events.

Prints ONE JSON line (rank 0).  `--impl reference` times the CPU fp64 oracle
(test infrastructure) on a bounded sample of the same workload instead.
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


def _init_dist(backend="nccl"):
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world > 1 and torch.cuda.is_available():
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


def _max_over_ranks(v: float, world: int, device) -> float:
    if world == 1:
        return v
    t = torch.tensor([v], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def _oracle_sample(layers, target_s_per_layer: float):
    """Time the fp64 oracle's direct conv (Eq. 4) on a K-slice of every layer, the slice
    sized for about target_s_per_layer seconds; returns (flops, seconds, description)."""
    import oracle
    total_flops, total_s, desc = 0, 0.0, []
    for cfg in layers:
        x, w = make_inputs(cfg)
        per_k = 18 * cfg.N * cfg.C * cfg.H * cfg.W
        t0 = time.perf_counter()
        oracle.direct_conv(x, w[..., :1].contiguous())
        t1 = time.perf_counter() - t0
        ks = int(max(1, min(cfg.K, target_s_per_layer / max(t1, 1e-6))))
        t0 = time.perf_counter()
        oracle.direct_conv(x, w[..., :ks].contiguous())
        dt = time.perf_counter() - t0
        total_flops += per_k * ks
        total_s += dt
        desc.append(f"{cfg.name}: k 0..{ks - 1} of {cfg.K}")
    return total_flops, total_s, "; ".join(desc)


def run_reference(args, layers, rank, world):
    """--impl reference: the CPU fp64 oracle, as it stands, on a bounded sample."""
    if rank != 0:
        return None
    import oracle
    cores = oracle.num_threads()
    # calibrate the per-layer K-slice once, then time warmup + steps with that slice
    slices = []
    for cfg in layers:
        x, w = make_inputs(cfg)
        t0 = time.perf_counter()
        oracle.direct_conv(x, w[..., :1].contiguous())
        t1 = time.perf_counter() - t0
        slices.append((cfg, x, w[..., :int(max(1, min(cfg.K, args.ref_step_s / len(layers) / max(t1, 1e-6))))]
                       .contiguous()))
    flops_step = sum(18 * c.N * c.C * c.H * c.W * wk.shape[3] for c, _, wk in slices)
    for _ in range(args.warmup):
        for c, x, wk in slices:
            oracle.direct_conv(x, wk)
    t0 = time.perf_counter()
    for _ in range(args.steps):
        for c, x, wk in slices:
            oracle.direct_conv(x, wk)
    dt = time.perf_counter() - t0
    value = flops_step * args.steps / dt / 1e12
    sample = "; ".join(f"{c.name}: k 0..{wk.shape[3] - 1} of {c.K} (direct fp64, Eq. 4)" for c, _, wk in slices)
    return {
        "impl": "reference", "metric": METRIC, "value": value, "unit": "TFLOPS", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": dt / args.steps * 1e3,
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
        "l2": "flushed before every timed step by a 512 MiB write + 256 MiB read (outside the events)",
        "step": "per layer: FTF + fused ITF/16xGEMM/OTF kernel (FTFs on a side stream, each conv waits for "
                "its own FTF; fp32: all layers' FTFs in one wino_filter_transform_multi launch, convs through "
                "wino_conv2d_f2x3_fwd_ws with a stream-K workspace, the planner picks regular / split-C / "
                "stream-K + fixup per layer); the whole step replayed from one CUDA graph",
    }


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--workload", default="resnet_3x3", choices=["resnet_3x3", *RESNET_LAYERS, "tiny"])
    ap.add_argument("--variant", default="fp32", choices=["fp32", "tf32", "3xtf32", "f4_fp32", "fp32_nchw",
                                                            "nonfused_fp32", "nonfused_tf32", "fp16", "bf16"])
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-variants", action="store_true", help="skip timing the other kernel variants")
    ap.add_argument("--dist-backend", default="nccl", choices=["nccl", "gloo"],
                    help="gloo only to exercise the multi-rank logic with several ranks on one GPU")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-baseline-s", type=float, default=3.0, help="oracle seconds per layer")
    ap.add_argument("--ref-step-s", type=float, default=4.0, help="oracle seconds per reference step")
    ap.add_argument("--out", default=None)
    ap.add_argument("--shard-of", type=int, default=0,
                    help="diagnostic: on one process / GPU, run rank 0's batch shard of a P-rank job (the per-rank "
                         "step of --gpus P); not a bench line (the JSON is marked 'diagnostic')")
    args = ap.parse_args()
    if args.warmup < 3 and args.impl == "ours":
        print("warning: --warmup < 3 violates the timing rules; using 3", file=sys.stderr)
        args.warmup = 3

    rank, world, local = _init_dist(args.dist_backend)
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
        d = {"cfg": cfg, "n": n_loc, "x": xs.to(dev), "w": w.to(dev),
             "y": torch.empty((cfg.K, cfg.H, cfg.W, max(n_loc, 1)), dtype=torch.float32, device=dev)}
        if args.impl == "ours" and not args.no_e2e:
            d["x_h"] = xs.pin_memory()
            d["w_h"] = w.pin_memory()
            d["y_h"] = torch.empty((cfg.K, cfg.H, cfg.W, max(n_loc, 1)), dtype=torch.float32).pin_memory()
        per.append(d)
    flush = torch.empty(L2_FLUSH_BYTES // 4, dtype=torch.float32, device=dev)
    flush_rd = torch.ones(L2_FLUSH_BYTES // 8, dtype=torch.float32, device=dev)

    def flush_l2(v):
        # write > L2 (126 MB), then read another 256 MiB so the dirty lines are written
        # back here, outside the timed events, instead of inside the first timed kernel
        flush.fill_(v)
        flush_rd.sum()
    mk = lambda: torch.cuda.Event(enable_timing=True)  # noqa: E731

    def measure(variant, sample_clocks):
        """Warm up, capture the step in a CUDA graph, time args.steps replays (L2 flushed
        before each, outside the events), then a per-layer breakdown.  Max over ranks."""
        f4 = variant == "f4_fp32"  # NEXT row N1: fused F(4x4,3x3), FTF4 + one fused launch per layer
        tc = variant in ("tf32", "3xtf32")
        nchw = variant == "fp32_nchw"  # NEXT row N2: NCHW / KCRS front end (Sec. 8.4)
        nonfused = variant in ("nonfused_fp32", "nonfused_tf32")  # NEXT row N3: ITF -> 16 cuBLAS GEMMs -> OTF
        half = variant in ("fp16", "bf16")  # NEXT row N4: 16-bit x, w, y on tcgen05 kind::f16 (Sec. 8.3)
        if f4:  # FTF4 + conv (+ a stream-K fixup where the planner takes it: counted as taken)
            launches = sum(3 for d in per if d["n"] > 0)
        elif half:  # FTF + conv (+ stream-K fixup with the workspace, variant 5 plans it)
            launches = sum(1 + wino.plan(d["n"], d["cfg"].C, d["cfg"].H, d["cfg"].W, d["cfg"].K, variant=5).launches
                           for d in per if d["n"] > 0)
        elif nchw:  # FTF, transpose, conv (+ stream-K fixup), transpose
            launches = sum(3 + wino.plan(d["n"], d["cfg"].C, d["cfg"].H, d["cfg"].W, d["cfg"].K, variant=4).launches
                           for d in per if d["n"] > 0)
        elif nonfused:
            launches = sum(3 for d in per if d["n"] > 0)  # FTF, ITF, OTF (the GEMMs are cuBLAS kernels)
        else:
            # fp32: with the stream-K workspace (variant 4 plans it), which may add a fixup launch
            vid = {"fp32": 4, "tf32": 6, "3xtf32": 7}[variant]  # plans with the stream-K workspaces
            launches = sum((1 if variant != "fp32" else 0) +
                           wino.plan(d["n"], d["cfg"].C, d["cfg"].H, d["cfg"].W, d["cfg"].K, variant=vid).launches
                           for d in per if d["n"] > 0) + (1 if variant == "fp32" else 0)  # fp32: one batched FTF
        for d in per:
            # transformed filter: computed on rank 0, broadcast once over NVLink (NCCL)
            if f4:
                d["u"] = torch.empty((d["cfg"].C, 6, 6, d["cfg"].K), dtype=torch.float32, device=dev)
                c = d["cfg"]
                d["ws_f4"] = torch.empty(max(wino.f4_workspace_bytes(max(d["n"], 1), c.C, c.H, c.W, c.K), 16),
                                         dtype=torch.uint8, device=dev)
                if rank == 0:
                    wino.filter_transform_f4(d["w"], out=d["u"])
                if world > 1:
                    dist.broadcast(d["u"], src=0)
            elif tc:
                d["u"] = wino.filter_transform_tc(d["w"], variant)
                c = d["cfg"]
                d["ws_tc"] = torch.empty(max(wino.tc_workspace_bytes(max(d["n"], 1), c.C, c.H, c.W, c.K), 16),
                                         dtype=torch.uint8, device=dev)
                if world > 1:
                    dist.broadcast(d["u"].data, src=0)
            elif half:
                # the synthetic fp32 inputs stored in the 16-bit type at setup (outside the timed region)
                dt16 = torch.float16 if variant == "fp16" else torch.bfloat16
                d["x16"], d["w16"] = d["x"].to(dt16), d["w"].to(dt16)
                d["y16"] = torch.empty(d["y"].shape, dtype=dt16, device=dev)
                d["u"] = wino.filter_transform_half(d["w16"])
                c = d["cfg"]
                d["ws16"] = torch.empty(max(wino.half_workspace_bytes(max(d["n"], 1), c.C, c.H, c.W, c.K), 16),
                                        dtype=torch.uint8, device=dev)
                if world > 1:
                    dist.broadcast(d["u"].data, src=0)
            elif nonfused:
                c = d["cfg"]
                d["u"] = torch.empty((c.C, 4, 4, c.K), dtype=torch.float32, device=dev)
                d["ws_nf"] = torch.empty(wino.nonfused_workspace_bytes(max(d["n"], 1), c.C, c.H, c.W, c.K),
                                         dtype=torch.uint8, device=dev)
                if rank == 0:
                    wino.filter_transform(d["w"], out=d["u"])
                if world > 1:
                    dist.broadcast(d["u"], src=0)
            elif nchw:
                # layout change of the synthetic inputs at setup (outside the timed region)
                d["x_nchw"] = d["x"].permute(3, 0, 1, 2).contiguous()
                d["w_kcrs"] = d["w"].permute(3, 0, 1, 2).contiguous()
                d["y_nchw"] = torch.empty((max(d["n"], 1), d["cfg"].K, d["cfg"].H, d["cfg"].W),
                                          dtype=torch.float32, device=dev)
                d["u"] = torch.empty((d["cfg"].C, 4, 4, d["cfg"].K), dtype=torch.float32, device=dev)
                c = d["cfg"]
                # workspace of the transpose -> CHWN fused kernel -> transpose path (DESIGN 7.8)
                d["ws_nchw"] = torch.empty(wino.nchw_workspace_bytes(max(d["n"], 1), c.C, c.H, c.W, c.K),
                                           dtype=torch.uint8, device=dev)
                wino.filter_transform_kcrs(d["w_kcrs"], out=d["u"])
            else:
                d["u"] = torch.empty((d["cfg"].C, 4, 4, d["cfg"].K), dtype=torch.float32, device=dev)
                c = d["cfg"]
                # device workspace of the stream-K plan (wino_conv2d_f2x3_fwd_ws; the planner decides)
                d["ws_sk"] = torch.empty(max(wino.conv_workspace_bytes(max(d["n"], 1), c.C, c.H, c.W, c.K), 16),
                                         dtype=torch.uint8, device=dev)
                if rank == 0:
                    wino.filter_transform(d["w"], out=d["u"])
                if world > 1:
                    dist.broadcast(d["u"], src=0)

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

        side = torch.cuda.Stream(dev)

        def step():
            # The layers' filter transforms (a1) do not depend on the convolutions, so they run
            # on a side stream: FTF of layer l+1 overlaps conv l (the persistent conv grids
            # leave SMs free at small per-rank batches).  conv l waits for its own FTF only.
            fork = torch.cuda.Event()
            fork.record(stream)
            side.wait_event(fork)
            ready = []
            if variant == "fp32":
                # every layer's FTF in one launch (wino_filter_transform_multi): one launch latency
                wino.filter_transform_multi([(d["w"], d["u"]) for d in per if d["n"] > 0], stream=side)
                ev = torch.cuda.Event()
                ev.record(side)
                ready = [ev] * len(per)
            else:
                for d in per:
                    run_layer(d, conv=False, ftf_stream=side)
                    ev = torch.cuda.Event()
                    ev.record(side)
                    ready.append(ev)
            for d, ev in zip(per, ready):
                stream.wait_event(ev)
                run_layer(d, ftf=False)

        for _ in range(args.warmup):
            flush_l2(1.0)
            step()
        torch.cuda.synchronize()
        # The timed step is replayed from a CUDA graph (captured once, after warm-up):
        # host launch latency stays out of the device timeline, as in a serving loop.
        g_step = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g_step):
            step()
        g_layer = []
        for d in per:
            gf, gc = torch.cuda.CUDAGraph(), torch.cuda.CUDAGraph()
            with torch.cuda.graph(gf):
                run_layer(d, conv=False)
            with torch.cuda.graph(gc):
                run_layer(d, ftf=False)
            g_layer.append((gf, gc))
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

        # per-layer breakdown (same graphs split per kernel, L2 flushed before each layer)
        lay_ev = [[[mk(), mk(), mk()] for _ in per] for _ in range(args.steps)]
        for s in range(args.steps):
            for i, (gf, gc) in enumerate(g_layer):
                flush_l2(float(s))
                e0, e1, e2 = lay_ev[s][i]
                e0.record(stream)
                gf.replay()
                e1.record(stream)
                gc.replay()
                e2.record(stream)
        torch.cuda.synchronize()
        ftf_ms, conv_ms = [0.0] * len(per), [0.0] * len(per)
        for s in range(args.steps):
            for i, d in enumerate(per):
                if d["n"] == 0:
                    continue
                e0, e1, e2 = lay_ev[s][i]
                ftf_ms[i] += e0.elapsed_time(e1) / args.steps
                conv_ms[i] += e1.elapsed_time(e2) / args.steps
        return {"ms_step": _max_over_ranks(ms_step, world, dev),
                "conv_ms": [_max_over_ranks(v, world, dev) for v in conv_ms],
                "ftf_ms": [_max_over_ranks(v, world, dev) for v in ftf_ms],
                "launches": launches, "wall": wall, "clocks": clocks}

    main_m = measure(args.variant, sample_clocks=True)
    others = {}
    if not args.no_variants:
        for v in ("fp32", "tf32", "3xtf32", "f4_fp32", "fp32_nchw", "nonfused_fp32", "nonfused_tf32", "fp16", "bf16"):
            if v == "f4_fp32" and any(d["n"] % 16 for d in per if d["n"]):
                continue  # the F(4x4) kernel needs N % 16 == 0 per rank
            if v != args.variant:
                others[v] = measure(v, sample_clocks=False)
    ms_step, conv_ms, ftf_ms = main_m["ms_step"], main_m["conv_ms"], main_m["ftf_ms"]
    launches_per_step, wall, clocks = main_m["launches"], main_m["wall"], main_m["clocks"]

    # ---- e2e: the public C-ABI host entry point, host buffers, copies in the timed region ----
    e2e = None
    if not args.no_e2e:
        # layers are independent: order them so the largest transfer is neither first nor last
        # (copy-in of layer l+1 and copy-out of layer l-1 then overlap its compute on PCIe)
        order = sorted((d for d in per if d["n"]), key=lambda d: d["x_h"].numel())
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
        h2d = sum(d["x_h"].numel() * 4 + d["w_h"].numel() * 4 for d in per if d["n"]) * world
        d2h = sum(d["y_h"].numel() * 4 for d in per if d["n"]) * world
        total_flops = sum(c.eff_flops for c in layers)
        e2e = {"value": total_flops / (e_ms * 1e-3) / 1e12, "unit": "TFLOPS", "ms_per_step": e_ms,
               "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h,
               "api": "wino_conv2d_f2x3_fwd_host_multi (pinned host x,w -> H2D | FTF+fused FP32 conv | D2H, "
                      "copy/compute overlapped on library streams)"}

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
        eff = c.eff_flops / (conv_ms[i] * 1e-3) / 1e12
        ew = _ewmm_flops(c, args.variant)
        ewmm_flops += ew
        conv_total_ms += conv_ms[i]
        layer_rep[c.name] = {
            "conv_us": conv_ms[i] * 1e3, "ftf_us": ftf_ms[i] * 1e3,
            "eff_tflops": eff, "pct_fp32_peak_eff": 100 * eff / fp32_peak,
            "ffma_pipe_pct": 100 * ew / (conv_ms[i] * 1e-3) / 1e12 / fp32_peak,
            "eff_tflops_incl_ftf": c.eff_flops / ((conv_ms[i] + ftf_ms[i]) * 1e-3) / 1e12,
        }
    achieved = ewmm_flops / (conv_total_ms * 1e-3) / 1e12
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
        "layers": layer_rep,
        "roofline": {"bound": "alu", "kernel": f"wino fused_{args.variant}", "achieved": achieved,
                     "peak": fp32_peak, "unit": "TFLOP/s", "frac": achieved / fp32_peak, "traffic": traffic,
                     "achieved_def": "EWMM flops 32*K*C*N*ceil(H/2)*ceil(W/2) per launch summed over layers / "
                                     "summed CUDA-event conv durations",
                     "peak_def": FP32_PEAK_NOTE},
        "gpu_launches": launches_per_step * args.steps,
        "clocks": clocks, "wall_s_timed_region": wall,
    }
    if e2e:
        res["e2e"] = e2e
    tf32_peak = _tf32_peak()
    vrep = {}
    for v, m in others.items():
        val = total_eff / (m["ms_step"] * 1e-3) / 1e12
        vrep[v] = {"value": val, "ms_per_step": m["ms_step"], "pct_fp32_peak_eff": 100 * val / fp32_peak,
                   "layers_eff_tflops": {d["cfg"].name: d["cfg"].eff_flops / (m["conv_ms"][i] * 1e-3) / 1e12
                                         for i, d in enumerate(per) if d["n"]},
                   "tolerance": {"fp32": 1e-4, "tf32": 5e-3, "3xtf32": 1e-4, "f4_fp32": 1e-4, "fp32_nchw": 1e-4,
                                 "nonfused_fp32": 1e-4, "nonfused_tf32": 5e-3, "fp16": 5e-3, "bf16": 3e-2}[v]}
        if v == "nonfused_tf32":
            vrep[v]["note"] = ("NEXT row N3 ablation with tensor-core GEMMs: ITF kernel -> V workspace, 16 "
                               "strided-batched cuBLAS GEMMs in TF32 tensor-op math -> OTF kernel")
        if v == "nonfused_fp32":
            vrep[v]["note"] = ("NEXT row N3 ablation: ITF kernel -> V workspace, 16 strided-batched cuBLAS "
                               "SGEMMs (pedantic FP32) -> OTF kernel; FTF as in the fused step")
        if v == "fp32_nchw":
            ach = sum(_ewmm_flops(d["cfg"], "fp32") for d in per if d["n"]) / (sum(m["conv_ms"]) * 1e-3) / 1e12
            vrep[v]["roofline"] = {"bound": "alu", "achieved": ach, "peak": fp32_peak, "unit": "TFLOP/s",
                                   "frac": ach / fp32_peak,
                                   "achieved_def": "EWMM flops 32*K*C*N*ceil(H/2)*ceil(W/2) / conv time (NCHW)"}
        if v == "f4_fp32":
            ach = sum(_ewmm_flops(d["cfg"], v) for d in per if d["n"]) / (sum(m["conv_ms"]) * 1e-3) / 1e12
            vrep[v]["roofline"] = {"bound": "alu", "achieved": ach, "peak": fp32_peak, "unit": "TFLOP/s",
                                   "frac": ach / fp32_peak,
                                   "achieved_def": "F(4x4) EWMM flops 72*K*C*N*ceil(H/4)*ceil(W/4) / conv time"}
        if v in ("tf32", "3xtf32"):
            ach = ewmm_flops / (sum(m["conv_ms"]) * 1e-3) / 1e12
            mult = 3 if v == "3xtf32" else 1
            vrep[v]["roofline"] = {"bound": "tensor", "achieved": ach * mult, "peak": tf32_peak,
                                   "unit": "TFLOP/s", "frac": ach * mult / tf32_peak,
                                   "achieved_def": f"{mult} x EWMM flops (tcgen05 kind::tf32 work) / conv time",
                                   "peak_def": "MEASURED_PEAKS bf16_tflops x 0.5 (nominal tf32:bf16 dense ratio)"}
        if v in ("fp16", "bf16"):
            ach = ewmm_flops / (sum(m["conv_ms"]) * 1e-3) / 1e12
            vrep[v]["note"] = ("NEXT row N4: x, w, y stored in " + v + "; FP32 transforms and accumulation, "
                               "tcgen05 kind::f16 Winograd-domain GEMM")
            vrep[v]["roofline"] = {"bound": "tensor", "achieved": ach, "peak": _bf16_peak(), "unit": "TFLOP/s",
                                   "frac": ach / _bf16_peak(),
                                   "achieved_def": "EWMM flops 32*K*C*N*ceil(H/2)*ceil(W/2) (kind::f16 work) / "
                                                   "conv time",
                                   "peak_def": "MEASURED_PEAKS bf16_tflops (fp16 and bf16 share the dense rate)"}
    if vrep:
        res["variants"] = vrep
    if world == 1 and not args.no_cpu_baseline:
        import oracle
        fl, sec, sample = _oracle_sample(layers, args.cpu_baseline_s)
        res["cpu_baseline"] = {"value": fl / sec / 1e12, "unit": "TFLOPS", "cores": oracle.num_threads(),
                               "kind": "oracle", "sample": f"direct fp64 conv (Eq. 4) on {sample}; {sec:.1f} s"}
    if args.shard_of:
        res = {"diagnostic": f"rank 0 shard of a {args.shard_of}-rank job timed alone on one GPU", "ms_per_step": ms_step,
               "projected_value_if_all_ranks_equal": total_eff / (ms_step * 1e-3) / 1e12,
               "layers_us": {k: {"conv_us": v["conv_us"], "ftf_us": v["ftf_us"]} for k, v in layer_rep.items()},
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
