"""Batch-sharded multi-GPU dispatch (data parallelism over the batch N).

Eq. 4 (L177-187) never mixes images n, so the batched convolution partitions
into independent per-image problems: rank r of P takes the contiguous batch
shard n in [lo_r, hi_r) of every layer in its own dense (C,H,W,N_r) tensor and
writes (K,H,W,N_r).  The transformed filter u (16*K*C floats, L993) is computed
once on the source rank by the FTF kernel and broadcast over NVLink/NVSwitch
with one NCCL broadcast at setup; there is no collective on the conv path
(BASELINE north_star).  One process per GPU (torchrun), plumbing
through torch.distributed.

The compute callables are injectable so the host-side logic (sharding,
broadcast, gather) is testable on CPU with the gloo backend.
"""
from __future__ import annotations

from typing import Callable, Optional

import torch
import torch.distributed as dist


def shard_range(n_total: int, rank: int, world: int) -> tuple[int, int]:
    """Contiguous batch shard [lo, hi) of `rank` out of `world`; the remainder goes to the
    lowest ranks, so every rank gets floor(N/P) or ceil(N/P) images."""
    if world <= 0 or not 0 <= rank < world or n_total < 0:
        raise ValueError(f"bad shard request n={n_total} rank={rank} world={world}")
    base, rem = divmod(n_total, world)
    lo = rank * base + min(rank, rem)
    hi = lo + base + (1 if rank < rem else 0)
    return lo, hi


def shard_batch(x_chwn: torch.Tensor, rank: int, world: int) -> torch.Tensor:
    """This rank's contiguous (C,H,W,N_r) copy of the CHWN batch."""
    lo, hi = shard_range(x_chwn.shape[-1], rank, world)
    return x_chwn[..., lo:hi].contiguous()


def _default_ftf(w):
    from . import filter_transform
    return filter_transform(w)


def _default_conv(x, u):
    from . import conv2d
    return conv2d(x, u)


class BatchShardedConv:
    """One ResNet-style 3x3 layer sharded over the batch across a process group.

    >>> layer = BatchShardedConv(w, group=None, src=0)   # FTF on src + NCCL broadcast of u
    >>> y_local = layer(x_local)                          # fused Winograd on this rank's shard

    `src` is the source rank within `group` (the default group: the global rank).
    """

    def __init__(self, w_crsk: Optional[torch.Tensor], C: int, K: int, *, device=None, group=None, src: int = 0,
                 ftf: Callable = _default_ftf, conv: Callable = _default_conv):
        self.group = group
        self.world = dist.get_world_size(group) if dist.is_initialized() else 1
        self.rank = dist.get_rank(group) if dist.is_initialized() else 0
        self.conv = conv
        if self.rank == src:
            if w_crsk is None:
                raise ValueError("the source rank must supply the filter")
            self.u = ftf(w_crsk).contiguous()
        else:
            self.u = torch.empty((C, 4, 4, K), dtype=torch.float32, device=device)
        if self.world > 1:
            # src is a rank of `group` (the comparison above uses the group-local rank);
            # dist.broadcast takes a global rank
            gsrc = dist.get_global_rank(group, src) if group is not None else src
            dist.broadcast(self.u, src=gsrc, group=group)

    def __call__(self, x_local: torch.Tensor) -> torch.Tensor:
        return self.conv(x_local, self.u)


def gather_batch(y_local: torch.Tensor, n_total: int, group=None) -> torch.Tensor:
    """All-gather the per-rank (K,H,W,N_r) outputs into (K,H,W,N) (tests / parity only;
    never on the timed conv path)."""
    world = dist.get_world_size(group) if dist.is_initialized() else 1
    if world == 1:
        return y_local
    K, H, W = y_local.shape[:3]
    parts = []
    for r in range(world):
        lo, hi = shard_range(n_total, r, world)
        parts.append(torch.empty((K, H, W, hi - lo), dtype=y_local.dtype, device=y_local.device))
    # uneven shards: gather flattened, padded to the largest shard
    nmax = max(p.shape[-1] for p in parts)
    pad = torch.zeros((K, H, W, nmax), dtype=y_local.dtype, device=y_local.device)
    pad[..., :y_local.shape[-1]] = y_local
    bufs = [torch.empty_like(pad) for _ in range(world)]
    dist.all_gather(bufs, pad.contiguous(), group=group)
    return torch.cat([b[..., :p.shape[-1]] for b, p in zip(bufs, parts)], dim=-1).contiguous()
