"""Batch-sharded dispatch host logic on CPU: world_size 2 (and 3) over gloo.

The per-rank compute is the fp64 oracle here (the CUDA kernels are covered by
the GPU tests); what is tested is the sharding, the one-time broadcast of the
transformed filter from the source rank and the reassembly along N."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_ppopp_yanwc20_b200.dist import BatchShardedConv, gather_batch, shard_batch, shard_range


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


@pytest.mark.parametrize("n,world", [(256, 8), (32, 8), (7, 3), (1, 2), (5, 2), (0, 4)])
def test_shard_range_partitions(n, world):
    ranges = [shard_range(n, r, world) for r in range(world)]
    assert ranges[0][0] == 0 and ranges[-1][1] == n
    for (a, b), (c, d) in zip(ranges, ranges[1:]):
        assert b == c
    sizes = [b - a for a, b in ranges]
    assert max(sizes) - min(sizes) <= 1


def test_shard_range_rejects_bad():
    with pytest.raises(ValueError):
        shard_range(4, 2, 2)
    with pytest.raises(ValueError):
        shard_range(4, 0, 0)


def _oracle_ftf(w):
    import oracle
    return torch.from_numpy(oracle.filter_transform(w)).to(torch.float32)


def _oracle_conv_from_u(x, u, w_holder):
    # the oracle convolves with w; check that the broadcast u equals G w G^T of that w first
    import oracle
    assert torch.equal(u, torch.from_numpy(oracle.filter_transform(w_holder[0])).to(torch.float32))
    return torch.from_numpy(oracle.direct_conv(x, w_holder[0]))


def _worker(rank, world, port, N, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from synth_inputs import Conv3x3Config, make_inputs
        cfg = Conv3x3Config("d", N, 5, 6, 7, 6)
        x, w = make_inputs(cfg, kind="smallint")
        w_holder = [w]
        layer = BatchShardedConv(w if rank == 0 else None, cfg.C, cfg.K, src=0, ftf=_oracle_ftf,
                                 conv=lambda xl, u: _oracle_conv_from_u(xl, u, w_holder))
        y_local = layer(shard_batch(x, rank, world))
        y = gather_batch(y_local.double(), N)
        if rank == 0:
            import oracle
            q.put(bool(np.array_equal(y.numpy(), oracle.direct_conv(x, w))))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,N", [(2, 6), (2, 5), (3, 7)])
def test_batch_sharded_matches_full(world, N):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, N, q)) for r in range(world)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(timeout=180)
    assert all(p.exitcode == 0 for p in procs), [p.exitcode for p in procs]
    assert q.get(timeout=10) is True


def _worker_subgroup(rank, world, port, q):
    """Ranks 1 and 2 of 3 form a subgroup; src=0 names the subgroup's first rank (global 1)."""
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from synth_inputs import Conv3x3Config, make_inputs
        sub = dist.new_group([1, 2])
        if rank in (1, 2):
            cfg = Conv3x3Config("d", 4, 5, 6, 7, 6)
            x, w = make_inputs(cfg, kind="smallint")
            w_holder = [w]
            layer = BatchShardedConv(w if rank == 1 else None, cfg.C, cfg.K, group=sub, src=0, ftf=_oracle_ftf,
                                     conv=lambda xl, u: _oracle_conv_from_u(xl, u, w_holder))
            lr = dist.get_rank(sub)
            y_local = layer(shard_batch(x, lr, 2))
            y = gather_batch(y_local.double(), cfg.N, group=sub)
            if rank == 1:
                import oracle
                q.put(bool(np.array_equal(y.numpy(), oracle.direct_conv(x, w))))
        dist.barrier()
    finally:
        dist.destroy_process_group()


def test_batch_sharded_subgroup_src_is_group_rank():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker_subgroup, args=(r, 3, port, q)) for r in range(3)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(timeout=180)
    assert all(p.exitcode == 0 for p in procs), [p.exitcode for p in procs]
    assert q.get(timeout=10) is True
