"""World-size-2 gloo tests (CPU) of the multi-GPU orchestration:
row sharding, ncclUniqueId exchange through torch.distributed, and the
combine semantics libkde uses (per-rank raw sums S_0 gathered and summed in
rank order, divided by the GLOBAL sample size) -- checked with oracle partial
sums against the oracle estimate on the whole sample."""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, out):
    import torch
    import torch.distributed as dist

    import oracle
    import synth
    from paper_conf_sigmod_heimelkm15_b200.dist import exchange_unique_id, shard_range
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        # 1. every rank receives rank 0's ncclUniqueId bytes
        nid = exchange_unique_id()
        ids = [None] * world
        dist.all_gather_object(ids, nid)
        assert len(nid) == 128 and all(x == ids[0] for x in ids)
        # 2. each rank owns a contiguous row block and computes raw sums on it
        n, d = 4099, 3
        S = synth.make_data("gauss", n, d, seed=5)
        h = oracle.scott(S)
        lo, hi = synth.mixed_workload(S, 16, seed=6)
        off, k = shard_range(n, rank, world)
        part = oracle.estimate(S[off:off + k], h, lo, hi) * k  # S_0 of this shard
        g = [torch.zeros(len(lo), dtype=torch.float64) for _ in range(world)]
        dist.all_gather(g, torch.from_numpy(part))
        tot = np.zeros(len(lo))
        for r in range(world):  # fixed rank order, as combine_ranks_kernel
            tot += g[r].numpy()
        est = tot / n
        ref = oracle.estimate(S, h, lo, hi)
        out[rank] = float(np.max(np.abs(est - ref)))
    finally:
        dist.destroy_process_group()


def test_two_rank_gloo_combine_matches_full_estimate():
    world = 2
    port = _free_port()
    ctx = mp.get_context("spawn")
    mgr = ctx.Manager()
    out = mgr.dict()
    procs = [ctx.Process(target=_worker, args=(r, world, port, out)) for r in range(world)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(timeout=180)
        assert p.exitcode == 0
    assert len(out) == world
    for r in range(world):
        assert out[r] <= 1e-14


def _worker_bootstrap(rank, world, port, out):
    """The world > 1 host plumbing the GPU path relies on, on CPU: the strong-scaling sample
    (every rank generates exactly its contiguous shard of ONE global sample), the IPC-handle
    all-gather helper of dist.py, and libkde's host reservoir decision (identical on every rank)."""
    import torch.distributed as dist

    import bench
    import paper_conf_sigmod_heimelkm15_b200 as K
    import synth
    from paper_conf_sigmod_heimelkm15_b200.dist import all_gather_bytes
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        cfg = dict(bench.CONFIGS["c4"], n=3_000_017, d=3)
        off, k, n_global = bench.shard_of(cfg, rank, world)
        shard = synth.gaussian_clusters_rows(n_global, 3, 7, off, off + k)
        parts = [None] * world
        dist.all_gather_object(parts, shard)
        whole = synth.gaussian_clusters_rows(n_global, 3, 7, 0, n_global)
        got = all_gather_bytes(bytes([rank]) * 64)           # the kde_peer_handle exchange
        sel = K.kde_reservoir_select(99, n_global, n_global, 4096)
        sels = [None] * world
        dist.all_gather_object(sels, sel)
        out[rank] = dict(strong=bool(np.array_equal(np.concatenate(parts), whole)),
                         handles=got == [bytes([r]) * 64 for r in range(world)],
                         reservoir=all(np.array_equal(s, sels[0]) for s in sels))
    finally:
        dist.destroy_process_group()


def test_two_rank_gloo_bootstrap_shards_and_reservoir():
    world = 2
    port = _free_port()
    ctx = mp.get_context("spawn")
    mgr = ctx.Manager()
    out = mgr.dict()
    procs = [ctx.Process(target=_worker_bootstrap, args=(r, world, port, out)) for r in range(world)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(timeout=300)
        assert p.exitcode == 0
    for r in range(world):
        assert out[r]["strong"] and out[r]["handles"] and out[r]["reservoir"], out[r]
