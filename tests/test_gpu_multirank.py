"""World > 1 on ONE GPU: 2 and 3 processes (one rank each) share cuda:0 and run the
sharded model over the peer-memory exchange (KDE_COMM_PEER, peer.cu; fused: the scan /
reduce_splits tails push their sums into every rank's window, else a separate all-gather) -- the same
consumers the NCCL path feeds: rank-order combine of the per-box sums
(combine_ranks_kernel), Chan merge of the shard moments (moments_merge_ranks_kernel,
Scott's rule over the global sample), the rank-ordered karma index gather, and
shard-routed replacement / reservoir inserts.  Every rank's results are compared
with the fp64 oracle on the WHOLE sample.

torch.distributed (gloo) only bootstraps: it all-gathers the IPC handles."""
import os
import socket

import numpy as np
import pytest

pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _sel_ok(gpu, ora):
    return bool(np.all(np.abs(np.asarray(gpu) - ora) <= 1e-7 + 1e-5 * np.abs(ora)))


def _grad_ok(gpu, ora, scale, h, fscale=1.0):
    floor = 2.0 ** -60 / (np.sqrt(np.pi) * np.sqrt(np.log2(np.e)) * np.asarray(h)) * fscale
    return bool(np.all(np.abs(np.asarray(gpu) - ora) <= 1e-4 * np.abs(ora) + 1e-4 * scale + floor))


def _worker(rank, world, port, out, fused):
    import torch
    import torch.distributed as dist

    import oracle
    import paper_conf_sigmod_heimelkm15_b200 as K
    import synth
    from paper_conf_sigmod_heimelkm15_b200.dist import create_sharded, shard_range
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    os.environ.setdefault("KDE_PEER_TIMEOUT_S", "60")
    os.environ["KDE_PEER_FUSED"] = "1" if fused else "0"  # producer-tail push vs separate all-gather
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    res = {}
    try:
        oracle.set_threads(max(1, (os.cpu_count() or 2) // world))
        n, d = 30011, 4
        S = synth.make_data("gauss", n, d, seed=900 + world)
        off, k = shard_range(n, rank, world)
        m = create_sharded(S[off:off + k], off, n, None, transport="peer")   # Scott over the global sample
        h = m.bandwidth
        res["scott"] = bool(np.allclose(h, oracle.scott(S), rtol=1e-12, atol=0))
        res["h"] = h
        # batched (q > 1, culled full CTAs) and single-box estimates + gradients
        lo, hi = synth.mixed_workload(S, 300, seed=901)
        est_o, g_o = oracle.estimate_grad(S, h, lo, hi)
        mabs = oracle.grad_abs_scale(S, h, lo, hi)
        est, g = m.estimate(lo, hi, grad=True)
        res["batched"] = _sel_ok(est, est_o) and _grad_ok(g, g_o, mabs, h)
        res["est"] = est
        e1, g1 = m.estimate(lo[:1], hi[:1], grad=True)
        res["single"] = _sel_ok(e1, est_o[:1]) and _grad_ok(g1, g_o[:1], mabs[:1], h)
        # loss + gradient (eq. 5 / 14) with the partials combined across ranks
        p = np.clip(est_o * 1.3, 0, 1)
        L, gl = m.loss_and_grad(lo, hi, p, K.LOSS_SQUARED)
        L_o, gl_o, _ = oracle.loss_and_grad(S, h, lo, hi, p, 0, 0.0, False)
        dL = 2 * np.abs(est_o - p)
        res["loss"] = abs(L - L_o) <= 1e-6 * abs(L_o) + 1e-12 and \
            _grad_ok(gl, gl_o, (dL[:, None] * mabs).mean(axis=0), h, np.mean(dL))
        # karma: local passes, flags gathered in rank order = ascending GLOBAL indices
        tau = -1.0 / (n - 1)
        kp = K.karma_params(loss=K.LOSS_ABSOLUTE, threshold=tau)
        Ko = np.zeros(n)
        flags_ok = True
        for q in range(6):
            box_lo, box_hi = lo[10 + q], hi[10 + q]
            pt = 0.0 if q == 3 else float(est_o[10 + q]) * 0.5
            idx, nf, trunc = m.karma_update(box_lo, box_hi, pt, kp)
            c_o = oracle.contributions(S, h, box_lo, box_hi)
            thr = oracle.empty_region_threshold(h, box_lo, box_hi)[0] if pt == 0.0 else np.inf
            idx_o = oracle.karma_update(c_o, c_o.mean(), pt, K.LOSS_ABSOLUTE, 0.0, 4.0, tau, thr, Ko)
            amb = np.abs(Ko - tau) < 1e-6 / (n - 1)
            if np.isfinite(thr):
                amb |= np.abs(c_o - thr) < 1e-6 * thr
            fg = np.zeros(n, bool); fg[idx] = True
            fo = np.zeros(n, bool); fo[idx_o] = True
            flags_ok &= (not trunc) and nf == len(idx) and bool(np.all(np.diff(idx) > 0)) and \
                np.array_equal(fg[~amb], fo[~amb])
        res["karma"] = flags_ok
        res["karma_local"] = bool(np.all(np.abs(m.karma - Ko[off:off + k]) <= 1e-4 * (np.abs(Ko[off:off + k]) + 1.0 / (n - 1))))
        # truncated gather: the first idx_cap of the global ascending list
        idx_c, nf_c, tr_c = m.karma_update(lo[0], hi[0], 0.0, K.karma_params(loss=K.LOSS_ABSOLUTE, threshold=1.0),
                                           cap=7)
        res["trunc"] = tr_c and nf_c == n and np.array_equal(idx_c, np.arange(7))
        # replacement routed to the owning shard, then reservoir inserts
        rep = np.array([0, n // 3, n // 2, n - 1], np.int64)   # the same global indices on every rank
        rows = synth.make_data("gauss", len(rep), d, seed=902)
        m.replace_points(rep, rows)
        S2 = S.copy()
        S2[rep] = rows
        arrivals = synth.make_data("gauss", 5000, d, seed=903)
        n_seen, nw = m.insert_rows(arrivals, seed=77, n_seen=n)
        content = oracle.reservoir_run(77, n, n + 5000)
        newer = content > n
        S2[newer] = arrivals[content[newer] - n - 1]
        res["sample"] = bool(np.array_equal(m.sample, S2[off:off + k]))
        est2 = m.estimate(lo[:40], hi[:40])
        res["after_replace"] = _sel_ok(est2, oracle.estimate(S2, h, lo[:40], hi[:40]))
        m.close()
    except Exception as e:  # reported to the parent
        res["error"] = repr(e)
    finally:
        dist.destroy_process_group()
    out[rank] = res


@pytest.mark.parametrize("world,fused", [(2, True), (3, True), (2, False)])
def test_peer_exchange_multirank_on_one_gpu(world, fused):
    import torch
    import torch.multiprocessing as mp
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    port = _free_port()
    ctx = mp.get_context("spawn")
    mgr = ctx.Manager()
    out = mgr.dict()
    procs = [ctx.Process(target=_worker, args=(r, world, port, out, fused)) for r in range(world)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(timeout=900)
    for p in procs:
        if p.is_alive():
            p.kill()
    assert all(p.exitcode == 0 for p in procs)
    assert len(out) == world
    for r in range(world):
        res = out[r]
        assert "error" not in res, (r, res.get("error"))
        for key in ("scott", "batched", "single", "loss", "karma", "karma_local", "trunc", "sample", "after_replace"):
            assert res[key], (r, key)
    for r in range(1, world):  # every rank holds the same, deterministic combined result
        assert np.array_equal(out[r]["h"], out[0]["h"]) and np.array_equal(out[r]["est"], out[0]["est"])
