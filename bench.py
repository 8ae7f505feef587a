#!/usr/bin/env python
"""bench.py -- throughput of the KDE range-selectivity hot path on B200.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config c3|c2|c4|c5|...] [--impl cuda|reference]

A "step" is one pass of the hot path over one batch of synthetic input.  The
default workload is BASELINE.json configs[2] ("c3", the largest single-GPU
configuration): d = 5, N = 2^24 sample points per GPU (correlated Gaussian
clusters), a 4096-box DT/DV/UT/UV batch, estimate + loss + bandwidth gradient
(kde_loss_and_grad, eq. 5/14/17).  The same line carries the configs[2]
single-query leg ("single_query": one DT box per step, the HBM-streaming scan)
with its own roofline, so one run covers both north-star targets.

--gpus N > 1 launches N ranks itself (torch.distributed.run) unless started by
a launcher (WORLD_SIZE set, which must equal N).  c2/c3 scale weakly (N rows
per GPU); c4 (configs[3]) is STRONG scaling: one 2^28-row sample, generated
chunk-wise from one seed, split into contiguous row shards; per-box partial
sums are combined inside libkde over peer device memory (--comm peer, default)
or NCCL (--comm nccl).

value   = point*query evaluations per second over the whole job
          (N_global * q / step time, max over ranks, CUDA events, inputs
          resident in HBM, L2 flushed between timed steps when the sample fits).
e2e     = the same metric through the host-pointer C-ABI call (inputs copied
          host->device and results device->host inside the timed region).
roofline: the dominant kernel's own CUDA-event time (recorded inside libkde on
          its stream) against the SFU ceiling 148 SMs x 16 MUFU/clk x 1965 MHz /
          (2d) point*query/s (batched), or measured HBM bandwidth (single box).
cpu_baseline / --impl reference: the fp64 C oracle (oracle/) as it stands,
          on the host cores, over a bounded sample of the same workload.
"""
from __future__ import annotations

import argparse
import json
import os
import socket
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "range-KDE estimates/sec & point·query evals/sec at 1/2/4/8 B200; % HBM/SFU roofline"
SM_COUNT_NOMINAL = 148
MUFU_PER_SM_CLK = 16
SM_MAX_MHZ = 1965.0

CONFIGS = {
    # name: d, rows (per GPU, or global when strong), boxes, path, description
    "c3": dict(d=5, n=1 << 24, q=4096, path="loss_grad", data="gauss", single_leg=True,
               desc="configs[2]: d=5, N=2^24/GPU correlated Gaussian clusters, 4096-box DT/DV/UT/UV batch, "
                    "estimate + L2 loss + bandwidth gradient; single_query leg: one DT box per step"),
    "c2": dict(d=3, n=1 << 20, q=10000, path="loss_grad", data="gauss",
               desc="configs[1]: d=3, N=2^20/GPU, 10k-box batch, estimate + L2 loss + bandwidth gradient"),
    "c3s": dict(d=5, n=1 << 24, q=1, path="single", grad=False, retain=False, data="gauss",
                desc="configs[2] single box: d=5, N=2^24/GPU, one DT box per step, estimate (HBM-streaming scan)"),
    "c3sg": dict(d=5, n=1 << 24, q=1, path="single", grad=True, retain=False, data="gauss",
                 desc="configs[2] single box: d=5, N=2^24/GPU, one DT box per step, estimate + bandwidth gradient"),
    "c4": dict(d=8, n=1 << 28, q=4096, path="loss_grad", data="gauss_rows", strong=True,
               desc="configs[3]: d=8, N=2^28 GLOBAL rows (one seed) split row-wise over the GPUs (strong scaling), "
                    "4096-box batch, estimate + L2 loss + gradient, partials all-gathered + rank-order sum"),
    "c4w": dict(d=8, n=1 << 25, q=4096, path="loss_grad", data="gauss",
                desc="configs[3] per-GPU shard, weak: d=8, 2^25 rows/GPU, 4096 boxes, estimate + L2 loss + gradient"),
    "c5s": dict(d=10, n=1 << 22, q=1, path="single", grad=True, retain=True, data="gauss",
                desc="configs[4] estimate step: d=10, N=2^22/GPU, one DT box, estimate + gradient + retained "
                     "contributions (Adaptive, P:L240)"),
    "c5": dict(d=10, n=1 << 22, q=16, path="stream", grad=True, retain=True, data="stream",
               desc="configs[4] streaming: d=10, N=2^22 sample of a cluster database (3 clusters x 2^22 rows, one "
                    "new cluster inserted per cycle, the oldest deleted); one step = one 2^16-row insert chunk "
                    "through the reservoir (kde_insert_rows) + 16 DT queries, each a device-resident streaming step "
                    "(estimate + gradient + retained p^(i), karma + compaction, Listing 1 step, replacement; "
                    "kde_stream_step_dev, CUDA graphs), single GPU"),
    "c2e": dict(d=3, n=1 << 20, q=10000, path="loss_grad", data="gauss", kernel="epan",
                desc="configs[1] with the Epanechnikov product kernel (NEXT-4, reading R14): d=3, N=2^20/GPU, "
                     "10k-box batch, estimate + L2 loss + bandwidth gradient"),
    "c3se": dict(d=5, n=1 << 24, q=1, path="single", grad=False, retain=False, data="gauss", kernel="epan",
                 desc="configs[2] single box with the Epanechnikov product kernel: d=5, N=2^24/GPU, estimate"),
}


# ---------------------------------------------------------------- helpers
class ClockSampler:
    """nvidia-smi sampling of SM clocks and throttle reasons during the timed region."""
    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.proc = None
        self.lines = []

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.FIELDS}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except OSError:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def __exit__(self, *a):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except subprocess.TimeoutExpired:
                self.proc.kill()
            self.t.join(timeout=2)

    def summary(self):
        sm, mx, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            p = [x.strip() for x in ln.split(",")]
            if len(p) < 8:
                continue
            try:
                sm.append(float(p[0]))
                mx.append(float(p[1]))
            except ValueError:
                continue
            for nm, v in zip(names, p[4:8]):
                if v.lower() == "active":
                    reasons.add(nm)
        if not sm:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": [], "samples": 0}
        return {"sm_mhz": statistics.median(sm), "sm_max_mhz": max(mx), "reasons": sorted(reasons),
                "samples": len(sm)}


def shard_of(cfg, rank: int, world: int):
    """(row_offset, local rows, global rows) of this rank."""
    from paper_conf_sigmod_heimelkm15_b200.dist import shard_range
    if cfg.get("strong"):
        off, k = shard_range(cfg["n"], rank, world)
        return off, k, cfg["n"]
    return rank * cfg["n"], cfg["n"], cfg["n"] * world


def make_inputs(cfg, rank: int, world: int, seed: int = 7):
    """Seeded synthetic inputs: this rank's sample shard S, a database R whose exact box
    counts are the true selectivities, and the (replicated) boxes."""
    import synth
    d, n, q = cfg["d"], cfg["n"], cfg["q"]
    off, k, n_global = shard_of(cfg, rank, world)
    if cfg["data"] == "gauss_rows":
        # one global sample generated chunk-wise from one seed: every world size sees the same rows
        S = synth.gaussian_clusters_rows(n_global, d, seed, off, off + k)
        R = synth.gaussian_clusters_rows(1 << 22, d, seed + 1, 0, 1 << 22)   # independent draw for the truths
        Q = synth.gaussian_clusters_rows(n_global, d, seed, 0, 1 << 16)
    elif n <= (1 << 21):
        # the "database" R has 4x the rows; the sample is a without-replacement draw from it
        R = synth.make_data(cfg["data"], 4 * n, d, seed=seed + 1000 * rank)
        S = R[synth.rng(seed, 500 + rank).choice(len(R), size=n, replace=False)]
        Q = synth.make_data(cfg["data"], 1 << 16, d, seed=seed)
    else:
        # large samples: S is drawn directly; true selectivities are counted on a 2^22-row subsample
        S = synth.make_data(cfg["data"], n, d, seed=seed + 1000 * rank)
        R = S[synth.rng(seed, 600 + rank).choice(n, size=1 << 22, replace=False)]
        Q = synth.make_data(cfg["data"], 1 << 16, d, seed=seed)
    if q == 1 or cfg.get("single_leg"):
        lo1, hi1 = synth.workload(Q, 64, seed + 1, "DT")
    else:
        lo1 = hi1 = None
    if q > 1:
        lo, hi = synth.mixed_workload(Q, q, seed + 1)
    else:
        lo, hi = lo1, hi1
    return R, S, lo, hi, lo1, hi1


def true_selectivities(R, lo, hi):
    """Exact counts over R on the GPU (harness kernel kde_count_in_box_dev)."""
    import torch

    import paper_conf_sigmod_heimelkm15_b200 as K
    dR = torch.from_numpy(np.ascontiguousarray(R)).cuda()
    dlo = torch.from_numpy(lo).cuda()
    dhi = torch.from_numpy(hi).cuda()
    cnt = torch.zeros(len(lo), dtype=torch.int64, device="cuda")
    K.kde_count_in_box_dev(dR, dlo, dhi, cnt, stream=torch.cuda.current_stream())
    torch.cuda.synchronize()
    return (cnt.double() / len(R)).cpu().numpy()


def cpu_oracle_rate(S, h, lo, hi, p, path, budget_s=12.0, per_step=False):
    """The fp64 oracle as it stands on the host cores over a bounded sample:
    k boxes x the full shard.  Returns (pt*q/s, cores used, sample string, seconds)."""
    import oracle
    cores = os.cpu_count() or 1
    n = len(S)
    oracle.set_threads(1)
    t0 = time.perf_counter()
    if path in ("single", "stream"):
        oracle.estimate_grad(S, h, lo[:1], hi[:1])
    else:
        oracle.loss_and_grad(S, h, lo[:1], hi[:1], p[:1], 0, 0.0, False)
    t1 = time.perf_counter() - t0
    k = int(max(1, min(len(lo), round(budget_s * cores / max(t1, 1e-6)))))
    k = max(1, min(k, len(lo)))
    use = min(cores, k)
    oracle.set_threads(use)
    t0 = time.perf_counter()
    if path in ("single", "stream"):
        oracle.estimate_grad(S, h, lo[:k], hi[:k])
    else:
        oracle.loss_and_grad(S, h, lo[:k], hi[:k], p[:k], 0, 0.0, False)
    dt = time.perf_counter() - t0
    return k * n / dt, use, f"{k} boxes x {n} points (of {len(lo)} boxes), fp64 oracle, {use} threads", dt, k


# ---------------------------------------------------------------- reference arm (the oracle)
def run_reference(args, cfg, rank, world):
    if rank != 0:
        return
    import oracle
    oracle.build()
    if cfg["path"] == "stream":
        import synth
        sc = synth.StreamClusters(cfg["d"], 1 << 22, seed=11)
        S = np.concatenate([sc.cluster_rows(c, 0, cfg["n"] // 3 + 1) for c in range(3)])[:cfg["n"]]
        lo, hi = sc.queries([0, 1, 2], 64, seed=12)
        p = None
        sample_note = "first N/3 rows of each of the 3 initial clusters"
    else:
        c2 = dict(cfg)
        if cfg.get("strong"):  # the oracle's rate is per point*query: a 2^24-row slice of the global sample
            c2["n"] = 1 << 24
        R, S, lo, hi, _, _ = make_inputs(c2, 0, 1)
        p = np.clip(synth_true_cpu(R, lo, hi, cfg), 0, 1)
        sample_note = "the rank-0 shard" if not cfg.get("strong") else "a 2^24-row slice of the 2^28-row sample"
    h = oracle.scott(S)
    # size one step to ~3 s of all-core CPU work
    path = "single" if cfg["path"] in ("single", "stream") else cfg["path"]
    rate, use, sample, dt, k = cpu_oracle_rate(S, h, lo, hi, p, path, budget_s=3.0)
    times = []
    for i in range(args.warmup + args.steps):
        t0 = time.perf_counter()
        if path == "single":
            oracle.estimate_grad(S, h, lo[:k], hi[:k])
        else:
            oracle.loss_and_grad(S, h, lo[:k], hi[:k], p[:k], 0, 0.0, False)
        if i >= args.warmup:
            times.append(time.perf_counter() - t0)
    tot = sum(times)
    value = args.steps * k * len(S) / tot
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": "point·query evals/s",
        "n_gpus": world, "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * tot / args.steps,
        "higher_is_better": True, "scaling": "strong" if cfg.get("strong") else "weak", "vs_baseline": None,
        "dtype": "f64", "data": "synthetic",
        "config": {"workload": cfg["desc"], "d": cfg["d"], "n": cfg["n"], "q": cfg["q"],
                   "reference_sample_boxes": k, "reference_sample_rows": len(S), "sample_rows": sample_note},
        "cpu_baseline": {"value": value, "unit": "point·query evals/s", "cores": use, "kind": "oracle",
                         "sample": sample},
        "e2e": {"value": value, "unit": "point·query evals/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def synth_true_cpu(R, lo, hi, cfg):
    """True selectivities for the reference arm without a GPU: counted on a
    2^16-row subsample of R (the values only enter the loss, not the timing)."""
    import synth
    sub = R[synth.rng(3, 3).choice(len(R), size=min(len(R), 1 << 16), replace=False)]
    return synth.true_selectivity_cpu(sub, lo, hi)


# ---------------------------------------------------------------- CUDA arm
def timed_steps(step, steps, warmup, stream, m, K, flush=None, barrier=None, clock_index=0, min_region_s=1.0):
    """W untimed warm-up steps, then `steps` steps bracketed by CUDA events on `stream` (the
    launching stream), clocks sampled by nvidia-smi; short regions get an identical untimed soak
    so the sampler sees the load.  libkde's profiling counters give the dominant kernel's time."""
    import torch
    with torch.cuda.stream(stream):
        for i in range(warmup):
            step(i)
    torch.cuda.synchronize()
    K.kde_set_profiling(m.handle, True)
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(steps)]
    if barrier:
        barrier()
    torch.cuda.synchronize()
    with ClockSampler(clock_index) as clk:
        t_start = time.perf_counter()
        with torch.cuda.stream(stream):
            for i in range(steps):
                if flush is not None:
                    flush(i)
                evs[i][0].record(stream)
                step(warmup + i)
                evs[i][1].record(stream)
        torch.cuda.synchronize()
        soak = 0
        while time.perf_counter() - t_start < min_region_s and soak < 100000:
            with torch.cuda.stream(stream):
                for _ in range(8):
                    step(warmup + steps + soak)
                    soak += 1
            torch.cuda.synchronize()
    if barrier:
        barrier()
    torch.cuda.synchronize()
    scan_ms, scan_launches, launches = K.kde_get_profile(m.handle)
    cstats = K.kde_get_cells(m.handle, stats=True)[2]  # cells-scan counters (zeros when not used)
    K.kde_set_profiling(m.handle, False)
    frac = steps / max(steps + soak, 1)  # the soak launched the same kernels: keep the timed steps' share
    step_ms = [a.elapsed_time(b) for a, b in evs]
    return dict(step_ms=step_ms, scan_ms=scan_ms * frac, scan_launches=int(round(scan_launches * frac)),
                launches=int(round(launches * frac)), clocks=clk.summary(), soak=soak, events=evs,
                cells_stats=[c / max(scan_launches, 1) for c in cstats])  # per scan launch


def max_over_ranks(x, world, dev):
    import torch
    import torch.distributed as dist
    if world > 1 and dist.get_backend() == "gloo":
        dev = "cpu"
    t = torch.tensor([float(x)], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def roofline_batched(cfg, args, n_local, q, avg_ms, sms, config_name, cells_stats=None):
    d = cfg["d"]
    achieved = n_local * q / (avg_ms * 1e-3) / 1e9
    cells = bool(cells_stats and cells_stats[0] > 0)
    kname = (f"scan_cells_kernel<{d},grad> (culled, ordered copy)" if cells else
             f"scan_batched_kernel<{d},grad>{'' if args.no_cull else ' (culled)'}")
    extra = {}
    if cells:  # what the culled scan actually evaluated (kde_get_cells profiling counters)
        ev = cells_stats[2] / (n_local * q)
        extra = {"evaluated_pairs_frac": ev, "classified_pairs_frac": cells_stats[3] / (n_local * q),
                 "items_per_launch": cells_stats[0], "full_items_frac": cells_stats[1] / max(cells_stats[0], 1)}
    if cfg.get("kernel") == "epan":
        peak = sms * 128 * SM_MAX_MHZ * 1e6 / (6 * d) / 1e9
        return {"bound": "alu", "achieved": achieved, "peak": peak, "unit": "Gpt·q/s", "frac": achieved / peak,
                "traffic": _traffic(config_name), "kernel": kname + " (Epanechnikov)", **extra,
                "algorithmic": f"{n_local} points x {q} boxes per launch; 6d FP32 ops per point*box",
                "peak_source": f"FP32 ceiling {sms} SMs x 128 lanes x {SM_MAX_MHZ:.0f} MHz / (6d)"}
    peak = sms * MUFU_PER_SM_CLK * SM_MAX_MHZ * 1e6 / (2 * d) / 1e9
    return {"bound": "alu", "achieved": achieved, "peak": peak, "unit": "Gpt·q/s", "frac": achieved / peak,
            "traffic": _traffic(config_name), "ncu_pipes": _pipes(config_name),
            "kernel": kname,
            "algorithmic": f"{n_local} points x {q} boxes per launch (per GPU); 2d MUFU.EX2 per point*box"
                           + ("" if args.no_cull else " (brute-force count: culled pairs are counted as "
                              "evaluated, so frac is throughput against the unculled SFU ceiling; "
                              "evaluated_pairs_frac x frac is the fraction of the ceiling the pairs that "
                              "reached eq. 13 alone use)"),
            **extra,
            **({"evaluated_work_frac": achieved * extra["evaluated_pairs_frac"] /
                (sms * MUFU_PER_SM_CLK * SM_MAX_MHZ * 1e6 / (2 * d) / 1e9)} if extra else {}),
            "peak_source": f"SFU ceiling {sms} SMs x {MUFU_PER_SM_CLK} MUFU/clk x {SM_MAX_MHZ:.0f} MHz / (2d) "
                           "(guide unit counts; 16/clk/SM re-measured by tools/pipe_rates.cu)"}


def roofline_single(d, n_local, grad, retain, avg_ms, cull, config_name, cells_stats=None):
    alg_bytes = n_local * d * 4 + (n_local * 4 if retain else 0)  # 4d B/point read (+4 B/point retained c)
    achieved = alg_bytes / (avg_ms * 1e-3) / 1e9
    peak = _measured_hbm()
    cells = bool(cells_stats and cells_stats[0] > 0)
    g = 'grad' if grad else 'est'
    out = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
           "traffic": None if cells else _traffic(config_name), "ncu_pipes": None if cells else _pipes(config_name),
           "kernel": (f"scan_cells_single_kernel<{d},{g}> (ordered copy: far cells not read)" if cells else
                      f"scan_single_tma_kernel<{d},{g},cull>" if cull else
                      f"{'scan_single_tma_kernel' if d <= 8 else 'scan_single_kernel'}<{d},{g}>"),
           "algorithmic": f"4*d bytes/point{' + 4 B/point retained' if retain else ''} x {n_local} points per launch",
           "peak_source": "MEASURED_PEAKS.json hbm_gbs (measured copy)"}
    if cells:  # kde_get_cells counters: the cells actually read (effective vs read bandwidth)
        read = cells_stats[0] * 256 / n_local
        out.update({"sample_read_frac": read, "read_bytes_GBps": achieved * read, "read_frac": achieved * read / peak,
                    "points_evaluated_frac": cells_stats[2] / n_local,
                    "note": "frac counts the whole sample as read (effective); read_frac is the bandwidth of the "
                            "cells actually read"})
    return out


def graphed_queries(K, m, call, stream, per=16, groups=4):
    """Single-box queries replayed from CUDA graphs (one launch per `per` queries instead of one host
    call per query: the scans are tens of microseconds, comparable to the host enqueue cost).  The
    kernel time, launch count and cells counters per query come from a profiled eager pass first."""
    import torch
    with torch.cuda.stream(stream):  # untimed: first launches (lazy module loading, attributes)
        for i in range(per):
            call(i)
    torch.cuda.synchronize()
    K.kde_set_profiling(m.handle, True)
    with torch.cuda.stream(stream):
        for i in range(2 * per):
            call(i)
    torch.cuda.synchronize()
    scan_ms, scan_launches, launches = K.kde_get_profile(m.handle)
    cst = K.kde_get_cells(m.handle, stats=True)[2]
    K.kde_set_profiling(m.handle, False)
    prof = {"kernel_ms": scan_ms / max(scan_launches, 1), "launches_per_query": launches / (2 * per),
            "cells_stats": [c / max(scan_launches, 1) for c in cst]}
    graphs = []
    for gi in range(groups):
        gr = torch.cuda.CUDAGraph()
        with torch.cuda.graph(gr, stream=stream):
            for j in range(per):
                call(gi * per + j)
        graphs.append(gr)
    torch.cuda.synchronize()

    def gstep(i):
        graphs[i % groups].replay()
    return gstep, prof


def run_cuda(args, cfg, rank, world, local_rank):
    import torch
    import torch.distributed as dist

    import paper_conf_sigmod_heimelkm15_b200 as K
    from paper_conf_sigmod_heimelkm15_b200.dist import create_sharded

    gpu = 0 if args.share_gpu else local_rank
    torch.cuda.set_device(gpu)
    dev = torch.device("cuda", gpu)
    if cfg["path"] == "stream":
        if world > 1:
            raise SystemExit("c5 (device-resident streaming) is single-GPU")
        return run_stream(args, cfg, dev)
    d, q = cfg["d"], cfg["q"]
    R, S, lo, hi, lo1, hi1 = make_inputs(cfg, rank, world)
    off, n_local, n_global = shard_of(cfg, rank, world)
    p = true_selectivities(R, lo, hi) if cfg["path"] == "loss_grad" else None
    del R
    if world > 1:
        m = create_sharded(S, off, n_global, None, transport=args.comm)
    else:
        m = K.KDEModel.create(S)
    if cfg.get("kernel") == "epan":
        m.set_kernel("epan")
        m.bandwidth = m.bandwidth * np.sqrt(5.0)  # variance-matched to Scott's Gaussian bandwidth
    h = m.bandwidth
    m.cull = not args.no_cull
    m.cells = not args.no_cells
    if cfg.get("retain"):
        m.set_retain(True)
    if cfg["path"] == "single" and not args.no_cull and not args.no_cells and not cfg.get("retain"):
        # the ordered copy is a property of the sample version: build it once (one culled batched
        # call, untimed) so single-box estimates read only the cells near the box (DESIGN R17)
        m.estimate(lo[:1].repeat(2, axis=0), hi[:1].repeat(2, axis=0))

    stream = torch.cuda.Stream(device=dev)
    d_lo, d_hi = torch.from_numpy(lo).to(dev), torch.from_numpy(hi).to(dev)
    d_true = torch.from_numpy(p).to(dev) if p is not None else None
    d_loss = torch.zeros(1, dtype=torch.float64, device=dev)
    d_grad = torch.zeros(d, dtype=torch.float64, device=dev)
    d_est = torch.zeros(q, dtype=torch.float64, device=dev)
    d_dpdh = torch.zeros((q, d), dtype=torch.float64, device=dev)
    l2 = torch.cuda.get_device_properties(dev).L2_cache_size
    flush_buf = torch.empty(max(4 * l2, 256 << 20) // 4, dtype=torch.float32, device=dev)
    flush_l2 = n_local * d * 4 < 2 * l2  # sample smaller than ~2x L2 -> flush between timed steps
    flush = (lambda i: flush_buf.fill_(float(i))) if flush_l2 else None
    barrier = dist.barrier if world > 1 else None
    nbox = len(lo)

    def step(i):
        if cfg["path"] == "single":
            k = i % nbox
            K.kde_estimate_batch_dev(m.handle, d_lo[k:k + 1], d_hi[k:k + 1], d_est[:1],
                                     d_dpdh[:1] if cfg.get("grad") else None, stream=stream)
        else:
            K.kde_loss_and_grad_dev(m.handle, d_lo, d_hi, d_true, d_loss, d_grad, K.LOSS_SQUARED, 0.0, False,
                                    stream=stream)

    first_ms = None
    if cfg["path"] != "single":  # the first culled batched call builds the ordered copy (cells.cu)
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        with torch.cuda.stream(stream):
            step(0)
        torch.cuda.synchronize()
        first_ms = (time.perf_counter() - t0) * 1e3
    per = 1
    if cfg["path"] == "single" and not args.no_graph:
        per = 16
        gstep, prof = graphed_queries(K, m, step, stream, per)
        T = timed_steps(gstep, args.steps, args.warmup, stream, m, K, flush, barrier, gpu)
        T["scan_ms"], T["scan_launches"] = sum(T["step_ms"]) / (per * len(T["step_ms"])), 1  # as single leg
        T["launches"] = int(round(prof["launches_per_query"] * per * args.steps))
        T["cells_stats"] = prof["cells_stats"]
        T["step_ms"] = [x / per for x in T["step_ms"]]
    else:
        T = timed_steps(step, args.steps, args.warmup, stream, m, K, flush, barrier, gpu)
    ms_per_step = max_over_ranks(sum(T["step_ms"]), world, dev) / args.steps
    cells_info = None
    if first_ms is not None:
        on, builds = K.kde_get_cells(m.handle)
        if on and builds:
            # the rebuild alone: rewrite one row with itself (the sample changes generation, not
            # content), then one step = rebuild + scan; allocations and module loading are done
            off0 = shard_of(cfg, rank, world)[0]
            m.replace_points(np.array([off0], np.int64), np.ascontiguousarray(S[:1]))

            def wall_step():
                torch.cuda.synchronize()
                t0 = time.perf_counter()
                with torch.cuda.stream(stream):
                    step(0)
                torch.cuda.synchronize()
                return (time.perf_counter() - t0) * 1e3
            rebuild_step_ms = wall_step()
            plain_step_ms = wall_step()  # same measurement without a rebuild
            cells_info = {"builds": K.kde_get_cells(m.handle)[1], "first_call_ms": first_ms,
                          "rebuild_ms": max(rebuild_step_ms - plain_step_ms, 0.0),
                          "note": "the Morton-ordered copy of the sample is built by the first culled batched "
                                  "call (before the timed region, with the copy's allocations; the sample "
                                  "does not change between steps) and rebuilt after any call that changes "
                                  "sample rows; rebuild_ms = a step after a one-row replace minus the next step (wall clock)"}
    units_per_step = n_global * q
    value = units_per_step / (ms_per_step * 1e-3)

    # ---------------- e2e: host-pointer C-ABI call, copies inside the timed region
    e2e_steps = max(1, min(args.steps, 20))
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for i in range(e2e_steps):
        if cfg["path"] == "single":
            k = i % nbox
            m.estimate(lo[k:k + 1], hi[k:k + 1], grad=bool(cfg.get("grad")))
        else:
            m.loss_and_grad(lo, hi, p, K.LOSS_SQUARED, 0.0, False)
    torch.cuda.synchronize()
    e2e_s = max_over_ranks(time.perf_counter() - t0, world, dev)
    if cfg["path"] == "single":
        h2d, d2h = 2 * d * 4, 8 * (1 + (d if cfg.get("grad") else 0))
    else:
        h2d, d2h = 2 * q * d * 4 + q * 8, 8 * (1 + d)

    # ---------------- the configs[2] single-query leg on the same model (HBM-streaming scan)
    single = None
    if cfg.get("single_leg"):
        d_lo1, d_hi1 = torch.from_numpy(lo1).to(dev), torch.from_numpy(hi1).to(dev)

        def step1(i):
            k = i % len(lo1)
            K.kde_estimate_batch_dev(m.handle, d_lo1[k:k + 1], d_hi1[k:k + 1], d_est[:1], None, stream=stream)

        per1 = 1
        if args.no_graph:
            T1 = timed_steps(step1, max(args.steps, 20), args.warmup, stream, m, K, None, barrier, gpu)
        else:
            per1 = 16
            gstep1, prof1 = graphed_queries(K, m, step1, stream, per1)
            T1 = timed_steps(gstep1, max(args.steps, 8), args.warmup, stream, m, K, None, barrier, gpu)
            # kernel time = per-query time of the back-to-back graph replays (one kernel per query: an
            # upper bound of its duration; the eager profiled pass's events include host launch gaps)
            T1["scan_ms"], T1["scan_launches"] = sum(T1["step_ms"]) / (per1 * len(T1["step_ms"])), 1
            T1["launches"] = int(round(prof1["launches_per_query"] * per1 * len(T1["step_ms"])))
            T1["cells_stats"] = prof1["cells_stats"]
            T1["step_ms"] = [x / per1 for x in T1["step_ms"] for _ in range(per1)]
        ms1 = max_over_ranks(sum(T1["step_ms"]), world, dev) / len(T1["step_ms"])
        if world > 1:
            dist.barrier()
        t0 = time.perf_counter()
        for i in range(e2e_steps):
            m.estimate(lo1[i % len(lo1):i % len(lo1) + 1], hi1[i % len(lo1):i % len(lo1) + 1])
        e2e1 = max_over_ranks(time.perf_counter() - t0, world, dev)
        avg1 = T1["scan_ms"] / max(T1["scan_launches"], 1)
        roof1 = roofline_single(d, n_local, False, False, avg1, not args.no_cull, "c3s", T1.get("cells_stats"))
        single = {"workload": "configs[2] single DT box per step, estimate (kde_estimate_batch_dev, q = 1)"
                              + ("" if args.no_graph else f"; {per1} queries per CUDA-graph replay, ms_per_step "
                                                          "per query"),
                  "value": n_global / (ms1 * 1e-3), "unit": "point·query evals/s",
                  "estimates_per_s": 1e3 / ms1, "ms_per_step": ms1, "steps": len(T1["step_ms"]),
                  "e2e": {"value": n_global * e2e_steps / e2e1, "unit": "point·query evals/s",
                          "h2d_bytes_per_step": 2 * d * 4, "d2h_bytes_per_step": 8, "steps": e2e_steps},
                  "gpu_launches": T1["launches"], "roofline": roof1, "clocks": T1["clocks"],
                  "step_ms": {"min": min(T1["step_ms"]), "median": statistics.median(T1["step_ms"]),
                              "max": max(T1["step_ms"])}}

    if rank != 0:
        return
    clocks = T["clocks"]
    avg_scan_ms = T["scan_ms"] / max(T["scan_launches"], 1)
    sms = torch.cuda.get_device_properties(dev).multi_processor_count
    if cfg["path"] == "single":
        roof = roofline_single(d, n_local, cfg.get("grad"), cfg.get("retain"), avg_scan_ms, not args.no_cull,
                               args.config, T.get("cells_stats"))
    else:
        roof = roofline_batched(cfg, args, n_local, q, avg_scan_ms, sms, args.config, T.get("cells_stats"))
    if clocks.get("sm_mhz"):
        roof["frac_at_measured_clock"] = roof["frac"] * SM_MAX_MHZ / clocks["sm_mhz"] if roof["bound"] == "alu" \
            else roof["frac"]
    cpu = None
    if world == 1 and not args.no_cpu:
        rate, use, sample, dt, k = cpu_oracle_rate(S, h, lo, hi, p, cfg["path"], budget_s=args.cpu_budget)
        cpu = {"value": rate, "unit": "point·query evals/s", "cores": use, "kind": "oracle", "sample": sample,
               "seconds": dt}
    line = {
        "metric": METRIC, "value": value, "unit": "point·query evals/s", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True,
        "scaling": "strong" if cfg.get("strong") else "weak", "vs_baseline": None, "dtype": "f32",
        "data": "synthetic",
        "config": {"workload": cfg["desc"], "d": d, "n_per_gpu": n_local, "n_global": n_global, "q": q,
                   **({"cuda_graph": f"{per} single-box queries per graph replay; ms_per_step per query"}
                      if per > 1 else {}),
                   "comm": (args.comm if world > 1 else "none"),
                   **({"shared_gpu": "all ranks on cuda:0 (time-sliced): a functional check of the world > 1 "
                                     "path, NOT a scaling measurement"} if args.share_gpu else {}),
                   "l2": "flushed between timed steps" if flush_l2 else "sample larger than L2",
                   "cull": ("off" if args.no_cull else
                            "on: (point, box) pairs whose contribution is provably < 2^-64 are skipped (DESIGN R15)"),
                   "clock_sampling": "nvidia-smi every 100 ms over the timed steps"
                                     + (f" + {T['soak']} identical untimed soak steps (timed region < 1 s)"
                                        if T["soak"] else ""),
                   "accumulation": ("fp32 per (box, 256-point cell) item, fp64 above" if cells_info else
                                    "fp32 per <=32 points, fp64 above")},
        "estimates_per_s": q / (ms_per_step * 1e-3),
        "e2e": {"value": units_per_step * e2e_steps / e2e_s, "unit": "point·query evals/s",
                "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h, "steps": e2e_steps},
        "gpu_launches": T["launches"], "scan_launches": T["scan_launches"],
        "roofline": roof, "cpu_baseline": cpu, "clocks": clocks,
        "step_ms": {"min": min(T["step_ms"]), "median": statistics.median(T["step_ms"]), "max": max(T["step_ms"])},
    }
    if cells_info is not None:
        line["cells_index"] = cells_info
    if single is not None:
        line["single_query"] = single
    print(json.dumps(line), flush=True)


def run_stream(args, cfg, dev):
    """configs[4]: reservoir inserts + deletes + device-resident streaming queries (single GPU).
    Database: clusters of 2^22 rows; cycle c inserts cluster c + 3 in 2^16-row chunks (64 chunks)
    through the reservoir, then deletes cluster c.  The timed steps cross the end of cycle 0: the
    first PRE chunks of cluster 3 are inserted untimed, so the timed region sees the last chunks of
    cycle 0, the deletion of cluster 0 and the first chunks of cluster 4."""
    import torch

    import paper_conf_sigmod_heimelkm15_b200 as K
    import synth
    d, N = cfg["d"], cfg["n"]
    rows = 1 << 22            # rows per database cluster
    chunk = 1 << 16           # arrivals per insert chunk
    per_cycle = rows // chunk
    qpc = cfg["q"]            # queries per chunk
    cap = 1 << 16
    res_seed = 0xC5
    P = args.warmup + args.steps
    PRE = max(0, per_cycle - 4)  # untimed prefill: the timed steps cross the cycle boundary
    sc = synth.StreamClusters(d, rows, seed=11)
    cl = {c: sc.cluster_rows(c) for c in range(4)}   # R0 = clusters 0..2; cluster 3 = cycle 0's inserts
    n_c4 = max(0, PRE + P - per_cycle) * chunk
    if n_c4:
        cl[4] = sc.cluster_rows(4, 0, min(rows, n_c4))
    # the sample: the reservoir after R0's 3 x 2^22 arrivals
    base = np.concatenate([cl[0], cl[1], cl[2]])
    n0 = len(base)
    sl = K.kde_reservoir_select(res_seed, N, N, n0 - N)
    content = np.arange(N)
    ids = np.arange(N, n0)
    ok = sl >= 0
    rev_s, rev_i = sl[ok][::-1], ids[ok][::-1]
    u, first = np.unique(rev_s, return_index=True)  # the last arrival per slot wins
    content[u] = rev_i[first]
    S = base[content]
    del base
    m = K.KDEModel.create(S)
    m.set_retain(True)
    m.cull = not args.no_cull
    state = {"n_seen": n0, "written": []}

    def chunk_rows(t):  # arrivals of global chunk t
        c = 3 + t // per_cycle
        a = (t % per_cycle) * chunk
        return cl[c][a:a + chunk]

    for t in range(PRE):  # untimed prefill of cycle 0
        state["n_seen"], _ = m.insert_rows(chunk_rows(t), res_seed, state["n_seen"])

    def live_after(t):  # (full clusters, partial cluster, inserted rows of it) after chunk t's insert
        c = t // per_cycle
        return [c, c + 1, c + 2], c + 3, (t % per_cycle + 1) * chunk

    ts = [PRE + i for i in range(P)]
    Qlo = np.empty((P * qpc, d), np.float32)
    Qhi = np.empty((P * qpc, d), np.float32)
    p = np.empty(P * qpc)
    dcl = {}
    for i, t in enumerate(ts):
        full, part, ins = live_after(t)
        lo_t, hi_t = sc.queries(full + [part], qpc, seed=1000 + t)
        Qlo[i * qpc:(i + 1) * qpc], Qhi[i * qpc:(i + 1) * qpc] = lo_t, hi_t
        dlo_t, dhi_t = torch.from_numpy(lo_t).to(dev), torch.from_numpy(hi_t).to(dev)
        tot = torch.zeros(qpc, dtype=torch.int64, device=dev)
        for c in full + [part]:
            if c not in dcl:
                dcl[c] = torch.from_numpy(cl[c]).to(dev)
            rows_c = dcl[c] if c != part else dcl[c][:ins]
            cnt = torch.zeros(qpc, dtype=torch.int64, device=dev)
            K.kde_count_in_box_dev(rows_c, dlo_t, dhi_t, cnt)
            tot += cnt
        torch.cuda.synchronize()
        p[i * qpc:(i + 1) * qpc] = (tot.double() / (len(full) * rows + ins)).cpu().numpy()
    del dcl
    # karma replacement pool: rows of the live database at the cycle boundary
    g = synth.rng(14)
    pool = np.concatenate([cl[c][g.integers(0, rows, size=1 << 15)] for c in (1, 2, 3)] +
                          [chunk_rows(ts[-1])[: 1 << 15]])
    d_pool = torch.from_numpy(pool).to(dev)
    npool = len(pool) - cap
    stream = torch.cuda.Stream(device=dev)
    d_lo, d_hi = torch.from_numpy(Qlo).to(dev), torch.from_numpy(Qhi).to(dev)
    d_true = torch.from_numpy(p).to(dev)
    kp = K.karma_params(loss=K.LOSS_ABSOLUTE, threshold=-1.0 / (N - 1), k_max=4.0)
    op = K.online_params(minibatch=10, loss=K.LOSS_ABSOLUTE, log_bandwidth=True)
    d_idx = torch.zeros(cap, dtype=torch.int64, device=dev)
    d_cnt = torch.zeros(1, dtype=torch.int64, device=dev)
    d_est = torch.zeros(1, dtype=torch.float64, device=dev)
    d_dpdh = torch.zeros(d, dtype=torch.float64, device=dev)

    def query(qi):
        off = (qi * 977) % npool
        K.kde_stream_step_dev(m.handle, d_lo[qi:qi + 1], d_hi[qi:qi + 1], d_true[qi:qi + 1], kp, op, d_idx, d_cnt,
                              d_pool[off:off + cap], d_est, d_dpdh, stream=stream)

    # launch statistics of one query step (libkde's counters), then one CUDA graph per chunk
    with torch.cuda.stream(stream):  # untimed first launches (lazy module loading, attributes)
        for qi in range(8):
            query(qi)
    torch.cuda.synchronize()
    K.kde_set_profiling(m.handle, True)
    with torch.cuda.stream(stream):
        for qi in range(min(P * qpc, 64)):
            query(qi)
    torch.cuda.synchronize()
    prof_pre = K.kde_get_profile(m.handle)
    n_pre = min(P * qpc, 64)
    K.kde_set_profiling(m.handle, False)
    graphs = []
    if not args.no_graph:
        for i in range(P):
            gr = torch.cuda.CUDAGraph()
            with torch.cuda.graph(gr, stream=stream):
                for qi in range(i * qpc, (i + 1) * qpc):
                    query(qi)
            graphs.append(gr)
        with torch.cuda.stream(stream):
            for gr in graphs:
                gr.replay()
        torch.cuda.synchronize()

    split_ev = []

    def step(i):
        i = i % P
        # host reservoir decision, only accepted rows cross PCIe; the deletion of a cluster
        # at a cycle boundary changes only the database (true selectivities), not the sample
        t_ins = time.perf_counter()
        # async: the decisions for this chunk overlap the device's previous queries
        n_seen, nw = K.kde_insert_rows_async(m.handle, chunk_rows(ts[i]), res_seed, state["n_seen"], stream=stream)
        state["n_seen"] = n_seen
        state["written"].append(nw)
        ev = torch.cuda.Event(enable_timing=True)
        ev.record(stream)  # the queries' share of the step starts here
        split_ev.append((time.perf_counter() - t_ins, ev))
        if graphs:
            graphs[i].replay()
        else:
            for qi in range(i * qpc, (i + 1) * qpc):
                query(qi)

    T = timed_steps(step, args.steps, args.warmup, stream, m, K, None, None, 0)
    ms_per_step = sum(T["step_ms"]) / args.steps
    value = N * qpc / (ms_per_step * 1e-3)
    # breakdown of the timed steps: host insert call (wall) and the queries' device time
    timed = split_ev[args.warmup:args.warmup + args.steps]
    ins_ms = 1e3 * float(np.mean([w for w, _ in timed]))
    q_ms = float(np.mean([ev.elapsed_time(T["events"][k][1]) for k, (_, ev) in enumerate(timed)]))
    launches = T["launches"] + int(round(prof_pre[2] / n_pre * qpc * args.steps)) if graphs else T["launches"]
    avg_scan_ms = prof_pre[0] / max(prof_pre[1], 1)
    written = float(np.mean(state["written"])) if state["written"] else 0.0

    # e2e: the host-pointer calls (inserts, estimate + gradient, karma, Listing 1, replacement)
    flagged = []
    e2e_steps = max(1, min(args.steps, 5))
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for i in range(e2e_steps):
        ns, _ = m.insert_rows(chunk_rows(ts[i % P]), res_seed, state["n_seen"])
        state["n_seen"] = ns
        for qi in range((i % P) * qpc, (i % P + 1) * qpc):
            m.estimate(Qlo[qi:qi + 1], Qhi[qi:qi + 1], grad=True)
            idx, nf, _ = m.karma_update(Qlo[qi], Qhi[qi], p[qi], kp, cap=cap)
            m.online_update(Qlo[qi], Qhi[qi], p[qi], op)
            off = (qi * 977) % npool
            m.replace_points(idx, pool[off:off + len(idx)])
            flagged.append(nf)
    torch.cuda.synchronize()
    e2e_s = time.perf_counter() - t0
    mean_flag = float(np.mean(flagged)) if flagged else 0.0
    h2d = int(written * (8 + 4 * d)) + qpc * (2 * d * 4 * 3 + 8 * 2 + int(mean_flag * (8 + 4 * d)))
    d2h = qpc * (8 * (1 + d) + int(mean_flag * 8) + 8 + 4)
    roof = roofline_single(d, N, True, True, avg_scan_ms, not args.no_cull, "c5s")
    clocks = T["clocks"]
    cpu = None
    if not args.no_cpu:
        h = m.bandwidth
        rate, use, sample, dt, k = cpu_oracle_rate(S, h, Qlo, Qhi, None, "single", budget_s=args.cpu_budget)
        cpu = {"value": rate, "unit": "point·query evals/s", "cores": use, "kind": "oracle", "sample": sample,
               "seconds": dt}
    line = {
        "metric": METRIC, "value": value, "unit": "point·query evals/s", "n_gpus": 1, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "f32", "data": "synthetic",
        "config": {"workload": cfg["desc"], "d": d, "n_per_gpu": N, "n_global": N, "q": qpc,
                   "insert_chunk": chunk, "chunks_per_cycle": per_cycle,
                   "timed_chunks": f"global chunks {ts[0]}..{ts[-1]} (cycle boundary, delete of cluster 0, "
                                   f"after chunk {per_cycle - 1})",
                   "cuda_graph": bool(graphs), "l2": "sample larger than L2",
                   "cull": "off" if args.no_cull else "on (DESIGN R15)",
                   "clock_sampling": "nvidia-smi every 100 ms over the timed steps"
                                     + (f" + {T['soak']} identical untimed soak steps" if T["soak"] else "")},
        "estimates_per_s": qpc / (ms_per_step * 1e-3),
        "stream": {"queries_per_s": qpc * 1e3 / ms_per_step, "inserts_per_s": chunk * 1e3 / ms_per_step,
                   "rows_written_per_chunk": written, "mean_flagged_per_query_e2e": mean_flag,
                   "insert_call_ms": ins_ms, "queries_device_ms": q_ms,
                   "us_per_query_device": 1e3 * q_ms / qpc},
        "e2e": {"value": N * qpc * e2e_steps / e2e_s, "unit": "point·query evals/s",
                "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h, "steps": e2e_steps,
                "queries_per_s": qpc * e2e_steps / e2e_s},
        "gpu_launches": launches, "roofline": roof, "cpu_baseline": cpu, "clocks": clocks,
        "step_ms": {"min": min(T["step_ms"]), "median": statistics.median(T["step_ms"]), "max": max(T["step_ms"])},
    }
    print(json.dumps(line), flush=True)


def _measured_hbm():
    try:
        return float(json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"])
    except Exception:
        return 6650.0  # B200_PROFILING.md fallback


def _pipes(config):
    """ncu pipe utilisation of the dominant kernel from the committed capture, if any."""
    try:
        t = json.load(open(os.path.join(ROOT, "profiles", "ncu_pipes.json")))
        return t.get(config)
    except Exception:
        return None


def _traffic(config):
    """dram bytes per launch of the dominant kernel from the committed ncu capture, if any."""
    try:
        t = json.load(open(os.path.join(ROOT, "profiles", "traffic.json")))
        return t.get(config)
    except Exception:
        return None


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="c3", choices=sorted(CONFIGS))
    ap.add_argument("--impl", default="cuda", choices=["cuda", "reference"])
    ap.add_argument("--comm", default="peer", choices=["peer", "nccl"],
                    help="world > 1: all-gather of the partial sums over peer device memory (libkde) or NCCL")
    ap.add_argument("--no-cpu", action="store_true", help="skip the cpu_baseline leg")
    ap.add_argument("--no-cull", action="store_true",
                    help="evaluate every (point, box) pair (kde_set_cull(0)); default culls provably < 2^-64")
    ap.add_argument("--no-cells", action="store_true",
                    help="culled scans over the sample's own order instead of the Morton-ordered copy (A/B)")
    ap.add_argument("--no-graph", action="store_true", help="stream configs: launch eagerly instead of CUDA graphs")
    ap.add_argument("--cpu-budget", type=float, default=12.0, help="seconds of all-core oracle work")
    ap.add_argument("--rows", type=int, default=0,
                    help="override the config's sample rows (per GPU, or global for strong configs); recorded in "
                         "config -- for functional checks, not the named workload")
    ap.add_argument("--share-gpu", action="store_true",
                    help="run every rank on cuda:0 (gloo process group, peer transport): exercises the world > 1 "
                         "path on a one-GPU box; not a scaling measurement")
    args = ap.parse_args()
    if args.warmup < 3:
        args.warmup = 3
    if "WORLD_SIZE" not in os.environ and args.gpus > 1:
        # launch one rank per GPU ourselves (the driver may also start us under torchrun)
        cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
               "--master-addr", "127.0.0.1", "--master-port", str(_free_port()), os.path.abspath(__file__)] + sys.argv[1:]
        raise SystemExit(subprocess.call(cmd))
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if world != args.gpus:
        raise SystemExit(f"--gpus {args.gpus} but WORLD_SIZE {world}")
    cfg = dict(CONFIGS[args.config])
    if args.rows:
        cfg["n"] = args.rows
        cfg["desc"] = cfg["desc"] + f" [rows overridden: {args.rows}]"
    if args.impl == "reference":
        run_reference(args, cfg, rank, world)
        return
    if args.share_gpu and args.comm != "peer":
        raise SystemExit("--share-gpu needs --comm peer (NCCL rejects two ranks on one GPU)")
    if world > 1:
        import torch
        import torch.distributed as dist
        if args.share_gpu:
            torch.cuda.set_device(0)
            dist.init_process_group("gloo")
        else:
            torch.cuda.set_device(local_rank)
            dist.init_process_group("nccl", device_id=torch.device("cuda", local_rank))
    try:
        run_cuda(args, cfg, rank, world, local_rank)
    finally:
        if world > 1:
            import torch.distributed as dist
            dist.destroy_process_group()


if __name__ == "__main__":
    main()
