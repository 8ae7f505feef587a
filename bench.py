#!/usr/bin/env python
"""bench.py -- throughput of the KDE range-selectivity hot path on B200.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config c2|c3|c3s|c4|c5s] [--impl cuda|reference]

A "step" is one pass of the hot path over one batch of synthetic input.  The
default workload is BASELINE.json configs[1] ("c2"): d = 3, N = 2^20 sample
points per GPU, a 10k-box batch, estimate + loss + bandwidth gradient
(kde_loss_and_grad, eq. 5/14/17) -- the inner call of batch bandwidth
optimisation.  With --gpus N > 1 (torchrun, one process per GPU) every rank
holds its own 2^20-row shard of an N*2^20-row sample (weak scaling); the
per-box partial sums are combined with NCCL inside libkde.

value   = point*query evaluations per second over the whole job
          (N_global * q / step time, max over ranks, CUDA events, inputs
          resident in HBM, L2 flushed between timed steps).
e2e     = the same metric through the host-pointer C-ABI call (bounds and
          true selectivities copied host->device, loss + gradient copied back,
          inside the timed region).
roofline: the batched scan kernel against the SFU ceiling 148 SMs x 16
          MUFU/clk x 1965 MHz / (2d) point*query/s (two exp per dimension are
          the algorithmic minimum: Phi and the gradient share e^{-z^2}).
cpu_baseline / --impl reference: the fp64 C oracle (oracle/) as it stands,
          on the host cores, over a bounded sample of the same workload.
"""
from __future__ import annotations

import argparse
import json
import os
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
    # name: d, rows per GPU, boxes, path, description
    "c2": dict(d=3, n=1 << 20, q=10000, path="loss_grad", data="gauss",
               desc="configs[1]: d=3, N=2^20/GPU, 10k-box batch, estimate + L2 loss + bandwidth gradient"),
    "c3": dict(d=5, n=1 << 24, q=4096, path="loss_grad", data="gauss",
               desc="configs[2] batched: d=5, N=2^24/GPU, 4096-box DT/DV/UT/UV batch, estimate + gradient"),
    "c3s": dict(d=5, n=1 << 24, q=1, path="single", grad=False, retain=False, data="gauss",
                desc="configs[2] single box: d=5, N=2^24/GPU, one DT box per step, estimate (HBM-streaming scan)"),
    "c3sg": dict(d=5, n=1 << 24, q=1, path="single", grad=True, retain=False, data="gauss",
                 desc="configs[2] single box: d=5, N=2^24/GPU, one DT box per step, estimate + bandwidth gradient"),
    "c5s": dict(d=10, n=1 << 22, q=1, path="single", grad=True, retain=True, data="gauss",
                desc="configs[4] estimate step: d=10, N=2^22/GPU, one DT box, estimate + gradient + retained "
                     "contributions (Adaptive, P:L240)"),
    "c5": dict(d=10, n=1 << 22, q=1, path="stream", grad=True, retain=True, data="gauss",
               desc="configs[4] streaming step: d=10, N=2^22, one DT box per step: estimate + gradient + retained "
                    "contributions, karma pass + compaction, Listing 1 bandwidth step, replacement of flagged points "
                    "(device-resident kde_stream_step_dev: 3 kernels, single GPU)"),
    "c2e": dict(d=3, n=1 << 20, q=10000, path="loss_grad", data="gauss", kernel="epan",
                desc="configs[1] with the Epanechnikov product kernel (NEXT-4, reading R14): d=3, N=2^20/GPU, "
                     "10k-box batch, estimate + L2 loss + bandwidth gradient"),
    "c3se": dict(d=5, n=1 << 24, q=1, path="single", grad=False, retain=False, data="gauss", kernel="epan",
                 desc="configs[2] single box with the Epanechnikov product kernel: d=5, N=2^24/GPU, estimate"),
    "c4": dict(d=8, n=1 << 25, q=4096, path="loss_grad", data="gauss",
               desc="configs[3] per-GPU shard: d=8, 2^25 rows/GPU (2^28 at 8 GPUs), 4096 boxes, estimate + gradient + NCCL"),
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


def make_inputs(cfg, rank: int, seed: int = 7):
    """Seeded synthetic inputs: this rank's sample shard, the (replicated)
    boxes and, for loss/grad, true selectivities counted on a database R."""
    import synth
    d, n, q = cfg["d"], cfg["n"], cfg["q"]
    if n <= (1 << 21):
        # the "database" R has 4x the rows; the sample is a without-replacement draw from it
        R = synth.make_data(cfg["data"], 4 * n, d, seed=seed + 1000 * rank)
        S = R[synth.rng(seed, 500 + rank).choice(len(R), size=n, replace=False)]
    else:
        # large samples: S is drawn directly; true selectivities are counted on a 2^22-row subsample
        S = synth.make_data(cfg["data"], n, d, seed=seed + 1000 * rank)
        R = S[synth.rng(seed, 600 + rank).choice(n, size=1 << 22, replace=False)]
    Q = synth.make_data(cfg["data"], 1 << 16, d, seed=seed)  # rank-independent box generator
    if q == 1:
        lo, hi = synth.workload(Q, 64, seed + 1, "DT")
    else:
        lo, hi = synth.mixed_workload(Q, q, seed + 1)
    return R, S, lo, hi


def true_selectivities(R, lo, hi):
    """Exact counts over R on the GPU (harness kernel kde_count_in_box_dev)."""
    import torch

    import paper_conf_sigmod_heimelkm15_b200 as K
    dR = torch.from_numpy(R).cuda()
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
    R, S, lo, hi = make_inputs(cfg, 0)
    import oracle
    oracle.build()
    h = oracle.scott(S)
    p = np.clip(synth_true_cpu(R, lo, hi, cfg), 0, 1)
    # size one step to ~3 s of all-core CPU work
    rate, use, sample, dt, k = cpu_oracle_rate(S, h, lo, hi, p, cfg["path"], budget_s=3.0)
    times = []
    for i in range(args.warmup + args.steps):
        t0 = time.perf_counter()
        if cfg["path"] in ("single", "stream"):
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
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": cfg["desc"], "d": cfg["d"], "n_per_gpu": cfg["n"], "q": cfg["q"],
                   "reference_sample_boxes": k},
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
def run_cuda(args, cfg, rank, world, local_rank):
    import torch
    import torch.distributed as dist

    import paper_conf_sigmod_heimelkm15_b200 as K
    from paper_conf_sigmod_heimelkm15_b200.dist import exchange_unique_id

    torch.cuda.set_device(local_rank)
    dev = torch.device("cuda", local_rank)
    d, n, q = cfg["d"], cfg["n"], cfg["q"]
    R, S, lo, hi = make_inputs(cfg, rank)
    p = true_selectivities(R, lo, hi) if cfg["path"] != "single" else None
    if cfg["path"] == "stream" and world > 1:
        raise SystemExit("c5 (device-resident streaming) is single-GPU")

    n_global = n * world
    if world > 1:
        nid = exchange_unique_id()
        m = K.KDEModel.create_sharded(S, rank * n, n_global, None, nid, rank, world)
    else:
        m = K.KDEModel.create(S)
    if cfg.get("kernel") == "epan":
        m.set_kernel("epan")
        m.bandwidth = m.bandwidth * np.sqrt(5.0)  # variance-matched to Scott's Gaussian bandwidth
    h = m.bandwidth
    m.cull = not args.no_cull

    stream = torch.cuda.Stream(device=dev)
    d_lo = torch.from_numpy(lo).to(dev)
    d_hi = torch.from_numpy(hi).to(dev)
    d_true = torch.from_numpy(p).to(dev) if p is not None else None
    d_loss = torch.zeros(1, dtype=torch.float64, device=dev)
    d_grad = torch.zeros(d, dtype=torch.float64, device=dev)
    d_est = torch.zeros(q, dtype=torch.float64, device=dev)
    d_dpdh = torch.zeros((q, d), dtype=torch.float64, device=dev)
    l2 = torch.cuda.get_device_properties(dev).L2_cache_size
    flush_buf = torch.empty(max(4 * l2, 256 << 20) // 4, dtype=torch.float32, device=dev)
    flush_l2 = cfg["n"] * d * 4 < 2 * l2  # sample smaller than ~2x L2 -> flush between timed steps
    nbox = len(lo)

    if cfg.get("retain"):
        m.set_retain(True)
    use_graph = cfg["path"] == "stream" and not args.no_graph
    if cfg["path"] == "stream":
        cap = 1 << 16
        kp = K.karma_params(loss=K.LOSS_ABSOLUTE, threshold=-1.0 / (n_global - 1), k_max=4.0)
        op = K.online_params(minibatch=10, loss=K.LOSS_ABSOLUTE, log_bandwidth=True)
        d_pool = torch.from_numpy(R).to(dev)  # replacement rows drawn from the database R
        d_idx = torch.zeros(cap, dtype=torch.int64, device=dev)
        d_cnt = torch.zeros(1, dtype=torch.int64, device=dev)
        npool = len(R) - cap
        flagged = []

    def step(i):
        if cfg["path"] == "stream":
            k = i % nbox
            off = (k * 977) % npool
            K.kde_stream_step_dev(m.handle, d_lo[k:k + 1], d_hi[k:k + 1], d_true[k:k + 1], kp, op, d_idx, d_cnt,
                                  d_pool[off:off + cap], d_est[:1], d_dpdh[0], stream=stream)
            return
        if cfg["path"] == "single":
            k = i % nbox
            K.kde_estimate_batch_dev(m.handle, d_lo[k:k + 1], d_hi[k:k + 1], d_est[:1],
                                     d_dpdh[:1] if cfg.get("grad") else None, stream=stream)
        else:
            K.kde_loss_and_grad_dev(m.handle, d_lo, d_hi, d_true, d_loss, d_grad, K.LOSS_SQUARED, 0.0, False,
                                    stream=stream)

    with torch.cuda.stream(stream):
        for i in range(args.warmup):
            step(i)
    torch.cuda.synchronize()

    graphs = None
    prof_pre = None
    if use_graph:
        # launch-bound multi-kernel steps: one CUDA graph per box (the step's
        # arguments depend only on the box index), replayed per step.  The scan
        # kernel's own duration for the roofline is taken from profiled eager
        # steps first (kernel events cannot be read back from a replayed graph).
        K.kde_set_profiling(m.handle, True)
        with torch.cuda.stream(stream):
            for i in range(args.warmup, args.warmup + max(args.steps, 8)):
                step(i)
        torch.cuda.synchronize()
        prof_pre = K.kde_get_profile(m.handle)
        K.kde_set_profiling(m.handle, False)
        graphs = []
        for k in range(nbox):
            g = torch.cuda.CUDAGraph()
            with torch.cuda.graph(g, stream=stream):
                step(k)
            graphs.append(g)
        torch.cuda.synchronize()
        # the first replay of a graph uploads it (~0.7 ms): replay each once, untimed
        with torch.cuda.stream(stream):
            for g in graphs:
                g.replay()
        torch.cuda.synchronize()

        def step(i):  # noqa: F811
            graphs[i % nbox].replay()

    K.kde_set_profiling(m.handle, True)
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    with ClockSampler(local_rank) as clk:
        t_start = time.perf_counter()
        with torch.cuda.stream(stream):
            for i in range(args.steps):
                if flush_l2:
                    flush_buf.fill_(float(i))
                evs[i][0].record(stream)
                step(i)
                evs[i][1].record(stream)
        torch.cuda.synchronize()
        # short timed regions (< 1 s) are followed by an identical untimed soak so
        # that nvidia-smi (100 ms period) samples the clocks under this load
        soak = 0
        while time.perf_counter() - t_start < 1.0 and soak < 100000:
            with torch.cuda.stream(stream):
                for _ in range(8):
                    step(args.steps + soak)
                    soak += 1
            torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    scan_ms, scan_launches, launches = K.kde_get_profile(m.handle)
    # the soak steps launched the same kernels: keep the timed steps' share
    per_step = launches / max(args.steps + soak, 1)
    launches = int(round(per_step * args.steps))
    scan_ms *= args.steps / max(args.steps + soak, 1)
    scan_launches = int(round(scan_launches * args.steps / max(args.steps + soak, 1)))
    if graphs is not None:  # graph replays bypass libkde's host-side counters
        ms_pre, sl_pre, l_pre = prof_pre
        n_pre = max(args.steps, 8)
        launches = int(round(l_pre / n_pre * args.steps))
        scan_launches = int(round(sl_pre / n_pre * args.steps))
        scan_ms = ms_pre / n_pre * args.steps
    K.kde_set_profiling(m.handle, False)
    step_ms = [a.elapsed_time(b) for a, b in evs]
    tot_ms = sum(step_ms)
    t = torch.tensor([tot_ms], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    tot_ms = float(t.item())
    ms_per_step = tot_ms / args.steps
    units_per_step = n_global * q
    value = units_per_step / (ms_per_step * 1e-3)

    # ---------------- e2e: host-pointer C-ABI call, copies inside the timed region
    e2e_steps = max(1, min(args.steps, 20))
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for i in range(e2e_steps):
        if cfg["path"] == "stream":
            k = i % nbox
            m.estimate(lo[k:k + 1], hi[k:k + 1], grad=True)
            idx, nf, _ = m.karma_update(lo[k], hi[k], p[k], kp, cap=cap)
            m.online_update(lo[k], hi[k], p[k], op)
            off = (i * 977) % npool
            m.replace_points(idx, R[off:off + len(idx)])
            flagged.append(nf)
        elif cfg["path"] == "single":
            k = i % nbox
            m.estimate(lo[k:k + 1], hi[k:k + 1], grad=bool(cfg.get("grad")))
        else:
            m.loss_and_grad(lo, hi, p, K.LOSS_SQUARED, 0.0, False)
    torch.cuda.synchronize()
    e2e_s = time.perf_counter() - t0
    t = torch.tensor([e2e_s], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    e2e_s = float(t.item())
    if cfg["path"] == "stream":
        mean_flag = float(np.mean(flagged)) if flagged else 0.0
        h2d = 2 * d * 4 * 3 + 8 * 2 + int(mean_flag * (8 + 4 * d))  # bounds (3 calls), true sel (2), replacement idx+rows
        d2h = 8 * (1 + d) + int(mean_flag * 8) + 8 + 4  # estimate+gradient, flagged indices, count, update flag
    elif cfg["path"] == "single":
        h2d, d2h = 2 * d * 4, 8 * (1 + (d if cfg.get("grad") else 0))
    else:
        h2d, d2h = 2 * q * d * 4 + q * 8, 8 * (1 + d)

    if rank != 0:
        return
    # ---------------- roofline of the dominant (scan) kernel, per GPU
    clocks = clk.summary()
    avg_scan_ms = scan_ms / max(scan_launches, 1)
    sms = torch.cuda.get_device_properties(dev).multi_processor_count
    if cfg["path"] in ("single", "stream"):
        alg_bytes = n * d * 4 + (n * 4 if cfg.get("retain") else 0)  # 4d B/point read (+4 B/point retained c)
        achieved = alg_bytes / (avg_scan_ms * 1e-3) / 1e9
        peak = _measured_hbm()
        roof = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
                "traffic": _traffic(args.config), "kernel": (f"scan_single_tma_kernel<{d},{'grad' if cfg.get('grad') else 'est'},cull>" if not args.no_cull else
                           f"{'scan_single_tma_kernel' if d <= 8 else 'scan_single_kernel'}<{d},{'grad' if cfg.get('grad') else 'est'}>"),
                "algorithmic": f"4*d bytes/point{' + 4 B/point retained' if cfg.get('retain') else ''} x {n} points per launch",
                "peak_source": "MEASURED_PEAKS.json hbm_gbs (measured copy)"}
    elif cfg.get("kernel") == "epan":
        # no transcendental: the algorithmic minimum is the FP32 work, 6 FP32 ops per dimension
        # (2 subtract-scale, 2 products of the S = a^2 + ab + b^2 form, 2 for D) -> FP32 ceiling
        achieved = n * q / (avg_scan_ms * 1e-3) / 1e9
        peak = sms * 128 * SM_MAX_MHZ * 1e6 / (6 * d) / 1e9
        roof = {"bound": "alu", "achieved": achieved, "peak": peak, "unit": "Gpt·q/s", "frac": achieved / peak,
                "traffic": _traffic(args.config), "kernel": f"scan_batched_kernel<{d},grad> (Epanechnikov)",
                "algorithmic": f"{n} points x {q} boxes per launch; 6d FP32 ops per point*box",
                "peak_source": f"FP32 ceiling {sms} SMs x 128 lanes x {SM_MAX_MHZ:.0f} MHz / (6d)"}
    else:
        achieved = n * q / (avg_scan_ms * 1e-3) / 1e9
        peak = sms * MUFU_PER_SM_CLK * SM_MAX_MHZ * 1e6 / (2 * d) / 1e9
        roof = {"bound": "alu", "achieved": achieved, "peak": peak, "unit": "Gpt·q/s",
                "frac": achieved / peak, "traffic": _traffic(args.config),
                "kernel": f"scan_batched_kernel<{d},grad>{'' if args.no_cull else ' (culled)'}",
                "algorithmic": f"{n} points x {q} boxes per launch; 2d MUFU.EX2 per point*box"
                               + ("" if args.no_cull else " (brute-force count: culled pairs are counted as "
                                  "evaluated, so frac is throughput against the unculled SFU ceiling)"),
                "peak_source": f"SFU ceiling {sms} SMs x {MUFU_PER_SM_CLK} MUFU/clk x {SM_MAX_MHZ:.0f} MHz / (2d) "
                               "(guide unit counts; 16/clk/SM re-measured by tools/pipe_rates.cu)"}
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
        "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "f32", "data": "synthetic",
        "config": {"workload": cfg["desc"], "d": d, "n_per_gpu": n, "n_global": n_global, "q": q,
                   "l2": "flushed between timed steps" if flush_l2 else "sample larger than L2",
                   "cuda_graph": bool(graphs is not None),
                   "cull": ("off" if args.no_cull else
                            "on: (point, box) pairs whose contribution is provably < 2^-64 are skipped (DESIGN R15)"),
                   "clock_sampling": "nvidia-smi every 100 ms over the timed steps"
                                     + (f" + {soak} identical untimed soak steps (timed region < 1 s)" if soak else ""),
                   "accumulation": "fp32 per <=32 points, fp64 above"},
        "estimates_per_s": q / (ms_per_step * 1e-3),
        **({"stream": {"queries_per_s": 1e3 / ms_per_step, "mean_flagged_per_query_e2e": float(np.mean(flagged))}}
           if cfg["path"] == "stream" else {}),
        "e2e": {"value": units_per_step * e2e_steps / e2e_s, "unit": "point·query evals/s",
                "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h, "steps": e2e_steps},
        "gpu_launches": launches, "scan_launches": scan_launches,
        "roofline": roof, "cpu_baseline": cpu, "clocks": clocks,
        "step_ms": {"min": min(step_ms), "median": statistics.median(step_ms), "max": max(step_ms)},
    }
    print(json.dumps(line), flush=True)


def _measured_hbm():
    try:
        return float(json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"])
    except Exception:
        return 6650.0  # B200_PROFILING.md fallback


def _traffic(config):
    """dram bytes per launch of the dominant kernel from the committed ncu capture, if any."""
    try:
        t = json.load(open(os.path.join(ROOT, "profiles", "traffic.json")))
        return t.get(config)
    except Exception:
        return None


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="c2", choices=sorted(CONFIGS))
    ap.add_argument("--impl", default="cuda", choices=["cuda", "reference"])
    ap.add_argument("--no-cpu", action="store_true", help="skip the cpu_baseline leg")
    ap.add_argument("--no-cull", action="store_true",
                    help="single-box scans evaluate every point (kde_set_cull(0)); default culls provably < 2^-64")
    ap.add_argument("--no-graph", action="store_true", help="stream configs: launch eagerly instead of CUDA graphs")
    ap.add_argument("--cpu-budget", type=float, default=12.0, help="seconds of all-core oracle work")
    args = ap.parse_args()
    if args.warmup < 3:
        args.warmup = 3
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    cfg = CONFIGS[args.config]
    if args.impl == "reference":
        run_reference(args, cfg, rank, world)
        return
    if world > 1:
        import torch
        import torch.distributed as dist
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
