"""Synthetic analogues of the paper's quality experiments,
run end to end through libkde on one B200.

  python experiments/quality.py [--quick] > experiments/results.json

(1) model size (Fig. 6): 8-D real-data-like skewed table, DT
    workload, 100 training + 100 test boxes, sample sizes 2^10 .. 2^20
    (the paper stops at 32K points; its Fig. 7 runtime argument is that larger
    samples are affordable on a GPU).  Estimators: Heuristic (Scott, eq. 3),
    Batch (optimize_bandwidth: multistart + L-BFGS-B on eq. 5, Section 3.4),
    Adaptive (Listing 1 online updates over the training boxes, Section 4.1).
    Metric: mean absolute selectivity error on the test boxes.
(2) changing data (Fig. 8): 5-D clusters; the table starts with
    three clusters; each cycle inserts a new cluster gradually (reservoir
    sampling) and deletes the oldest cluster; DT boxes are biased
    towards newer clusters.  Heuristic keeps Scott's h and only reservoir
    inserts; Adaptive adds the online bandwidth updates and karma-based
    replacement with replacement rows sampled from the current
    table.  Metric: mean absolute error of the boxes of each cycle.
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sigmod_heimelkm15_b200 as K  # noqa: E402
import synth  # noqa: E402
from paper_conf_sigmod_heimelkm15_b200.optimize import optimize_bandwidth  # noqa: E402


def count_true(R, lo, hi):
    import torch
    dR = torch.from_numpy(np.ascontiguousarray(R, np.float32)).cuda()
    dlo, dhi = torch.from_numpy(lo).cuda(), torch.from_numpy(hi).cuda()
    c = torch.zeros(len(lo), dtype=torch.int64, device="cuda")
    K.kde_count_in_box_dev(dR, dlo, dhi, c)
    torch.cuda.synchronize()
    return (c.double() / len(R)).cpu().numpy()


def model_size(quick: bool):
    d = 8
    R = synth.make_data("skew", 1 << 21, d, seed=100)
    lo, hi = synth.workload(R, 200, seed=101, kind="DT", ref_rows=1 << 16)
    p = count_true(R, lo, hi)
    tr, te = slice(0, 100), slice(100, 200)
    sizes = [1 << k for k in (range(10, 21, 2) if not quick else (10, 14))]
    out = []
    g = synth.rng(102)
    for n in sizes:
        S = R[g.choice(len(R), n, replace=False)]
        m = K.KDEModel.create(S)
        row = {"n": n}
        row["heuristic"] = float(np.mean(np.abs(m.estimate(lo[te], hi[te]) - p[te])))
        h0 = m.bandwidth
        t0 = time.perf_counter()
        res = optimize_bandwidth(m, lo[tr], hi[tr], p[tr], loss=K.LOSS_SQUARED, n_starts=16, n_local=3)
        row["batch_seconds"] = time.perf_counter() - t0
        row["batch_evaluations"] = res.evaluations
        row["batch"] = float(np.mean(np.abs(m.estimate(lo[te], hi[te]) - p[te])))
        m.bandwidth = h0
        op = K.online_params(minibatch=10, loss=K.LOSS_SQUARED, log_bandwidth=True)
        for _ in range(3):  # three passes over the training boxes
            for k in range(100):
                m.estimate(lo[k:k + 1], hi[k:k + 1], grad=True)
                m.online_update(lo[k], hi[k], p[k], op)
        row["adaptive"] = float(np.mean(np.abs(m.estimate(lo[te], hi[te]) - p[te])))
        out.append(row)
        print(json.dumps(row), file=sys.stderr, flush=True)
        m.close()
    return out


def changing_data(quick: bool):
    d = 5
    g = synth.rng(200)
    n_sample = 4096
    cl_rows = 60000
    cycles = 10 if not quick else 3

    def cluster(seed):
        c = synth.rng(seed).uniform(0, 100, d)
        return (c + synth.rng(seed + 1).normal(0, 4.0, (cl_rows, d))).astype(np.float32)

    clusters = [cluster(300 + 2 * i) for i in range(3)]
    table = np.concatenate(clusters)
    S = table[g.choice(len(table), n_sample, replace=False)]
    heur = K.KDEModel.create(S)
    adap = K.KDEModel.create(S)
    adap.set_retain(True)
    seen = len(table)
    kp = K.karma_params(loss=K.LOSS_ABSOLUTE, threshold=-1.0 / (n_sample - 1), k_max=4.0)
    op = K.online_params(minibatch=10, loss=K.LOSS_ABSOLUTE, log_bandwidth=True)
    out = []
    for cyc in range(cycles):
        new = cluster(400 + 2 * cyc)
        errs_h, errs_a, replaced = [], [], 0
        chunk = cl_rows // 10
        for part in range(10):
            rows = new[part * chunk:(part + 1) * chunk]
            table = np.concatenate([table, rows])
            # reservoir sampling of the inserted rows (Vitter's Algorithm R), host-side decisions
            ins_idx, ins_rows = [], {}
            for r in rows:
                seen += 1
                j = int(g.integers(0, seen))
                if j < n_sample:
                    ins_rows[j] = r
            if ins_rows:
                idx = np.array(sorted(ins_rows), np.int64)
                rr = np.stack([ins_rows[i] for i in idx])
                heur.replace_points(idx, rr)
                adap.replace_points(idx, rr)
            # DT boxes biased towards the newest clusters
            weights = np.arange(1, len(clusters) + 2, dtype=float) ** 2
            src = g.choice(len(weights), 8, p=weights / weights.sum())
            pool = [*clusters, new[:(part + 1) * chunk]]
            for s_ in src:
                c_rows = pool[int(s_)]
                lo, hi = synth.workload(c_rows, 1, seed=int(g.integers(1 << 30)), kind="DT", ref_rows=4096,
                                        target=min(0.5, 0.01 * len(table) / len(c_rows)))
                ptrue = count_true(table, lo, hi)[0]
                errs_h.append(abs(heur.estimate(lo, hi)[0] - ptrue))
                e, _ = adap.estimate(lo, hi, grad=True)
                errs_a.append(abs(e[0] - ptrue))
                idx, nf, _ = adap.karma_update(lo[0], hi[0], ptrue, kp, cap=n_sample)
                adap.online_update(lo[0], hi[0], ptrue, op)
                if nf:
                    repl = table[g.integers(0, len(table), nf)]
                    adap.replace_points(idx, repl)
                    replaced += nf
        # delete the oldest cluster from the table (the sample only learns about it through karma)
        old = clusters.pop(0)
        table = np.concatenate([*clusters, new])
        clusters.append(new)
        row = {"cycle": cyc, "heuristic_mae": float(np.mean(errs_h)), "adaptive_mae": float(np.mean(errs_a)),
               "karma_replaced": int(replaced), "table_rows": int(len(table))}
        out.append(row)
        print(json.dumps(row), file=sys.stderr, flush=True)
        del old
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--quick", action="store_true")
    args = ap.parse_args()
    res = {"model_size": model_size(args.quick), "changing_data": changing_data(args.quick)}
    print(json.dumps(res, indent=1))


if __name__ == "__main__":
    main()
