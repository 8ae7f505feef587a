"""Seeded synthetic inputs shared by tests, bench.py and smoke().

This module holds NONE of the method's arithmetic: it only draws data
samples, query boxes and replacement rows with numpy's PCG64, so the same
arrays can be fed to the CUDA path and to the oracle.  Values are drawn in
fp64 and rounded to fp32 once.  Recipes:

  G-A  correlated Gaussian clusters (north star): 16 clusters, centres
       U[0,100]^d, covariance Q diag(s^2) Q^T with Q random orthogonal and
       s ~ U[1,8], Zipf(1) cluster weights (skew), 2% uniform noise over the
       bounding box (noise as in the paper's synthetic set).
  G-B  the synthetic set of [14] as described at P:L279: random
       hyper-rectangular clusters with uniform interiors plus uniform noise.
  G-C  real-data-like skew: Gaussian copula with random
       correlation, marginals mixing log-normal, Pareto(1.5) and exponential;
       two columns discretised to integers (ties), one column offset by 1e4.
  Q-R  random boxes: per dimension two U[min,max] draws, sorted.
  DT/DV/UT/UV (after [7]): centre is a random data row (D) or
       uniform in the bounding box (U); T = hypercube in sigma-scaled units
       whose half-side is the 1%-quantile of the sigma-scaled Chebyshev
       distance from the centre over a reference subsample (1% selectivity),
       V = side 0.01^(1/d) of the range per dimension (1% of the volume).
"""
from __future__ import annotations

import numpy as np

MASTER_SEED = 20150531


def rng(seed: int, stream: int = 0) -> np.random.Generator:
    return np.random.default_rng([int(seed), int(stream), MASTER_SEED])


# ---------------------------------------------------------------- data
def _random_orthogonal(g: np.random.Generator, d: int) -> np.ndarray:
    a = g.normal(size=(d, d))
    q, r = np.linalg.qr(a)
    return q * np.sign(np.diag(r))


def gaussian_clusters(n: int, d: int, seed: int, n_clusters: int = 16, noise: float = 0.02) -> np.ndarray:
    """G-A: correlated Gaussian clusters with Zipf(1) weights plus uniform noise."""
    g = rng(seed, 1)
    centres = g.uniform(0, 100, size=(n_clusters, d))
    w = 1.0 / np.arange(1, n_clusters + 1)
    w /= w.sum()
    n_noise = int(round(noise * n))
    n_cl = n - n_noise
    counts = g.multinomial(n_cl, w)
    out = np.empty((n, d), dtype=np.float32)
    pos = 0
    for c in range(n_clusters):
        k = int(counts[c])
        if k == 0:
            continue
        Q = _random_orthogonal(g, d)
        s = g.uniform(1, 8, size=d)
        L = Q * s  # covariance Q diag(s^2) Q^T = L L^T
        # chunked to bound temporary memory for very large n
        for a in range(0, k, 1 << 22):
            b = min(k, a + (1 << 22))
            z = g.standard_normal(size=(b - a, d))
            out[pos + a:pos + b] = (centres[c] + z @ L.T).astype(np.float32)
        pos += k
    if n_noise:
        lo = out[:pos].min(axis=0).astype(np.float64)
        hi = out[:pos].max(axis=0).astype(np.float64)
        out[pos:] = g.uniform(lo, hi, size=(n_noise, d)).astype(np.float32)
    perm = g.permutation(n)
    return out[perm]


def gaussian_clusters_rows(n_global: int, d: int, seed: int, row0: int, row1: int, n_clusters: int = 16,
                           noise: float = 0.02, chunk: int = 1 << 20) -> np.ndarray:
    """Rows [row0, row1) of a G-A-shaped sample of n_global rows, generated chunk by chunk
    (chunk c = rows [c*chunk, (c+1)*chunk) from its own stream), so any rank can draw exactly its
    contiguous shard and every world size sees the same global sample (strong scaling, C4).
    Each row picks a cluster by Zipf(1) weight (prob 1-noise) or uniform noise over [-25, 125]^d."""
    g = rng(seed, 40)
    centres = g.uniform(0, 100, size=(n_clusters, d))
    Ls = []
    for _ in range(n_clusters):
        Q = _random_orthogonal(g, d)
        Ls.append(Q * g.uniform(1, 8, size=d))
    w = 1.0 / np.arange(1, n_clusters + 1)
    w = np.concatenate([(1.0 - noise) * w / w.sum(), [noise]])
    out = np.empty((max(0, row1 - row0), d), dtype=np.float32)
    for c in range(row0 // chunk, (row1 + chunk - 1) // chunk):
        a, b = c * chunk, min(n_global, (c + 1) * chunk)
        gc = rng(seed, 100000 + c)
        lab = gc.choice(n_clusters + 1, size=b - a, p=w)
        z = gc.standard_normal(size=(b - a, d))
        x = np.empty((b - a, d))
        for k in range(n_clusters):
            sel = lab == k
            x[sel] = centres[k] + z[sel] @ Ls[k].T
        sel = lab == n_clusters
        x[sel] = gc.uniform(-25.0, 125.0, size=(int(sel.sum()), d))
        lo_, hi_ = max(a, row0), min(b, row1)
        out[lo_ - row0:hi_ - row0] = x[lo_ - a:hi_ - a].astype(np.float32)
    return out


class StreamClusters:
    """The insert/delete stream of configs[4] (after P:L367-373): the database
    is a sequence of Gaussian clusters of `rows` rows each (cluster c: its own centre in [0, 100]^d,
    rotation and scales U[1, 8]); cycle t inserts cluster t + 2 in chunks and deletes cluster t - 1.
    Queries are DT boxes centred on rows of live clusters, cluster c drawn with P ~ 2^c (newer
    clusters are asked more), sized to ~1% selectivity within their cluster."""

    def __init__(self, d: int, rows: int, seed: int):
        self.d, self.rows, self.seed = d, rows, seed

    def _params(self, c: int):
        g = rng(self.seed, 50000 + c)
        return g.uniform(0, 100, size=self.d), _random_orthogonal(g, self.d) * g.uniform(1, 8, size=self.d)

    def cluster_rows(self, c: int, a: int = 0, b: int | None = None) -> np.ndarray:
        """Rows [a, b) of cluster c (generated in 2^16-row pieces from their own streams)."""
        b = self.rows if b is None else b
        centre, L = self._params(c)
        piece = 1 << 16
        out = np.empty((b - a, self.d), dtype=np.float32)
        for p in range(a // piece, (b + piece - 1) // piece):
            z = rng(self.seed, 60000 + 4096 * c + p).standard_normal(size=(piece, self.d))
            x = (centre + z @ L.T).astype(np.float32)
            lo_, hi_ = max(a, p * piece), min(b, (p + 1) * piece)
            out[lo_ - a:hi_ - a] = x[lo_ - p * piece:hi_ - p * piece]
        return out

    def queries(self, live: list, q: int, seed: int):
        """q DT boxes over the live clusters, cluster c with probability ~ 2^c."""
        g = rng(seed, 70)
        w = np.array([2.0 ** c for c in live])
        pick = g.choice(len(live), size=q, p=w / w.sum())
        lo = np.empty((q, self.d), np.float32)
        hi = np.empty((q, self.d), np.float32)
        for i, k in enumerate(pick):
            c = live[k]
            centre, L = self._params(c)
            row = (centre + g.standard_normal(self.d) @ L.T)
            # half-side in each axis: the cluster's per-axis sd times the 1%-volume factor
            sd = np.sqrt((L ** 2).sum(axis=1))
            half = sd * 0.5 * 0.01 ** (1.0 / self.d) * 4.0
            lo[i] = (row - half).astype(np.float32)
            hi[i] = (row + half).astype(np.float32)
        return lo, hi


def rect_clusters(n: int, d: int, seed: int, n_clusters: int = 10, noise: float = 0.1) -> np.ndarray:
    """G-B: hyper-rectangular clusters with uniform interiors plus uniform noise."""
    g = rng(seed, 2)
    n_noise = int(round(noise * n))
    counts = g.multinomial(n - n_noise, np.full(n_clusters, 1.0 / n_clusters))
    parts = []
    for c in range(n_clusters):
        lo = g.uniform(0, 80, size=d)
        side = g.uniform(2, 20, size=d)
        parts.append(g.uniform(lo, lo + side, size=(int(counts[c]), d)))
    parts.append(g.uniform(0, 100, size=(n_noise, d)))
    out = np.concatenate(parts).astype(np.float32)
    return out[g.permutation(n)]


def skewed_real_like(n: int, d: int, seed: int) -> np.ndarray:
    """G-C: Gaussian copula, heavy-tailed marginals, ties, a large offset."""
    from scipy.special import ndtr
    g = rng(seed, 3)
    A = g.uniform(-1, 1, size=(d, d))
    C = A @ A.T + 0.1 * np.eye(d)
    s = np.sqrt(np.diag(C))
    C = C / np.outer(s, s)
    C = np.clip(C, -0.9, 0.9)
    np.fill_diagonal(C, 1.0)
    w, V = np.linalg.eigh(C)
    L = V * np.sqrt(np.clip(w, 1e-6, None))
    z = g.standard_normal(size=(n, d)) @ L.T
    u = np.clip(ndtr(z), 1e-12, 1 - 1e-12)
    out = np.empty((n, d))
    for j in range(d):
        kind = j % 3
        if kind == 0:
            out[:, j] = np.exp(z[:, j])  # log-normal(sigma=1)
        elif kind == 1:
            out[:, j] = (1 - u[:, j]) ** (-1 / 1.5)  # Pareto(1.5)
        else:
            out[:, j] = -np.log(1 - u[:, j])  # exponential
    if d >= 2:
        out[:, 0] = np.round(out[:, 0] * 4)
    if d >= 3:
        out[:, 2] = np.round(out[:, 2] * 10)
    out[:, d - 1] += 1e4
    return out.astype(np.float32)


def make_data(kind: str, n: int, d: int, seed: int) -> np.ndarray:
    return {"gauss": gaussian_clusters, "rect": rect_clusters, "skew": skewed_real_like}[kind](n, d, seed)


# ---------------------------------------------------------------- queries
def random_boxes(data: np.ndarray, q: int, seed: int):
    """Q-R: per dimension two uniform draws in [min, max], sorted."""
    g = rng(seed, 10)
    lo_d = data.min(axis=0).astype(np.float64)
    hi_d = data.max(axis=0).astype(np.float64)
    a = g.uniform(lo_d, hi_d, size=(q, data.shape[1]))
    b = g.uniform(lo_d, hi_d, size=(q, data.shape[1]))
    return np.minimum(a, b).astype(np.float32), np.maximum(a, b).astype(np.float32)


def _count(ref: np.ndarray, lo: np.ndarray, hi: np.ndarray) -> int:
    return int(np.count_nonzero(np.all((ref > lo) & (ref < hi), axis=1)))


def workload(data: np.ndarray, q: int, seed: int, kind: str = "DT", ref_rows: int = 1 << 15,
             target: float = 0.01):
    """DT / DV / UT / UV boxes.  T-queries size a hypercube (in
    per-dimension sigma units) to reach ``target`` selectivity on a
    ``ref_rows`` subsample of ``data``; V-queries take side 0.01^(1/d) of the
    range (1% of the data space volume)."""
    g = rng(seed, 11 + "DT DV UT UV".split().index(kind))
    n, d = data.shape
    ref = data[g.choice(n, size=min(n, ref_rows), replace=False)].astype(np.float64)
    lo_d, hi_d = ref.min(axis=0), ref.max(axis=0)
    rng_d = hi_d - lo_d
    sig = ref.std(axis=0)
    if kind[0] == "D":
        centres = data[g.integers(0, n, size=q)].astype(np.float64)
    else:
        centres = g.uniform(lo_d, hi_d, size=(q, d))
    lo = np.empty((q, d))
    hi = np.empty((q, d))
    if kind[1] == "V":
        half = 0.5 * rng_d * target ** (1.0 / d)
        lo[:] = centres - half
        hi[:] = centres + half
    else:
        # the hypercube side that captures `target` of the reference rows is the
        # k-th smallest sigma-scaled Chebyshev distance from the centre
        k_th = max(0, min(len(ref) - 1, int(round(target * len(ref)))))
        for a0 in range(0, q, 256):
            c = centres[a0:a0 + 256]
            dist = np.max(np.abs(ref[None] - c[:, None]) / sig, axis=2)
            m = np.partition(dist, k_th, axis=1)[:, k_th]
            lo[a0:a0 + 256] = c - m[:, None] * sig
            hi[a0:a0 + 256] = c + m[:, None] * sig
    return lo.astype(np.float32), hi.astype(np.float32)


def mixed_workload(data: np.ndarray, q: int, seed: int, ref_rows: int = 1 << 12):
    """25% each of DT / DV / UT / UV, interleaved in a seeded order."""
    per = [q // 4 + (1 if i < q % 4 else 0) for i in range(4)]
    parts = [workload(data, per[i], seed + i, k, ref_rows) for i, k in enumerate("DT DV UT UV".split())]
    lo = np.concatenate([p[0] for p in parts])
    hi = np.concatenate([p[1] for p in parts])
    perm = rng(seed, 20).permutation(q)
    return lo[perm], hi[perm]


def true_selectivity_cpu(R: np.ndarray, lo: np.ndarray, hi: np.ndarray) -> np.ndarray:
    """Exact |sigma_{x in Omega}(R)| / |R| by counting (the feedback of P:L240).
    Open box (l, u) as in P:L45.  CPU, for small R only."""
    out = np.empty(len(lo))
    for k in range(len(lo)):
        out[k] = _count(R, lo[k], hi[k]) / len(R)
    return out


def special_boxes(data: np.ndarray, seed: int):
    """Edge-case boxes: unbounded, half-open, l == u, narrow (w << h), far tail."""
    g = rng(seed, 30)
    n, d = data.shape
    lo_d = data.min(axis=0)
    hi_d = data.max(axis=0)
    mid = data[g.integers(0, n)]
    inf = np.float32(np.inf)
    boxes = []
    boxes.append((np.full(d, -inf), np.full(d, inf)))                       # unbounded
    l = np.full(d, -inf); l[0] = mid[0]; boxes.append((l, np.full(d, inf)))  # half-open
    u = np.full(d, inf); u[-1] = mid[-1]; boxes.append((np.full(d, -inf), u))
    boxes.append((mid.copy(), mid.copy()))                                   # l == u
    w = (hi_d - lo_d) * 1e-4
    boxes.append((mid - w, mid + w))                                         # narrow
    boxes.append((hi_d + (hi_d - lo_d), hi_d + 2 * (hi_d - lo_d)))           # far tail
    lo = np.array([b[0] for b in boxes], np.float32)
    hi = np.array([b[1] for b in boxes], np.float32)
    return lo, hi


def replacement_rows(R: np.ndarray, k: int, seed: int, step: int) -> np.ndarray:
    """The m-th replacement row is R[hash(seed, step, m) mod |R|] (reading 13)."""
    g = rng(seed, 1000 + step)
    return R[g.integers(0, len(R), size=k)].astype(np.float32)
