"""Batch bandwidth optimisation driver (paper Section 3.3-3.4, 5.3).

The paper solves problem (5)

    H* = argmin_H (1/q) sum_k L(p_hat_H(Omega_k), p_k)   s.t. h > 0

with NLopt: a coarse global stage (MLSL) followed by a local
L-BFGS-B refinement, every objective evaluation running the estimate and
its gradient (eq. 17) on the GPU.  This module is that host-side
driver over the C-ABI call ``kde_loss_and_grad`` (all arithmetic stays in
libkde's kernels):

* the search runs in log-bandwidth space theta = ln h (eq. 18), which
  removes the positivity constraint; the gradient w.r.t. theta is exactly
  what ``kde_loss_and_grad(..., log_bandwidth=True)`` returns;
* global stage: a multistart in the spirit of MLSL -- a scrambled Sobol
  design of start points around the current (e.g. Scott) bandwidth, each
  evaluated once; local searches start from the best few, skipping starts
  that lie within a critical distance of a better one (the MLSL clustering
  rule, simplified);
* local stage: SciPy's L-BFGS-B (the algorithm of [8]) with box bounds on
  theta (a generous band around the start, P:L146's h > 0 made explicit).

``QueryRing`` keeps the last q user queries with their observed
selectivities ("keeping the last q user queries in a ring buffer").
"""
from __future__ import annotations

from dataclasses import dataclass, field

import numpy as np

from . import LOSS_SQUARED, KDEModel


class QueryRing:
    """Ring buffer of the last ``capacity`` (lo, hi, true selectivity) triples."""

    def __init__(self, capacity: int, d: int):
        self.capacity = int(capacity)
        self.lo = np.zeros((capacity, d), np.float32)
        self.hi = np.zeros((capacity, d), np.float32)
        self.p = np.zeros(capacity, np.float64)
        self.n = 0
        self.head = 0

    def push(self, lo, hi, p: float):
        self.lo[self.head] = lo
        self.hi[self.head] = hi
        self.p[self.head] = p
        self.head = (self.head + 1) % self.capacity
        self.n = min(self.n + 1, self.capacity)

    def arrays(self):
        """The stored queries, oldest first."""
        if self.n < self.capacity:
            return self.lo[:self.n].copy(), self.hi[:self.n].copy(), self.p[:self.n].copy()
        idx = (np.arange(self.capacity) + self.head) % self.capacity
        return self.lo[idx], self.hi[idx], self.p[idx]


@dataclass
class OptimizeResult:
    h: np.ndarray
    loss: float
    loss_start: float
    h_start: np.ndarray
    evaluations: int
    local_runs: list = field(default_factory=list)


def _sobol(n: int, d: int, seed: int) -> np.ndarray:
    from scipy.stats import qmc
    m = int(np.ceil(np.log2(max(n, 2))))
    return qmc.Sobol(d, scramble=True, seed=seed).random_base2(m)[:n]


def optimize_bandwidth(model: KDEModel, lo, hi, true_sel, loss: int = LOSS_SQUARED, lam: float = 0.0,
                       n_starts: int = 16, n_local: int = 3, spread: float = 3.0, maxiter: int = 60,
                       seed: int = 0, set_result: bool = True) -> OptimizeResult:
    """Minimise eq. (5) over the diagonal bandwidth (Section 3.4 step 3).

    ``spread``: start points cover theta_0 +- ln(spread) per dimension (Sobol);
    the L-BFGS-B box is theta_0 +- ln(spread^3).  Returns the best bandwidth
    found; with ``set_result`` the model keeps it ("which we then
    transfer to the graphics card")."""
    from scipy.optimize import minimize

    lo = np.ascontiguousarray(lo, np.float32)
    hi = np.ascontiguousarray(hi, np.float32)
    p = np.ascontiguousarray(true_sel, np.float64)
    h0 = model.bandwidth.copy()
    th0 = np.log(h0)
    d = len(h0)
    evals = [0]

    def f(theta):
        model.bandwidth = np.exp(theta)
        L, g = model.loss_and_grad(lo, hi, p, loss, lam, log_bandwidth=True)
        evals[0] += 1
        return L, g

    L0, _ = f(th0)
    # global stage: Sobol multistart around theta_0
    w = np.log(spread)
    starts = th0 + (2.0 * _sobol(n_starts, d, seed) - 1.0) * w
    starts = np.vstack([th0[None], starts])
    vals = np.array([f(s)[0] for s in starts])
    order = np.argsort(vals)
    crit = 0.25 * w  # MLSL-style critical distance (in theta units)
    chosen = []
    for i in order:
        if all(np.max(np.abs(starts[i] - starts[j])) > crit for j in chosen):
            chosen.append(i)
        if len(chosen) >= n_local:
            break
    bounds = [(t - 3 * w, t + 3 * w) for t in th0]
    best_th, best_L = th0, L0
    runs = []
    for i in chosen:
        r = minimize(f, starts[i], jac=True, method="L-BFGS-B", bounds=bounds,
                     options={"maxiter": maxiter, "ftol": 1e-12, "gtol": 1e-12})
        runs.append({"start": float(vals[i]), "final": float(r.fun), "iters": int(r.nit), "msg": str(r.message)})
        if r.fun < best_L:
            best_L, best_th = float(r.fun), r.x
    h_best = np.exp(best_th)
    model.bandwidth = h_best if set_result else h0
    return OptimizeResult(h=h_best, loss=best_L, loss_start=L0, h_start=h0, evaluations=evals[0], local_runs=runs)
