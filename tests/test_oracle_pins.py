"""Pins the fp64 oracle to things other than itself (CPU only, ``-m "not gpu"``).

Each test names the PAPER.md passage ("P:L<n>") and what fixes the expected
value: an independent mpmath quadrature fixture, a closed form, an invariant,
a limit, finite differences, or brute force.  A plausible slip in the oracle
(dropped 1/2^d, wrong sign on the l-term of eq. 17, swapped u/l, sample- vs
population sigma, wrong leave-one-out denominator, ...) fails at least one.
"""
import json
import math
import os

import mpmath as mp
import numpy as np
import pytest

import oracle

GOLD = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "micro_example.json")))
INF = np.float32(np.inf)


def _micro():
    S = np.array(GOLD["sample"], np.float32)
    h = np.array(GOLD["h"], np.float64)
    lo = np.array([GOLD["lo"]], np.float32)
    hi = np.array([GOLD["hi"]], np.float32)
    return S, h, lo, hi


def _close(a, b, rel=1e-13, abs_=1e-15):
    a = np.asarray(a, np.float64)
    b = np.asarray([float(x) for x in np.atleast_1d(b)], np.float64)
    assert np.all(np.abs(a - b) <= abs_ + rel * np.abs(b)), (a, b)


# --- golden micro example (independent 50-digit quadrature) -----------------

def test_micro_contributions_and_estimate():
    """eq. (13) vs quadrature of eq. (12); eq. (2)."""
    S, h, lo, hi = _micro()
    _close(oracle.contributions(S, h, lo[0], hi[0]), GOLD["contributions"])
    _close(oracle.estimate(S, h, lo, hi), [GOLD["estimate"]])


def test_micro_gradient_and_loss():
    """eq. (17), eq. (18), eq. (14) + C.1 L2."""
    S, h, lo, hi = _micro()
    est, g = oracle.estimate_grad(S, h, lo, hi)
    _close(g[0], GOLD["dpdh"], rel=1e-12)
    L, gL, e2 = oracle.loss_and_grad(S, h, lo, hi, [GOLD["true_sel"]], oracle.LOSS_SQUARED, 0.0, False)
    _close([L], [GOLD["l2_loss"]])
    _close(gL, GOLD["l2_grad"], rel=1e-12)
    _, gl, _ = oracle.loss_and_grad(S, h, lo, hi, [GOLD["true_sel"]], oracle.LOSS_SQUARED, 0.0, True)
    _close(gl, [float(GOLD["l2_grad"][j]) * h[j] for j in range(2)], rel=1e-12)
    _close(g[0] * h, GOLD["dpdlnh"], rel=1e-12)


def test_micro_karma_and_threshold():
    """eq. (6)-(7) and eq. (19)-(20) vs quadrature."""
    S, h, lo, hi = _micro()
    c = oracle.contributions(S, h, lo[0], hi[0])
    est = oracle.estimate(S, h, lo, hi)[0]
    karma = np.zeros(3)
    oracle.karma_update(c, est, GOLD["true_sel"], oracle.LOSS_ABSOLUTE, 0.0, 4.0, -1e9, np.inf, karma)
    _close(karma, GOLD["karma_delta_l1"], rel=1e-12)
    thr, pmax = oracle.empty_region_threshold(h, lo[0], hi[0])
    _close([pmax], [GOLD["p_max"]])
    _close([thr], [GOLD["thr20"]])


def test_micro_scott():
    """eq. (3) with population sigma."""
    S, _, _, _ = _micro()
    _close(oracle.scott(S), GOLD["scott_h"])


# --- closed forms and limits -------------------------------------------------

@pytest.mark.parametrize("t,h,l,u", [(0.3, 0.7, -1.0, 2.0), (5.0, 0.1, 4.8, 5.05), (-2.0, 3.0, 1.0, 9.0),
                                     (0.0, 1.0, -np.inf, 0.5), (1.0, 2.0, 0.0, np.inf),
                                     # far tails (reading R16): Phi(8) - Phi(7) = 1.3e-12, Phi(12) - Phi(9) = 1.1e-19
                                     (0.0, 1.0, 7.0, 8.0), (0.0, 1.0, 9.0, 12.0), (0.0, 1.0, -12.0, -9.0),
                                     (0.0, 0.5, 4.0, np.inf)])
def test_d1_closed_form_vs_mpmath_ncdf(t, h, l, u):
    """d = 1, N = 1: eq. (13) is Phi((u-t)/h) - Phi((l-t)/h)."""
    mp.mp.dps = 40
    ref = mp.ncdf((mp.mpf(float(np.float32(u))) - mp.mpf(float(np.float32(t)))) / h) - \
        mp.ncdf((mp.mpf(float(np.float32(l))) - mp.mpf(float(np.float32(t)))) / h)
    got = oracle.point_mass(np.array([t], np.float32), [h], np.array([l], np.float32), np.array([u], np.float32))
    assert abs(got - float(ref)) <= 2e-16 + 1e-14 * abs(float(ref))


def test_unbounded_query_is_exactly_one():
    """erf(+-inf) = +-1 makes every factor of eq. (13) exactly 1; eq. (17) is exactly 0."""
    rng = np.random.default_rng(1)
    S = rng.normal(size=(200, 4)).astype(np.float32)
    h = rng.uniform(0.1, 2, 4)
    lo = np.full((1, 4), -INF, np.float32)
    hi = np.full((1, 4), INF, np.float32)
    est, g = oracle.estimate_grad(S, h, lo, hi)
    assert est[0] == 1.0
    assert np.all(g == 0.0)


def test_product_factorisation_and_marginalisation():
    """Product kernel: with all other dims unbounded, the d-dim estimate
    equals the 1-D estimate on column j; for N = 1 the mass is the product of 1-D masses."""
    rng = np.random.default_rng(2)
    S = rng.normal(size=(64, 3)).astype(np.float32)
    h = np.array([0.3, 0.8, 1.7])
    lo = np.array([-0.4, 0.1, -2.0], np.float32)
    hi = np.array([0.9, 1.1, 0.5], np.float32)
    for j in range(3):
        l2 = np.full(3, -INF, np.float32)
        u2 = np.full(3, INF, np.float32)
        l2[j], u2[j] = lo[j], hi[j]
        a = oracle.estimate(S, h, l2[None], u2[None])[0]
        b = oracle.estimate(S[:, j:j + 1], h[j:j + 1], lo[None, j:j + 1], hi[None, j:j + 1])[0]
        assert a == pytest.approx(b, rel=1e-15, abs=1e-16)
    t = S[0]
    prod = np.prod([oracle.point_mass(t[j:j + 1], h[j:j + 1], lo[j:j + 1], hi[j:j + 1]) for j in range(3)])
    assert oracle.point_mass(t, h, lo, hi) == pytest.approx(prod, rel=1e-14)


def test_additivity_along_a_dimension():
    """The box integral eq. (12) is additive: [l,c] + [c,u] = [l,u] on any axis."""
    rng = np.random.default_rng(3)
    S = rng.normal(size=(128, 3)).astype(np.float32)
    h = np.array([0.5, 0.25, 1.5])
    lo = np.array([-1.0, -0.5, -2.0], np.float32)
    hi = np.array([1.0, 0.75, 0.25], np.float32)
    for j in range(3):
        c = np.float32(0.125)
        hi1 = hi.copy(); hi1[j] = c
        lo2 = lo.copy(); lo2[j] = c
        a = oracle.estimate(S, h, lo[None], hi1[None])[0] + oracle.estimate(S, h, lo2[None], hi[None])[0]
        b = oracle.estimate(S, h, lo[None], hi[None])[0]
        assert a == pytest.approx(b, rel=1e-13, abs=1e-16)


def test_lower_equals_upper_gives_zero():
    """An empty interval has zero mass (eq. 12 integral over (l, l))."""
    S = np.array([[0.0, 1.0], [2.0, -1.0]], np.float32)
    est = oracle.estimate(S, [1.0, 1.0], np.array([[0.5, -3]], np.float32), np.array([[0.5, 3]], np.float32))
    assert est[0] == 0.0


def test_invariances():
    """Translation of (t, l, u), joint scaling of (t, l, u, h) by 2 (exact in fp32),
    and reflection t -> -t, (l, u) -> (-u, -l) leave eq. (13) unchanged."""
    rng = np.random.default_rng(4)
    # values on a 2^-10 grid so that adding 8 and scaling by 2 are exact in fp32
    S = (np.round(rng.normal(size=(100, 2)) * 1024) / 1024).astype(np.float32)
    h = np.array([0.4, 0.9])
    lo = np.array([[-0.5, -1.0]], np.float32)
    hi = np.array([[0.75, 0.5]], np.float32)
    base = oracle.estimate(S, h, lo, hi)[0]
    shift = np.float32(8.0)
    assert oracle.estimate(S + shift, h, lo + shift, hi + shift)[0] == pytest.approx(base, rel=1e-12)
    assert oracle.estimate(S * 2, h * 2, lo * 2, hi * 2)[0] == pytest.approx(base, rel=1e-14)
    assert oracle.estimate(-S, h, -hi, -lo)[0] == pytest.approx(base, rel=1e-14)


def test_small_bandwidth_limit_is_exact_count():
    """h -> 0 degrades to counting: with every point >= 10h from every
    face, each erf is exactly +-1 in fp64, so p_hat == count/N exactly."""
    rng = np.random.default_rng(5)
    S = rng.integers(-50, 50, size=(500, 3)).astype(np.float32)
    h = np.full(3, 0.01)
    lo = np.array([[-20.5, -10.5, -30.5]], np.float32)
    hi = np.array([[15.5, 30.5, 5.5]], np.float32)
    inside = np.all((S > lo) & (S < hi), axis=1).sum()
    assert oracle.estimate(S, h, lo, hi)[0] == inside / 500.0


# --- gradient: finite differences ---------------------------------------------

@pytest.mark.parametrize("log_bw", [False, True])
def test_gradient_matches_central_differences(log_bw):
    """eq. (17) and eq. (18) vs central FD of eq. (2)+(13)."""
    rng = np.random.default_rng(6)
    S = rng.normal(size=(50, 3)).astype(np.float32)
    h = np.array([0.3, 0.6, 1.1])
    lo = np.array([[-0.5, -1.0, -np.inf]], np.float32)
    hi = np.array([[0.8, 0.4, 0.9]], np.float32)
    est, g = oracle.estimate_grad(S, h, lo, hi)
    for j in range(3):
        if log_bw:
            dl = 1e-6
            hp, hm = h.copy(), h.copy()
            hp[j] = h[j] * math.exp(dl); hm[j] = h[j] * math.exp(-dl)
            fd = (oracle.estimate(S, hp, lo, hi)[0] - oracle.estimate(S, hm, lo, hi)[0]) / (2 * dl)
            ana = g[0, j] * h[j]
        else:
            dh = 1e-6 * h[j]
            hp, hm = h.copy(), h.copy()
            hp[j] += dh; hm[j] -= dh
            fd = (oracle.estimate(S, hp, lo, hi)[0] - oracle.estimate(S, hm, lo, hi)[0]) / (2 * dh)
            ana = g[0, j]
        assert ana == pytest.approx(fd, rel=1e-7, abs=1e-12)


@pytest.mark.parametrize("kind", range(5))
def test_loss_derivatives_match_finite_differences(kind):
    """C.1 derivatives vs central FD of the listed loss, away from kinks."""
    lam = 1e-3
    for phat, p in [(0.3, 0.1), (0.05, 0.2), (0.6, 0.61)]:
        L, dL = oracle.loss(kind, lam, phat, p)
        e = 1e-7
        fd = (oracle.loss(kind, lam, phat + e, p)[0] - oracle.loss(kind, lam, phat - e, p)[0]) / (2 * e)
        assert dL == pytest.approx(fd, rel=1e-6)


def test_loss_values_and_kinks():
    """C.1 values and the printed 0 derivative at equality for L1/relative."""
    lam = 0.01
    assert oracle.loss(0, lam, 0.3, 0.1)[0] == pytest.approx(0.04)
    assert oracle.loss(1, lam, 0.3, 0.1)[0] == pytest.approx(0.2)
    assert oracle.loss(2, lam, 0.3, 0.1)[0] == pytest.approx(0.2 / 0.11)
    assert oracle.loss(3, lam, 0.3, 0.1)[0] == pytest.approx((0.2 / 0.11) ** 2)
    assert oracle.loss(4, lam, 0.3, 0.1)[0] == pytest.approx((math.log(0.31) - math.log(0.11)) ** 2)
    assert oracle.loss(1, lam, 0.2, 0.2)[1] == 0.0
    assert oracle.loss(2, lam, 0.2, 0.2)[1] == 0.0
    assert oracle.loss(1, lam, 0.1, 0.2)[1] == -1.0
    assert oracle.loss(2, lam, 0.3, 0.2)[1] == pytest.approx(1 / 0.21)


def test_loss_and_grad_averages_over_queries():
    """eq. (5): loss and gradient are means over the q training queries."""
    rng = np.random.default_rng(7)
    S = rng.normal(size=(40, 2)).astype(np.float32)
    h = np.array([0.5, 0.7])
    lo = np.array([[-1, -1], [0, -0.5], [-2, 0.2]], np.float32)
    hi = np.array([[0.5, 1], [1, 0.5], [0, 2]], np.float32)
    p = np.array([0.2, 0.1, 0.3])
    L, g, est = oracle.loss_and_grad(S, h, lo, hi, p, 0, 0.0, False)
    Ls, gs = [], []
    for k in range(3):
        l1, g1, _ = oracle.loss_and_grad(S, h, lo[k:k + 1], hi[k:k + 1], p[k:k + 1], 0, 0.0, False)
        Ls.append(l1); gs.append(g1)
    assert L == pytest.approx(np.mean(Ls), rel=1e-14)
    assert np.allclose(g, np.mean(gs, axis=0), rtol=1e-13)


# --- Scott ----------------------------------------------------------------------

def test_scott_matches_numpy_population_std():
    """eq. (3), population sigma == numpy std(ddof=0)."""
    rng = np.random.default_rng(8)
    S = (rng.normal(size=(1000, 5)) * [1, 2, 3, 0.5, 10] + 1e3).astype(np.float32)
    ref = 1000 ** (-1 / 9) * S.astype(np.float64).std(axis=0, ddof=0)
    assert np.allclose(oracle.scott(S), ref, rtol=1e-12)


# --- karma ------------------------------------------------------------------------

def test_leave_one_out_matches_brute_force():
    """eq. (6) equals re-estimating on S \\ {t_i}."""
    rng = np.random.default_rng(9)
    S = rng.normal(size=(12, 2)).astype(np.float32)
    h = np.array([0.4, 0.6])
    lo = np.array([-0.5, -0.2], np.float32)
    hi = np.array([0.7, 1.0], np.float32)
    c = oracle.contributions(S, h, lo, hi)
    est = oracle.estimate(S, h, lo[None], hi[None])[0]
    p = 0.3
    karma = np.zeros(12)
    oracle.karma_update(c, est, p, oracle.LOSS_SQUARED, 0.0, 1e9, -1e9, np.inf, karma)
    for i in range(12):
        loo = oracle.estimate(np.delete(S, i, axis=0), h, lo[None], hi[None])[0]
        assert karma[i] == pytest.approx((loo - p) ** 2 - (est - p) ** 2, rel=1e-9, abs=1e-15)


def test_karma_saturation_and_threshold_by_hand():
    """eq. (8) min(K + dK, K_max) and the strict threshold of P:L204/L250, N = 4."""
    c = np.array([0.9, 0.1, 0.0, 0.5])
    n = 4
    phat = c.mean()
    p = 0.2
    # L1: L(p_hat) = |0.375 - 0.2| = 0.175; p^-(i) = (1.5 - c_i)/3
    loo = (phat * n - c) / (n - 1)
    dK = np.abs(loo - p) - abs(phat - p)
    karma = np.array([3.99, 0.0, -0.05, 0.0])
    k_max, tau = 4.0, -0.02
    idx = oracle.karma_update(c, phat, p, oracle.LOSS_ABSOLUTE, 0.0, k_max, tau, np.inf, karma)
    expect = np.minimum(np.array([3.99, 0.0, -0.05, 0.0]) + dK, k_max)
    assert np.allclose(karma, expect, rtol=0, atol=1e-15)
    assert list(idx) == [i for i in range(4) if expect[i] < tau]
    assert karma[0] <= k_max


def test_empty_region_rule_flags_only_inside_points():
    """P:L250 + eq. (20): with true selectivity 0 a point is flagged when its
    contribution reaches thr_20; such points are always inside the box."""
    rng = np.random.default_rng(10)
    for trial in range(30):
        d = rng.integers(1, 5)
        h = rng.uniform(0.05, 1.0, d)
        lo = rng.uniform(-1, 0, d).astype(np.float32)
        hi = (lo + rng.uniform(0.05, 2.0, d)).astype(np.float32)
        S = rng.uniform(-2, 2, size=(4000, d)).astype(np.float32)
        c = oracle.contributions(S, h, lo, hi)
        thr, pmax = oracle.empty_region_threshold(h, lo, hi)
        karma = np.zeros(len(S))
        idx = oracle.karma_update(c, c.mean(), 0.0, oracle.LOSS_ABSOLUTE, 0.0, 4.0, -1e300, thr, karma)
        inside = np.all((S >= lo) & (S <= hi), axis=1)
        assert inside[idx].all()
        assert c.max() <= pmax * (1 + 1e-12)


def test_eq19_centre_and_eq20_boundary_points():
    """eq. (19): the box centre attains p_max; eq. (20): the threshold is the
    largest mass among the centre moved to a face along one dimension."""
    h = np.array([0.3, 1.2, 0.7])
    lo = np.array([-1.0, 0.0, 2.0], np.float32)
    hi = np.array([0.5, 3.0, 2.5], np.float32)
    centre = ((lo.astype(np.float64) + hi) / 2).astype(np.float32)
    thr, pmax = oracle.empty_region_threshold(h, lo, hi)
    assert oracle.point_mass(centre, h, lo, hi) == pytest.approx(pmax, rel=1e-14)
    faces = []
    for j in range(3):
        t = centre.copy(); t[j] = lo[j]
        faces.append(oracle.point_mass(t, h, lo, hi))
    assert thr == pytest.approx(max(faces), rel=1e-13)
    # zero width disables the shortcut
    thr0, _ = oracle.empty_region_threshold(h, lo, lo)
    assert thr0 == np.inf


# --- Listing 1 (reconstruction, PARITY UNPINNED): sanity property only -----------

def test_online_update_reduces_training_loss():
    """Sanity property for the reconstructed Listing 1: on a static
    workload, SGD with the RMSprop-style step lowers the L2 loss from Scott's h."""
    rng = np.random.default_rng(11)
    R = np.concatenate([rng.normal(0, 0.3, (3000, 2)), rng.normal(3, 0.5, (3000, 2))]).astype(np.float32)
    S = R[rng.choice(len(R), 256, replace=False)]
    h = oracle.scott(S)
    c = R[rng.choice(len(R), 200)]
    w = rng.uniform(0.2, 1.0, (200, 2))
    lo = (c - w / 2).astype(np.float32)
    hi = (c + w / 2).astype(np.float32)
    p = np.array([np.all((R >= lo[k]) & (R <= hi[k]), axis=1).mean() for k in range(200)])
    L0, _, _ = oracle.loss_and_grad(S, h, lo, hi, p, 0, 0.0, True)
    st = oracle.OnlineState(2, lr0=0.1)
    for epoch in range(3):
        for k in range(200):
            _, g, _ = oracle.loss_and_grad(S, h, lo[k:k + 1], hi[k:k + 1], p[k:k + 1], 0, 0.0, True)
            oracle.online_step(st, h, g, log_bw=True)
    L1, _, _ = oracle.loss_and_grad(S, h, lo, hi, p, 0, 0.0, True)
    assert L1 < L0


def test_online_listing1_hand_trace_linear_mode():
    """Listing 1 as the prose fixes it, d = 1, mini-batch 2, traced by hand:
    average the mini-batch (line 12); running mean of the SQUARED gradient with alpha = 0.9
    ("average magnitude", RMSprop [42], line 14); rate x1.2 when the directions agree and x0.5
    when they do not (lines 15-16, first batch: no previous direction, rate kept); step
    lr * g / sqrt(ms) (line 17); a step towards zero is limited to half the bandwidth."""
    st = oracle.OnlineState(1, lr0=0.1)
    h = np.array([0.4])
    # batch 1: g = (0.2 + 0.4)/2 = 0.3, ms = 0.1 * 0.09 = 0.009, lr = 0.1 (no previous direction)
    # step = 0.1 * 0.3 / sqrt(0.009) = 0.316228 > h/2 = 0.2  ->  h = 0.4 - 0.2 = 0.2 (safeguard)
    assert not oracle.online_step(st, h, [0.2], batch=2, log_bw=False)
    assert h[0] == 0.4
    assert oracle.online_step(st, h, [0.4], batch=2, log_bw=False)
    assert st.ms[0] == pytest.approx(0.009, rel=1e-15) and st.lr[0] == 0.1
    assert h[0] == pytest.approx(0.2, rel=1e-15)
    # batch 2: g = 0.01 agrees with 0.3 -> lr = 0.12; ms = 0.9 * 0.009 + 0.1 * 1e-4 = 0.00811
    # step = 0.12 * 0.01 / sqrt(0.00811) = 0.0133250... < h/2  ->  h = 0.2 - step
    oracle.online_step(st, h, [0.01], batch=2, log_bw=False)
    oracle.online_step(st, h, [0.01], batch=2, log_bw=False)
    assert st.lr[0] == pytest.approx(0.12, rel=1e-15)
    assert st.ms[0] == pytest.approx(0.00811, rel=1e-14)
    assert h[0] == pytest.approx(0.2 - 0.12 * 0.01 / math.sqrt(0.00811), rel=1e-14)
    h2 = h[0]
    # batch 3: g = -0.05 disagrees -> lr = 0.06; ms = 0.9 * 0.00811 + 0.1 * 0.0025 = 0.007549
    # step = 0.06 * (-0.05) / sqrt(0.007549) < 0: a step away from zero is not limited
    oracle.online_step(st, h, [-0.05], batch=2, log_bw=False)
    oracle.online_step(st, h, [-0.05], batch=2, log_bw=False)
    assert st.lr[0] == pytest.approx(0.06, rel=1e-15)
    assert st.ms[0] == pytest.approx(0.007549, rel=1e-14)
    assert h[0] == pytest.approx(h2 + 0.06 * 0.05 / math.sqrt(0.007549), rel=1e-14)
    assert st.gprev[0] == pytest.approx(-0.05, rel=1e-15) and st.acc[0] == 0.0 and st.count == 0


def test_online_listing1_log_mode_has_no_safeguard():
    """eq. (18) / P:L561: in log mode the update is ln h <- ln h - step and the positivity
    safeguard of line 17 is removed -- a step larger than h/2 (even than h) is taken in full."""
    for lr0 in (0.1, 10.0):
        st = oracle.OnlineState(1, lr0=lr0)
        h = np.array([0.4])
        oracle.online_step(st, h, [0.3], batch=1, log_bw=True)
        step = lr0 * 0.3 / math.sqrt(0.1 * 0.09)          # ms = (1 - alpha) g^2
        assert step > 0.2
        assert h[0] == pytest.approx(0.4 * math.exp(-step), rel=1e-13)
    # the same gradient in linear mode stops at h/2
    st = oracle.OnlineState(1, lr0=10.0)
    h = np.array([0.4])
    oracle.online_step(st, h, [0.3], batch=1, log_bw=False)
    assert h[0] == 0.2


def test_online_listing1_rate_clamps():
    """learning rates stay in [lambda_min, lambda_max] = [1e-6, 50]: forty agreeing
    mini-batches saturate at exactly 50 (0.1 * 1.2^35 > 50), forty alternating ones at 1e-6."""
    st = oracle.OnlineState(2, lr0=0.1)
    h = np.array([0.4, 0.7])
    rates = []
    for k in range(40):
        oracle.online_step(st, h, [1.0, (-1.0) ** k], batch=1, log_bw=False)
        rates.append(st.lr.copy())
    rates = np.array(rates)
    assert rates[-1, 0] == 50.0 and rates[-1, 1] == 1e-6
    # the k-th agreeing batch (k >= 1) multiplies by 1.2 until the cap
    expect_up = np.minimum(0.1 * 1.2 ** np.arange(40), 50.0)
    assert np.allclose(rates[:, 0], expect_up, rtol=1e-12, atol=0)
    expect_dn = np.maximum(0.1 * 0.5 ** np.arange(40), 1e-6)
    assert np.allclose(rates[:, 1], expect_dn, rtol=1e-12, atol=0)
    assert np.all(h > 0)


def test_karma_threshold_is_strict_at_equality():
    """Reading R4: a point is flagged when its karma is BELOW the threshold
    after the update; karma landing exactly on tau is kept.  Binary-exact values (N = 5, L1):
    p^-(i) = (1.25 - c_i)/4, dK = |p^-(i) - 0.25|."""
    c = np.array([0.25, 0.75, 0.0, 0.75, 0.5])
    phat, p, tau = 0.25, 0.25, -0.5
    karma = np.array([-0.625, -0.625, -0.5625, -0.6250001, 0.0])
    idx = oracle.karma_update(c, phat, p, oracle.LOSS_ABSOLUTE, 0.0, 4.0, tau, np.inf, karma)
    # dK = (0, 0.125, 0.0625, 0.125, 0.0625)
    assert karma[1] == tau and karma[2] == tau           # exactly on the threshold: not flagged
    assert karma[3] < tau                                 # just below: flagged
    assert list(idx) == [0, 3]                            # point 0: -0.625 + 0 < tau


def test_grad_abs_scale_is_sum_of_per_point_derivative_magnitudes():
    """The gradient tolerance scale of SURVEY.md §8(c): m_j = (1/N) sum_i |d p^(i)/d h_j|,
    each per-point derivative taken by central finite differences of eq. (13) alone (not eq. 17)."""
    rng = np.random.default_rng(12)
    S = rng.normal(size=(40, 3)).astype(np.float32)
    h = np.array([0.35, 0.8, 1.3])
    lo = np.array([0.1, -1.0, -np.inf], np.float32)
    hi = np.array([0.9, 0.2, 0.4], np.float32)
    m = oracle.grad_abs_scale(S, h, lo[None], hi[None])[0]
    for j in range(3):
        dh = 1e-6 * h[j]
        hp, hm = h.copy(), h.copy()
        hp[j] += dh; hm[j] -= dh
        fd = (oracle.contributions(S, hp, lo, hi) - oracle.contributions(S, hm, lo, hi)) / (2 * dh)
        assert m[j] == pytest.approx(np.abs(fd).mean(), rel=1e-6)
        # and it is never below the magnitude of the gradient itself
        assert m[j] >= abs(oracle.estimate_grad(S, h, lo[None], hi[None])[1][0, j]) * (1 - 1e-12)


# --- property-based pins (hypothesis) ---------------------------------------------
from hypothesis import given, settings, strategies as st  # noqa: E402


@settings(max_examples=60, deadline=None)
@given(seed=st.integers(0, 2**31 - 1), d=st.integers(1, 4), n=st.integers(1, 30))
def test_property_mass_is_a_probability_and_additive(seed, d, n):
    """For any sample, bandwidth and box: 0 <= p_hat <= 1 (eq. 2 averages
    probabilities, eq. 13), splitting the box along a random axis adds up
    (eq. 12 integral), and widening the box never decreases p_hat."""
    g = np.random.default_rng(seed)
    S = g.normal(size=(n, d)).astype(np.float32)
    h = g.uniform(0.05, 3.0, d)
    lo = g.uniform(-2, 0, d).astype(np.float32)
    hi = (lo + g.uniform(0.01, 3, d)).astype(np.float32)
    p = oracle.estimate(S, h, lo[None], hi[None])[0]
    assert -1e-15 <= p <= 1 + 1e-15
    j = int(g.integers(0, d))
    c = np.float32(g.uniform(lo[j], hi[j]))
    h1, l2 = hi.copy(), lo.copy()
    h1[j] = c
    l2[j] = c
    parts = oracle.estimate(S, h, lo[None], h1[None])[0] + oracle.estimate(S, h, l2[None], hi[None])[0]
    assert parts == pytest.approx(p, rel=1e-12, abs=1e-15)
    wide = oracle.estimate(S, h, (lo - 1)[None], (hi + 1)[None])[0]
    assert wide >= p - 1e-15


@settings(max_examples=40, deadline=None)
@given(seed=st.integers(0, 2**31 - 1), d=st.integers(1, 3))
def test_property_gradient_along_h_matches_scaling_derivative(seed, d):
    """Scaling every h_j by (1+e) changes p_hat by sum_j h_j dp/dh_j * e to
    first order (eq. 17 contracted with the direction h)."""
    g = np.random.default_rng(seed)
    S = g.normal(size=(20, d)).astype(np.float32)
    h = g.uniform(0.2, 2.0, d)
    lo = g.uniform(-1.5, 0, d).astype(np.float32)
    hi = (lo + g.uniform(0.2, 2, d)).astype(np.float32)
    _, gr = oracle.estimate_grad(S, h, lo[None], hi[None])
    e = 1e-6
    fd = (oracle.estimate(S, h * (1 + e), lo[None], hi[None])[0]
          - oracle.estimate(S, h * (1 - e), lo[None], hi[None])[0]) / (2 * e)
    assert float(np.dot(h, gr[0])) == pytest.approx(fd, rel=1e-6, abs=1e-13)


# --- Epanechnikov product kernel (NEXT-4, reading R14) ----------------------------
def _epan_quad_mass(t, h, lo, hi):
    """Independent pin: numerical quadrature of the density 3/(4h)(1-(x/h)^2) on |x|<=h."""
    mp.mp.dps = 30
    m = mp.mpf(1)
    for tj, hj, lj, uj in zip(t, h, lo, hi):
        a = max(float(lj), float(tj) - hj)
        b = min(float(uj), float(tj) + hj)
        if b <= a:
            return 0.0
        m *= mp.quad(lambda x: mp.mpf(3) / (4 * hj) * (1 - ((x - float(tj)) / hj) ** 2), [a, b])
    return float(m)


def test_epan_point_mass_matches_quadrature():
    g = np.random.default_rng(20)
    for _ in range(25):
        d = int(g.integers(1, 4))
        t = g.normal(size=d).astype(np.float32)
        h = g.uniform(0.2, 2.0, d)
        lo = g.uniform(-2, 0.5, d).astype(np.float32)
        hi = (lo + g.uniform(0.05, 3, d)).astype(np.float32)
        assert oracle.epan_point_mass(t, h, lo, hi) == pytest.approx(_epan_quad_mass(t, h, lo, hi), rel=1e-12,
                                                                     abs=1e-15)


def test_epan_unbounded_is_one_and_far_is_zero():
    S = np.random.default_rng(21).normal(size=(50, 3)).astype(np.float32)
    h = np.array([0.5, 1.0, 2.0])
    est, g = oracle.epan_estimate_grad(S, h, np.full((1, 3), -np.inf, np.float32), np.full((1, 3), np.inf, np.float32))
    assert est[0] == 1.0 and np.all(g == 0.0)
    far = oracle.epan_estimate(S, h, np.full((1, 3), 100, np.float32), np.full((1, 3), 200, np.float32))
    assert far[0] == 0.0  # compact support: exactly zero


@pytest.mark.parametrize("log_bw", [False, True])
def test_epan_gradient_matches_central_differences(log_bw):
    g = np.random.default_rng(22)
    S = g.normal(size=(60, 3)).astype(np.float32)
    h = np.array([0.7, 1.1, 1.6])
    lo = np.array([[-0.5, -1.0, -np.inf]], np.float32)
    hi = np.array([[0.8, 0.4, 0.9]], np.float32)
    _, gr = oracle.epan_estimate_grad(S, h, lo, hi)
    for j in range(3):
        e = 1e-6
        hp, hm = h.copy(), h.copy()
        hp[j] *= (1 + e)
        hm[j] *= (1 - e)
        fd = (oracle.epan_estimate(S, hp, lo, hi)[0] - oracle.epan_estimate(S, hm, lo, hi)[0]) / (2 * e * h[j])
        assert gr[0, j] == pytest.approx(fd, rel=1e-6, abs=1e-12)


def test_epan_threshold_is_boundary_maximum_and_sound():
    """eq. (19)-(20) derivation for the Epanechnikov kernel: the threshold is the
    largest mass of the centre moved to a face, and no outside point reaches it."""
    h = np.array([0.6, 1.4])
    lo = np.array([-1.0, 0.0], np.float32)
    hi = np.array([0.5, 2.0], np.float32)
    centre = ((lo.astype(np.float64) + hi) / 2).astype(np.float32)
    thr, pmax = oracle.epan_empty_region_threshold(h, lo, hi)
    assert oracle.epan_point_mass(centre, h, lo, hi) == pytest.approx(pmax, rel=1e-14)
    faces = []
    for j in range(2):
        t = centre.copy(); t[j] = lo[j]
        faces.append(oracle.epan_point_mass(t, h, lo, hi))
    assert thr == pytest.approx(max(faces), rel=1e-13)
    S = np.random.default_rng(23).uniform(-3, 3, size=(20000, 2)).astype(np.float32)
    c = oracle.epan_contributions(S, h, lo, hi)
    outside = ~np.all((S >= lo) & (S <= hi), axis=1)
    assert np.all(c[outside] < thr * (1 + 1e-12))


# ------------------------------------------------------------------ reading R15 (tail culling bound)
def _outside_sq(S, h, lo, hi):
    """sum_j o_j^2 in y' units: o_j = distance of the point outside [l_j, u_j] / (sqrt2 h_j) * sqrt(log2 e)."""
    S = S.astype(np.float64)
    r = np.maximum(np.maximum(S - hi.astype(np.float64), lo.astype(np.float64) - S), 0.0)
    return ((r / (math.sqrt(2.0) * h)) ** 2).sum(axis=1) * math.log2(math.e)


@pytest.mark.parametrize("d", [1, 3, 6])
def test_r15_cull_bound_against_oracle(d):
    """DESIGN R15: a point with sum_j o_j^2 >= 64 contributes p^(i) <= 2^-sum o_j^2 (1/2 erfc(z) <= 1/2 e^{-z^2})
    and each gradient term |d p^(i)/d h_j| <= 2^-60 / (sqrt(pi) sqrt(log2 e) h_j); checked on the fp64 oracle
    (eq. 13 and eq. 17 as written, not the bound's algebra) for points at all distances from the box."""
    g = np.random.default_rng(1500 + d)
    n = 4000
    S = g.normal(0.0, 1.0, size=(n, d)).astype(np.float32) * np.float32(3.0)
    h = g.uniform(0.05, 0.4, d)
    for k in range(4):
        c = g.normal(0.0, 2.0, d)
        w = g.uniform(0.2, 3.0, d)
        lo, hi = (c - w).astype(np.float32), (c + w).astype(np.float32)
        o2 = _outside_sq(S, h, lo, hi)
        cvals = oracle.contributions(S, h, lo, hi)
        assert np.all(cvals <= np.exp2(-o2) * (1 + 1e-12) + 1e-300)
        far = np.nonzero(o2 >= 64.0)[0]
        assert len(far) > 50                       # the workload does contain culled points
        inside = np.all((S >= lo) & (S <= hi), axis=1)
        assert np.all(o2[inside] == 0.0)           # inside points are never culled
        gconst = 1.0 / (math.sqrt(math.pi) * math.sqrt(math.log2(math.e)) * h)
        for i in far[:60]:
            terms = oracle.grad_abs_scale(S[i:i + 1], h, lo, hi)[0]  # |d p^(i) / d h_j| of this point alone
            assert np.all(terms <= 2.0 ** -60 * gconst * (1 + 1e-9) + 1e-300), (o2[i], terms)


def test_r15_epanechnikov_support_is_exact():
    """Epanechnikov culling (R15): a point outside the support |t - b| >= h beyond the box in any dimension
    has contribution exactly 0 in the oracle (eq. 13 with the R14 kernel)."""
    g = np.random.default_rng(1600)
    S = g.normal(0.0, 1.0, size=(3000, 4)).astype(np.float32)
    h = g.uniform(0.2, 0.6, 4)
    lo, hi = np.full(4, -0.5, np.float32), np.full(4, 0.7, np.float32)
    r = np.maximum(np.maximum(S.astype(np.float64) - hi, lo - S.astype(np.float64)), 0.0) / h
    out = (r >= 1.0).any(axis=1)
    c = oracle.epan_contributions(S, h, lo, hi)
    assert out.sum() > 100 and np.all(c[out] == 0.0) and np.all(c[~out] > 0.0)


# --- reservoir sampling (Algorithm R, O11) ---------------------------------------

def test_reservoir_inclusion_frequencies_chi_square():
    """After n = 10 N arrivals every arrival is in the sample with probability N / n (P:L248:
    each insert enters with probability |S|/|R|): chi-square of the inclusion counts of the
    200 arrival ids over 4000 seeds against the uniform expectation."""
    from scipy.stats import chi2
    Ns, n_total, T = 20, 200, 4000
    counts = np.zeros(n_total + 1)
    for seed in range(T):
        content = oracle.reservoir_run(0x5EED0000 + seed, Ns, n_total)
        assert len(set(content.tolist())) == Ns and content.min() >= 1 and content.max() <= n_total
        counts[content] += 1
    counts = counts[1:]
    expect = T * Ns / n_total
    stat = float(((counts - expect) ** 2 / expect).sum())
    assert chi2.sf(stat, n_total - 1) > 1e-4, stat
    # late and early arrivals alike (no drift with the arrival index)
    assert abs(counts[:100].mean() - counts[100:].mean()) < 0.05 * expect


def test_reservoir_draws_are_uniform_on_0_a():
    """The a-th arrival draws j uniformly from [0, a): chi-square over 50000 draws for a = 7,
    and j / a over a counter sweep is U(0, 1) (KS)."""
    from scipy.stats import chi2, kstest
    a = 7
    js = np.array([oracle.reservoir_draw(s, a) for s in range(50000)])
    assert js.min() == 0 and js.max() == a - 1
    c = np.bincount(js, minlength=a)
    stat = float(((c - 50000 / a) ** 2 / (50000 / a)).sum())
    assert chi2.sf(stat, a - 1) > 1e-4
    arr = np.arange(1000, 21000)
    u = np.array([oracle.reservoir_draw(99, int(x)) for x in arr]) / arr
    assert kstest(u, "uniform").pvalue > 1e-4


def test_reservoir_slots_follow_algorithm_r():
    """The first N arrivals fill slots 0..N-1 in order; afterwards arrival a takes slot j iff its
    draw j < N; applying the per-chunk slot lists in order reproduces the whole-run content."""
    Ns, seed = 64, 1234
    first = oracle.reservoir_slots(seed, Ns, 0, Ns)
    assert np.array_equal(first, np.arange(Ns))
    content = np.arange(1, Ns + 1)
    n_seen = Ns
    for k in (1, 17, 300, 5000):
        sl = oracle.reservoir_slots(seed, Ns, n_seen, k)
        for r, j in enumerate(sl):
            a = n_seen + r + 1
            d = oracle.reservoir_draw(seed, a)
            assert j == (d if d < Ns else -1)
            if j >= 0:
                content[j] = a
        n_seen += k
    assert np.array_equal(content, oracle.reservoir_run(seed, Ns, n_seen))


@pytest.mark.parametrize("d", [2, 5, 8])
def test_r17_cell_skip_implies_r15_bound_for_every_point(d):
    """DESIGN R17: the cells scan skips a (box, cell) pair when, from the cell's bounding box alone,
    sum_j max(|c_cell - c_box| - hw_cell - hw_box, 0)^2 >= 64.5 in y' units (centres and half-widths
    scaled by ap_j = sqrt(log2 e) / (sqrt2 h_j)).  Every point inside the bounding box is then at
    least that far outside the box, so each one obeys the R15 bound on the fp64 oracle: p^(i) <= 2^-64
    and |d p^(i) / d h_j| <= 2^-60 gconst_j.  Cells are Morton-ordered chunks of a clustered sample;
    boxes anywhere, so both skipped and kept cells occur."""
    import synth
    n, C = 1 << 14, 256
    S = synth.make_data("gauss", n, d, seed=1700 + d)
    h = oracle.scott(S) * 0.5
    ap = math.sqrt(math.log2(math.e)) / (math.sqrt(2.0) * h)
    key = np.lexsort(tuple(np.floor((S[:, j] - S[:, j].min()) / (np.ptp(S[:, j]) + 1e-30) * 15.999).astype(int)
                           for j in range(d)))
    X = S[key].reshape(n // C, C, d).astype(np.float64)
    mn, mx = X.min(1), X.max(1)
    lo, hi = synth.random_boxes(S, 12, seed=1701 + d)
    gconst = 1.0 / (math.sqrt(math.pi) * math.sqrt(math.log2(math.e)) * h)
    skipped = 0
    for b in range(len(lo)):
        cb, hwb = 0.5 * (lo[b].astype(np.float64) + hi[b]) * ap, 0.5 * (hi[b].astype(np.float64) - lo[b]) * ap
        cc, chw = 0.5 * (mn + mx) * ap, 0.5 * (mx - mn) * ap
        o = np.maximum(np.abs(cc - cb) - chw - hwb, 0.0)
        skip = (o ** 2).sum(axis=1) >= 64.5
        for c in np.nonzero(skip)[0][:6]:
            skipped += 1
            pts = X[c].astype(np.float32)
            assert np.all(_outside_sq(pts, h, lo[b], hi[b]) >= 64.0)
            cv = oracle.contributions(pts, h, lo[b], hi[b])
            assert np.all(cv <= 2.0 ** -64 * (1 + 1e-12))
            for i in range(8):  # |d p^(i) / d h_j| of single points (grad_abs_scale of a one-point sample)
                t = oracle.grad_abs_scale(pts[i:i + 1], h, lo[b], hi[b])[0]
                assert np.all(t <= 2.0 ** -60 * gconst * (1 + 1e-9) + 1e-300)
    assert skipped >= 6
