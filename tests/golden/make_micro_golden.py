"""Writes tests/golden/micro_example.json: a worked example for the KDE box
estimator computed INDEPENDENTLY of oracle/ and of the CUDA path.

The paper prints no numeric worked example, so this fixture is computed from
the paper's *integral* definitions with 50-digit mpmath quadrature, never with
the closed forms the oracle implements:
  * p^(i)   = integral over the box of the kernel density, eq. (10)-(12)
              (P:L461-476); the product kernel lets the d-dim integral factor
              into 1-D integrals, each evaluated by mpmath.quad of the
              normal density N_{t,h^2}.
  * p_hat   = (1/s) sum_i p^(i), eq. (2).
  * dp/dh   = numerical derivative (mpmath.diff) of the quadrature estimate,
              the quantity eq. (15) differentiates.
  * L2 loss = (p_hat - p)^2 and its h-gradient via eq. (14).
  * eq. (6) leave-one-out estimates by re-averaging the sample without point i.
  * eq. (19) p_max = quadrature mass of the box-centre point.
  * eq. (20) threshold = largest quadrature mass of the points t_(j) moved to
              the lower face of dimension j, the bound derived at P:L576.
  * Scott's h, eq. (3), population sigma, in mpmath.
Run:  python tests/golden/make_micro_golden.py
"""
import json
import os

import mpmath as mp

mp.mp.dps = 50

S = [(0.0, 0.0), (1.0, 2.0), (-1.0, 0.5)]
H = (0.5, 1.0)
LO = (-0.5, 0.0)
HI = (1.0, 1.5)
P_TRUE = 0.4


def dens(x, mu, h):
    return mp.exp(-((x - mu) ** 2) / (2 * h * h)) / (mp.sqrt(2 * mp.pi) * h)


def mass1(t, h, l, u):
    return mp.quad(lambda x: dens(x, t, h), [l, t, u] if l < t < u else [l, u])


def point_mass(t, h, lo, hi):
    m = mp.mpf(1)
    for j in range(len(t)):
        m *= mass1(mp.mpf(t[j]), h[j], mp.mpf(lo[j]), mp.mpf(hi[j]))
    return m


def estimate(h, sample=S, lo=LO, hi=HI):
    return sum(point_mass(t, h, lo, hi) for t in sample) / len(sample)


def main():
    h = [mp.mpf(x) for x in H]
    c = [point_mass(t, h, LO, HI) for t in S]
    est = sum(c) / len(c)
    grad = []
    for j in range(2):
        def f(x, j=j):
            hh = list(h)
            hh[j] = x
            return estimate(hh)
        grad.append(mp.diff(f, h[j]))
    L2 = (est - P_TRUE) ** 2
    dL2 = [2 * (est - P_TRUE) * g for g in grad]
    loo = []
    for i in range(len(S)):
        rest = [t for k, t in enumerate(S) if k != i]
        loo.append(estimate(h, rest))
    # L1 karma, eq. (7) with C.1 argument order: |loo - p| - |est - p|
    dK_L1 = [abs(x - P_TRUE) - abs(est - P_TRUE) for x in loo]
    centre = [(LO[j] + HI[j]) / 2 for j in range(2)]
    pmax = point_mass(centre, h, LO, HI)
    bound = []
    for j in range(2):
        t = list(centre)
        t[j] = LO[j]
        bound.append(point_mass(t, h, LO, HI))
    thr = max(bound)
    n = len(S)
    scott = []
    for j in range(2):
        col = [mp.mpf(t[j]) for t in S]
        mean = sum(col) / n
        var = sum((x - mean) ** 2 for x in col) / n
        scott.append(mp.power(n, mp.mpf(-1) / (2 + 4)) * mp.sqrt(var))
    s = lambda x: mp.nstr(x, 25)
    out = {
        "citation": "No worked example is printed in PAPER.md. Values computed by "
                    "tests/golden/make_micro_golden.py from the integral definitions eq. (2), (10)-(12), "
                    "(15), (6), (19)-(20), (3) with 50-digit mpmath quadrature (independent of oracle/).",
        "sample": S, "h": H, "lo": LO, "hi": HI, "true_sel": P_TRUE,
        "contributions": [s(x) for x in c],
        "estimate": s(est),
        "dpdh": [s(x) for x in grad],
        "dpdlnh": [s(grad[j] * h[j]) for j in range(2)],
        "l2_loss": s(L2),
        "l2_grad": [s(x) for x in dL2],
        "leave_one_out": [s(x) for x in loo],
        "karma_delta_l1": [s(x) for x in dK_L1],
        "p_max": s(pmax),
        "thr20": s(thr),
        "scott_h": [s(x) for x in scott],
    }
    path = os.path.join(os.path.dirname(os.path.abspath(__file__)), "micro_example.json")
    with open(path, "w") as f:
        json.dump(out, f, indent=1)
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main()
