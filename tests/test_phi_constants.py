"""CPU pin of the CUDA-side erfc constants (csrc/phi_coeffs.h, written by
tools/fit_phi.py): the kernel's exact fp32 operation sequence -- t from the
pair reciprocal r = 1/(den_u den_l), Horner for Q(t), times e^{-x^2} -- is
replayed in numpy float32 and compared with scipy's erfc.  This checks the
committed constants against the mathematics (not against the oracle, which
uses libm erf and shares nothing with csrc/): relative error <= 8e-7 on
[0, 4.5] and absolute error <= 1e-12 beyond, the accuracy DESIGN.md §8 budgets
against the 1e-7 + 1e-5 selectivity tolerance."""
import os
import re

import numpy as np
from scipy.special import erfc

HDR = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                   "paper_conf_sigmod_heimelkm15_b200", "csrc", "phi_coeffs.h")


def _constants():
    s = open(HDR).read()
    deg = int(re.search(r"#define KDE_PHI_DEG (\d+)", s).group(1))
    p = float(re.search(r"#define KDE_PHI_P ([0-9.eE+-]+)f", s).group(1))
    coef = [float(c) for c in re.findall(r"k == \d+ \? ([0-9.eE+-]+)f", s)]
    assert len(coef) == deg + 1
    return np.float32(p), np.array(coef, np.float32)


def _kernel_erfc(xu, xl):
    f32 = np.float32
    p, c = _constants()
    du = (p * xu + f32(1)).astype(f32)
    dl = (p * xl + f32(1)).astype(f32)
    r = (f32(1) / (du * dl).astype(f32)).astype(f32)
    out = []
    for x, t in ((xu, (dl * r).astype(f32)), (xl, (du * r).astype(f32))):
        q = np.full_like(t, c[-1])
        for k in range(len(c) - 2, -1, -1):
            q = (q * t + c[k]).astype(f32)
        e = np.exp(-(x.astype(np.float64) ** 2)).astype(f32)
        out.append((e * q).astype(np.float64))
    return out


def test_erfc_constants_accuracy():
    rng = np.random.default_rng(0)
    xu = np.concatenate([np.linspace(0, 12, 200001), rng.uniform(0, 12, 200001)]).astype(np.float32)
    xl = np.concatenate([rng.uniform(0, 12, 200001), np.linspace(0, 12, 200001)]).astype(np.float32)
    for x, g in zip((xu, xl), _kernel_erfc(xu, xl)):
        ref = erfc(x.astype(np.float64))
        inside = x <= 4.5
        assert np.max(np.abs(g[inside] - ref[inside]) / ref[inside]) <= 8e-7
        assert np.max(np.abs(g[~inside] - ref[~inside])) <= 1e-12
        assert np.all(np.isfinite(g))


def test_erfc_constants_special_values():
    # erfc(0) = 1 to fp32 accuracy; the polynomial stays finite and bounded as t -> 0 (|x| -> inf)
    g0, _ = _kernel_erfc(np.zeros(1, np.float32), np.zeros(1, np.float32))
    assert abs(g0[0] - 1.0) <= 8e-7
    _, c = _constants()
    t = np.linspace(0, 1, 1001)
    q = np.polyval(c[::-1].astype(np.float64), t)
    assert np.all(np.isfinite(q)) and np.max(np.abs(q)) < 10
