# variant definitions for make_variants.py (each edits a copy of csrc/)
@variant("nohs")
def _nohs(d):
    edit(f"{d}/phi.cuh", "return fmaf(q.y, copysignf(E.y, y.y), fmaf(-q.x, copysignf(E.x, y.x), hs));",
         "return fmaf(q.y, E.y, -q.x * E.x);")

@variant("noclamp")
def _noclamp(d):
    edit(f"{d}/phi.cuh", "make_float2(fminf(fabsf(y.x), kYc), fminf(fabsf(y.y), kYc))",
         "make_float2(fabsf(y.x), fabsf(y.y))")

@variant("k5")
def _k5(d):
    edit(f"{d}/phi.cuh", "for (int k = KDE_PHI_DEG - 1; k >= 0; --k)", "for (int k = KDE_PHI_DEG - 2; k >= 0; --k)")

@variant("k4")
def _k4(d):
    edit(f"{d}/phi.cuh", "for (int k = KDE_PHI_DEG - 1; k >= 0; --k)", "for (int k = KDE_PHI_DEG - 3; k >= 0; --k)")

@variant("sgnA")
def _sgnA(d):
    edit(f"{d}/phi.cuh", "return fmaf(q.y, copysignf(E.y, y.y), fmaf(-q.x, copysignf(E.x, y.x), hs));",
         "(void)hs; const float2 A = __ffma2_rn(q, make_float2(-E.x, -E.y), f2(0.5f));\n"
         "  return copysignf(A.x, y.x) - copysignf(A.y, y.y);")

def _flags(**kw):
    def f(d):
        # prepend tuning macros to scan.cuh
        p = f"{d}/scan.cuh"
        s = open(p).read()
        open(p, "w").write("".join(f"#define KDE_TUNE_{k} {v}\n" for k, v in kw.items()) + s)
    return f

for _name, _kw in {
    "minb3": dict(MINB=3), "minb5": dict(MINB=5), "pu2": dict(PU=2), "minb5pu2": dict(MINB=5, PU=2),
    "s512x3o4": dict(SINGLE_TILE=512, SINGLE_STAGES=3, SINGLE_OCC=4),
    "s1024x3o3": dict(SINGLE_TILE=1024, SINGLE_STAGES=3, SINGLE_OCC=3),
    "s1024x2o3": dict(SINGLE_TILE=1024, SINGLE_STAGES=2, SINGLE_OCC=3),
    "s2048x2o2": dict(SINGLE_TILE=2048, SINGLE_STAGES=2, SINGLE_OCC=2),
    "s512x4o3": dict(SINGLE_TILE=512, SINGLE_STAGES=4, SINGLE_OCC=3),
}.items():
    VARIANTS[_name] = _flags(**_kw)

for _name, _kw in {
    "reg2": dict(SINGLE_TMA_MAXD=0, SINGLE_VW=2), "reg4": dict(SINGLE_TMA_MAXD=0, SINGLE_VW=4),
    "reg2pf": dict(SINGLE_TMA_MAXD=0, SINGLE_VW=2, SINGLE_PF=1), "reg4pf": dict(SINGLE_TMA_MAXD=0, SINGLE_VW=4, SINGLE_PF=1),
    "s2048x2o3": dict(SINGLE_TILE=2048, SINGLE_STAGES=2, SINGLE_OCC=3),
    "s4096x2o1": dict(SINGLE_TILE=4096, SINGLE_STAGES=2, SINGLE_OCC=1),
    "s2048x3o2": dict(SINGLE_TILE=2048, SINGLE_STAGES=3, SINGLE_OCC=2),
}.items():
    VARIANTS[_name] = _flags(**_kw)

@variant("nomem")
def _nomem(d):
    p = f"{d}/scan_single_tma.cuh"
    edit(p, "mbar_wait_parity(&full[st], (uint32_t)((k / STAGES) & 1));", "if (k < STAGES) mbar_wait_parity(&full[st], 0u);")
    edit(p, "if (tid == 0 && k + STAGES < ntiles) {", "if (false) {")

@variant("nobar")
def _nobar(d):
    # compute-only AND no per-tile CTA barrier (timing only)
    p = f"{d}/scan_single_tma.cuh"
    edit(p, "mbar_wait_parity(&full[st], (uint32_t)((k / STAGES) & 1));", "if (k < STAGES) mbar_wait_parity(&full[st], 0u);")
    edit(p, "if (tid == 0 && k + STAGES < ntiles) {", "if (false) {")
    edit(p, "    __syncthreads();  // every thread is done with stage st\n", "")

for _name, _kw in {
    "s1024x2o4": dict(SINGLE_TILE=1024, SINGLE_STAGES=2, SINGLE_OCC=4),
    "s2048x2o4": dict(SINGLE_TILE=2048, SINGLE_STAGES=2, SINGLE_OCC=4),
    "s1024x3o4": dict(SINGLE_TILE=1024, SINGLE_STAGES=3, SINGLE_OCC=4),
}.items():
    VARIANTS[_name] = _flags(**_kw)

@variant("nobar_o4")
def _nobar_o4(d):
    _flags(SINGLE_TILE=1024, SINGLE_STAGES=2, SINGLE_OCC=4)(d)
    _nobar(d)

for _name, _kw in {
    "w1024x4o2": dict(SINGLE_TILE=1024, SINGLE_STAGES=4, SINGLE_OCC=2),
    "w2048x2o2": dict(SINGLE_TILE=2048, SINGLE_STAGES=2, SINGLE_OCC=2),
    "w2048x3o1": dict(SINGLE_TILE=2048, SINGLE_STAGES=3, SINGLE_OCC=1),
    "w512x4o3": dict(SINGLE_TILE=512, SINGLE_STAGES=4, SINGLE_OCC=3),
    "w512x6o2": dict(SINGLE_TILE=512, SINGLE_STAGES=6, SINGLE_OCC=2),
    "w1024x3o3": dict(SINGLE_TILE=1024, SINGLE_STAGES=3, SINGLE_OCC=3),
}.items():
    VARIANTS[_name] = _flags(**_kw)
