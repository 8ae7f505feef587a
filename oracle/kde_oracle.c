/*
 * kde_oracle.c -- plain, slow, obviously-correct fp64 CPU oracle for the
 * KDE range-selectivity hot path of Heimel, Kiefer, Markl (SIGMOD 2015).
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and the
 * cpu_baseline / --impl reference legs of bench.py may load or call this
 * library.  The product path (paper_conf_sigmod_heimelkm15_b200/) never
 * links, imports or executes it, and it shares no code, header, table or
 * constant with the CUDA path.
 *
 * Citation convention: "P:L<n>" = line n of PAPER.md (the paper text).
 * Every function below writes out the paper's definition directly, in the
 * paper's order and notation, with libm's erf/exp/log as the only library
 * primitives.  No blocking, fusion or reordering: sums run in index order.
 *
 * Inputs are the SAME fp32 arrays the product receives (sample row-major
 * n x d, bounds lo/hi q x d), widened exactly to double; bandwidth h is
 * double.  +-inf bounds are allowed (half-open boxes); erf(+-inf) = +-1.
 *
 * Readings of the paper (listed in DESIGN.md "Readings"):
 *   R1 sigma in Scott's rule is the population std (1/n)
 *   R2 C.1 argument order L(estimate, truth) is used everywhere
 *   R3 x*exp(-x^2/2h^2) := 0 when x is infinite (limit value)       eq. 17
 *   R4 karma threshold compare is strict (<), after the update
 *   R5 eq. 20 is applied only when the true selectivity == 0 and
 *      every box width is > 0 (a zero width makes eq. 19 vanish)
 *   R7 squared-relative loss: the printed derivative lacks the
 *      square of (lambda + p); the true derivative of the printed loss
 *      is used (pinned by finite differences)
 *   R6 Listing 1 (adaptive bandwidth) is missing from the text; the
 *      update is reconstructed from the prose P:L179-183, L561.  The
 *      prose-fixed parts are pinned by hand traces; lr0 and the exact
 *      step form stay PARITY UNPINNED (no listing, no trace).
 *   R16 erf differences of eq. (13) with both arguments on one side of 0
 *      are evaluated as the equal erfc difference (fp64 erf saturates)
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define OR_SQRT2 1.41421356237309504880
#define OR_SQRTPI 1.77245385090551602730

/* ---------------------------------------------------------------------
 * eq. (13): the i-th point's probability mass in the box
 *   p^(i) = 1/2^d * prod_j [ erf((u_j - t_j)/(sqrt2 h_j)) - erf((l_j - t_j)/(sqrt2 h_j)) ]
 * ------------------------------------------------------------------- */
/* erf(b) - erf(a) for a <= b.  When both arguments have the same sign the
 * difference is taken through the exact identity erf(b) - erf(a) = erfc(a) -
 * erfc(b) (or erfc(-b) - erfc(-a)): fp64 erf saturates to +-1 beyond |z| ~ 5.9,
 * so the plain difference would return 0 for a box in the far tail of a point
 * (reading R16).  Same definition, no approximation. */
static double erf_diff(double a, double b)
{
    if (a >= 0.0) return erfc(a) - erfc(b);
    if (b <= 0.0) return erfc(-b) - erfc(-a);
    return erf(b) - erf(a);
}

double oracle_point_mass(const float *t, int32_t d, const double *h,
                         const float *lo, const float *hi)
{
    double prod = 1.0;
    for (int32_t j = 0; j < d; ++j) {
        double u = (double)hi[j], l = (double)lo[j], tj = (double)t[j];
        double diff = erf_diff((l - tj) / (OR_SQRT2 * h[j]), (u - tj) / (OR_SQRT2 * h[j]));
        prod *= diff;
    }
    return prod / pow(2.0, (double)d);
}

/* eq. (13) for every sample point of one query (the retained buffer).
 * Each value depends only on its own point, so the loop over points runs on
 * all host cores without changing any result. */
void oracle_contributions(const float *sample, int64_t n, int32_t d, const double *h,
                          const float *lo, const float *hi, double *c_out)
{
    #pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < n; ++i)
        c_out[i] = oracle_point_mass(sample + i * d, d, h, lo, hi);
}

/* ---------------------------------------------------------------------
 * Sums over the sample in index order, Neumaier-compensated (SURVEY.md
 * §8(c) O3): the result is the fp64 rounding of the exact sum of the fp64
 * terms up to ~2 ulp, independent of n.
 * ------------------------------------------------------------------- */
typedef struct { double s, c; } nsum_t;

static void nsum_add(nsum_t *a, double x)
{
    double t = a->s + x;
    a->c += fabs(a->s) >= fabs(x) ? (a->s - t) + x : (x - t) + a->s;
    a->s = t;
}

static double nsum_get(const nsum_t *a) { return a->s + a->c; }

/* x * exp(-x^2 / (2 h^2)) with the limit value 0 for infinite x (R3). */
static double xexp(double x, double h)
{
    if (isinf(x)) return 0.0;
    return x * exp(-(x * x) / (2.0 * h * h));
}

/* Per-point terms of one query, written literally:
 *   term[0]     = p^(i)                                            eq. (13)
 *   term[1 + i] = [ (l_i - t_i) e^{-(l_i-t_i)^2/2h_i^2} - (u_i - t_i) e^{-(u_i-t_i)^2/2h_i^2} ]
 *                 * prod_{k != i} [ erf((u_k - t_k)/(sqrt2 h_k)) - erf((l_k - t_k)/(sqrt2 h_k)) ]
 *                                                                  eq. (17), P:L545-547 (summand)
 * mode 1: the summand of eq. (17) in absolute value, |bracket| * |prod|
 * (the tolerance scale m_ij = sum_j |d p^(i)/d h_i| of SURVEY.md §8(c)).
 * The erf difference of dimension k is evaluated once per point and reused by
 * the products over k != i (the same libm values the formula names; the
 * product over k != i is still taken directly, O(d^2)). */
static void point_terms(const float *t, int32_t d, const double *h, const float *l, const float *u,
                        int mode, double *term)
{
    double diff[64];
    for (int32_t k = 0; k < d; ++k)
        diff[k] = erf_diff(((double)l[k] - (double)t[k]) / (OR_SQRT2 * h[k]),
                           ((double)u[k] - (double)t[k]) / (OR_SQRT2 * h[k]));
    double prod0 = 1.0;                                  /* eq. (13): the same factors, in order */
    for (int32_t k = 0; k < d; ++k) prod0 *= diff[k];
    term[0] = prod0 / pow(2.0, (double)d);
    for (int32_t i = 0; i < d; ++i) {
        double li = (double)l[i] - (double)t[i];
        double ui = (double)u[i] - (double)t[i];
        double bracket = xexp(li, h[i]) - xexp(ui, h[i]);
        double prod = 1.0;
        for (int32_t k = 0; k < d; ++k) {
            if (k == i) continue;
            prod *= diff[k];
        }
        term[1 + i] = mode == 1 ? fabs(bracket) * fabs(prod) : bracket * prod;
    }
}

/* Driver shared by eq. (2) and eq. (17): sums[qq][0..d] = Neumaier-compensated sums of the
 * per-point terms.  Many small queries run one query per thread, each summed in index order.  A
 * large sample is cut into fixed 8192-point chunks ("OpenMP over (query, fixed
 * sample chunk), partials combined in chunk order"): every chunk is summed in index order, the
 * chunk partials are then added in chunk order -- the result does not depend on the thread count. */
#define OR_CHUNK 8192
static void scan_queries(const float *sample, int64_t n, int32_t d, const double *h,
                         const float *lo, const float *hi, int64_t q, int mode, double *sums)
{
    const int32_t na = 1 + d;
    if (n < 4 * OR_CHUNK) {
        #pragma omp parallel for schedule(dynamic, 1)
        for (int64_t qq = 0; qq < q; ++qq) {
            nsum_t acc[65];
            double term[65];
            for (int32_t k = 0; k < na; ++k) acc[k].s = acc[k].c = 0.0;
            for (int64_t i = 0; i < n; ++i) {
                point_terms(sample + i * d, d, h, lo + qq * d, hi + qq * d, mode, term);
                for (int32_t k = 0; k < na; ++k) nsum_add(&acc[k], term[k]);
            }
            for (int32_t k = 0; k < na; ++k) sums[qq * na + k] = nsum_get(&acc[k]);
        }
        return;
    }
    const int64_t nch = (n + OR_CHUNK - 1) / OR_CHUNK;
    const int64_t QB = 64;  /* queries per block of (query, chunk) work items */
    nsum_t *part = (nsum_t *)malloc(sizeof(nsum_t) * (size_t)QB * (size_t)nch * (size_t)na);
    for (int64_t q0 = 0; q0 < q; q0 += QB) {
        const int64_t qn = q - q0 < QB ? q - q0 : QB;
        #pragma omp parallel for collapse(2) schedule(dynamic, 1)
        for (int64_t qq = 0; qq < qn; ++qq)
            for (int64_t c = 0; c < nch; ++c) {
                nsum_t acc[65];
                double term[65];
                for (int32_t k = 0; k < na; ++k) acc[k].s = acc[k].c = 0.0;
                const int64_t i1 = (c + 1) * OR_CHUNK < n ? (c + 1) * OR_CHUNK : n;
                for (int64_t i = c * OR_CHUNK; i < i1; ++i) {
                    point_terms(sample + i * d, d, h, lo + (q0 + qq) * d, hi + (q0 + qq) * d, mode, term);
                    for (int32_t k = 0; k < na; ++k) nsum_add(&acc[k], term[k]);
                }
                for (int32_t k = 0; k < na; ++k) part[(qq * nch + c) * na + k] = acc[k];
            }
        for (int64_t qq = 0; qq < qn; ++qq) {
            nsum_t tot[65];
            for (int32_t k = 0; k < na; ++k) tot[k].s = tot[k].c = 0.0;
            for (int64_t c = 0; c < nch; ++c)
                for (int32_t k = 0; k < na; ++k) {
                    nsum_add(&tot[k], part[(qq * nch + c) * na + k].s);
                    nsum_add(&tot[k], part[(qq * nch + c) * na + k].c);
                }
            for (int32_t k = 0; k < na; ++k) sums[(q0 + qq) * na + k] = nsum_get(&tot[k]);
        }
    }
    free(part);
}

/* ---------------------------------------------------------------------
 * eq. (2): p_H(Omega) = (1/s) sum_i p^(i)(Omega), index order.
 * ------------------------------------------------------------------- */
void oracle_estimate(const float *sample, int64_t n, int32_t d, const double *h,
                     const float *lo, const float *hi, int64_t q, double *est)
{
    double *sums = (double *)malloc(sizeof(double) * (size_t)q * (size_t)(1 + d));
    scan_queries(sample, n, d, h, lo, hi, q, 0, sums);
    for (int64_t k = 0; k < q; ++k) est[k] = sums[k * (1 + d)] / (double)n;
    free(sums);
}

/* ---------------------------------------------------------------------
 * eq. (17), written literally:
 *   dp/dh_i = sqrt2 / (sqrtpi h_i^2 2^d s) * sum_j [ (l_i - t_i) e^{-(l_i-t_i)^2/2h_i^2}
 *                                                - (u_i - t_i) e^{-(u_i-t_i)^2/2h_i^2} ]
 *             * prod_{k != i} [ erf((u_k - t_k)/(sqrt2 h_k)) - erf((l_k - t_k)/(sqrt2 h_k)) ]
 * Also returns the estimate (eq. 2) of the same query.
 * ------------------------------------------------------------------- */
void oracle_estimate_grad(const float *sample, int64_t n, int32_t d, const double *h,
                          const float *lo, const float *hi, int64_t q,
                          double *est, double *dpdh)
{
    double *sums = (double *)malloc(sizeof(double) * (size_t)q * (size_t)(1 + d));
    scan_queries(sample, n, d, h, lo, hi, q, 0, sums);
    for (int64_t qq = 0; qq < q; ++qq) {
        est[qq] = sums[qq * (1 + d)] / (double)n;
        for (int32_t i = 0; i < d; ++i)
            dpdh[qq * d + i] = OR_SQRT2 / (OR_SQRTPI * h[i] * h[i] * pow(2.0, (double)d) * (double)n)
                               * sums[qq * (1 + d) + 1 + i];
    }
    free(sums);
}

/* Gradient magnitude scale used by the parity tolerance (test infrastructure,
 * not a paper quantity), SURVEY.md §8(c) "Parity criteria":
 *   m_ij = (1/s) sum_j |d p^(i)/d h_i|
 *        = sqrt2 / (sqrtpi h_i^2 2^d s) * sum_j |bracket_ij| * |prod_{k != i} [...]|
 * i.e. eq. (17) with every per-point summand in absolute value. */
void oracle_grad_abs_scale(const float *sample, int64_t n, int32_t d, const double *h,
                           const float *lo, const float *hi, int64_t q, double *mabs)
{
    double *sums = (double *)malloc(sizeof(double) * (size_t)q * (size_t)(1 + d));
    scan_queries(sample, n, d, h, lo, hi, q, 1, sums);
    for (int64_t qq = 0; qq < q; ++qq)
        for (int32_t i = 0; i < d; ++i)
            mabs[qq * d + i] = OR_SQRT2 / (OR_SQRTPI * h[i] * h[i] * pow(2.0, (double)d) * (double)n)
                               * sums[qq * (1 + d) + 1 + i];
    free(sums);
}

/* ---------------------------------------------------------------------
 * Appendix C.1: loss L(p_hat, p) and dL/dp_hat.
 * kind: 0 quadratic, 1 absolute, 2 relative, 3 squared relative, 4 squared Q.
 * lambda: the smoothing constant of footnote 6.  log = natural log.
 * ------------------------------------------------------------------- */
static double sgn3(double a, double b) { return a < b ? -1.0 : (a > b ? 1.0 : 0.0); }

void oracle_loss(int32_t kind, double lambda, double phat, double p,
                 double *L, double *dL)
{
    switch (kind) {
    case 0: *L = (phat - p) * (phat - p);              *dL = 2.0 * (phat - p); break;
    case 1: *L = fabs(phat - p);                       *dL = sgn3(phat, p); break;
    case 2: *L = fabs(phat - p) / (lambda + p);        *dL = sgn3(phat, p) / (lambda + p); break;
    case 3: *L = ((phat - p) / (lambda + p)) * ((phat - p) / (lambda + p));
            /* R7: P:L520 prints 2(p_hat-p)/(lambda+p), which is not the derivative of the
             * loss printed on the same line; the derivative of that loss is used. */
            *dL = 2.0 * (phat - p) / ((lambda + p) * (lambda + p)); break;
    default: {
            double r = log(lambda + phat) - log(lambda + p);
            *L = r * r;
            *dL = 2.0 * r / (lambda + phat);
        }
    }
}

/* ---------------------------------------------------------------------
 * eq. (5): loss = (1/q) sum_k L(p_hat(Omega_k), p_k)
 * eq. (14): dL/dh_i = dL/dp_hat * dp_hat/dh_i, averaged over q
 * eq. (18): log mode multiplies dimension i by h_i
 * est_out (optional) receives the q estimates.
 * ------------------------------------------------------------------- */
void oracle_loss_and_grad(const float *sample, int64_t n, int32_t d, const double *h,
                          const float *lo, const float *hi, const double *true_sel,
                          int64_t q, int32_t kind, double lambda, int32_t log_bw,
                          double *loss_out, double *grad_out, double *est_out)
{
    double *est = (double *)malloc(sizeof(double) * (size_t)q);
    double *dpdh = (double *)malloc(sizeof(double) * (size_t)(q * d));
    oracle_estimate_grad(sample, n, d, h, lo, hi, q, est, dpdh);
    double loss = 0.0;
    for (int32_t i = 0; i < d; ++i) grad_out[i] = 0.0;
    for (int64_t k = 0; k < q; ++k) {
        double L, dL;
        oracle_loss(kind, lambda, est[k], true_sel[k], &L, &dL);
        loss += L;
        for (int32_t i = 0; i < d; ++i) grad_out[i] += dL * dpdh[k * d + i];
    }
    *loss_out = loss / (double)q;
    for (int32_t i = 0; i < d; ++i) {
        grad_out[i] /= (double)q;
        if (log_bw) grad_out[i] *= h[i];
    }
    if (est_out) memcpy(est_out, est, sizeof(double) * (size_t)q);
    free(est);
    free(dpdh);
}

/* ---------------------------------------------------------------------
 * eq. (3): h_i = s^(-1/(d+4)) * sigma_i, sigma = population std
 * of column i (R1).  Two passes: mean, then mean squared deviation.
 * ------------------------------------------------------------------- */
void oracle_scott(const float *sample, int64_t n, int32_t d, double *h)
{
    for (int32_t j = 0; j < d; ++j) {
        double mean = 0.0;
        for (int64_t i = 0; i < n; ++i) mean += (double)sample[i * d + j];
        mean /= (double)n;
        double var = 0.0;
        for (int64_t i = 0; i < n; ++i) {
            double dev = (double)sample[i * d + j] - mean;
            var += dev * dev;
        }
        var /= (double)n;
        h[j] = pow((double)n, -1.0 / ((double)d + 4.0)) * sqrt(var);
    }
}

/* ---------------------------------------------------------------------
 * eq. (19): p_max = prod_j erf((u_j - l_j) / (2 sqrt2 h_j))
 * eq. (20): thr  = p_max/2 * max_j erf(w_j/(sqrt2 h_j)) / erf(w_j/(2 sqrt2 h_j))
 * Returns thr; returns +inf (shortcut disabled, R5) when some width is 0.
 * An infinite width gives the ratio erf(inf)/erf(inf) = 1.
 * ------------------------------------------------------------------- */
double oracle_empty_region_threshold(int32_t d, const double *h, const float *lo, const float *hi,
                                     double *pmax_out)
{
    double pmax = 1.0, best = 0.0;
    int disabled = 0;
    for (int32_t j = 0; j < d; ++j) {
        double w = (double)hi[j] - (double)lo[j];
        if (!(w > 0.0)) { disabled = 1; continue; }
        double half = erf(w / (2.0 * OR_SQRT2 * h[j]));
        double full = erf(w / (OR_SQRT2 * h[j]));
        pmax *= half;
        double ratio = isinf(w) ? 1.0 : full / half;
        if (ratio > best) best = ratio;
    }
    if (pmax_out) *pmax_out = disabled ? 0.0 : pmax;
    if (disabled) return INFINITY;
    return pmax / 2.0 * best;
}

/* ---------------------------------------------------------------------
 * Karma pass for one query with true selectivity p, P:L193-204, L250:
 *   eq. (6)  p^-(i) = (p_hat * s - p^(i)) / (s - 1)
 *   eq. (7)  K^(i)  = L(p^-(i), p) - L(p_hat, p)      (argument order R2)
 *   eq. (8)  K_i   <- min(K_i + K^(i), K_max)
 *   flag_i   = K_i < tau  (R4)   or   (p == 0 and p^(i) >= thr_20)  (R5)
 * c[i] are the per-point contributions p^(i) and p_hat their mean, both as
 * computed by the caller (oracle_contributions / oracle_estimate).
 * Writes flagged indices ascending into idx_out (up to cap) and returns the
 * total number of flagged points.
 * ------------------------------------------------------------------- */
int64_t oracle_karma_update(const double *c, int64_t n, double phat, double p,
                            int32_t kind, double lambda, double k_max, double tau,
                            double thr20, double *karma, int64_t *idx_out, int64_t cap)
{
    double L_full, dummy;
    oracle_loss(kind, lambda, phat, p, &L_full, &dummy);
    int64_t nflag = 0;
    for (int64_t i = 0; i < n; ++i) {
        double p_minus = (phat * (double)n - c[i]) / ((double)n - 1.0);
        double L_minus;
        oracle_loss(kind, lambda, p_minus, p, &L_minus, &dummy);
        double dK = L_minus - L_full;
        double k = karma[i] + dK;
        karma[i] = k < k_max ? k : k_max;
        int flag = karma[i] < tau;
        if (p == 0.0 && c[i] >= thr20) flag = 1;
        if (flag) {
            if (nflag < cap) idx_out[nflag] = i;
            ++nflag;
        }
    }
    return nflag;
}

/* ---------------------------------------------------------------------
 * Adaptive bandwidth update (Section 4.1, Listing 1 reconstructed from the
 * prose P:L179-183 and P:L561; see R6 -- PARITY UNPINNED by the paper).
 * State per dimension: acc (mini-batch gradient sum), ms (running mean
 * square of gradients, "average magnitude of recent gradients"), lr
 * (per-dimension learning rate), gprev (previous averaged gradient).
 * oracle_online_accumulate adds one query's gradient (line 9).
 * oracle_online_apply runs lines 12-17 once the mini-batch is full.
 * ------------------------------------------------------------------- */
void oracle_online_accumulate(int32_t d, const double *grad, double *acc)
{
    for (int32_t j = 0; j < d; ++j) acc[j] += grad[j];
}

void oracle_online_apply(int32_t d, int32_t batch, double alpha, double lr_min, double lr_max,
                         double lr_inc, double lr_dec, int32_t log_bw,
                         double *h, double *acc, double *ms, double *lr, double *gprev)
{
    for (int32_t j = 0; j < d; ++j) {
        double g = acc[j] / (double)batch;                        /* line 12: average   */
        ms[j] = alpha * ms[j] + (1.0 - alpha) * g * g;            /* line 14: magnitude */
        if (g * gprev[j] > 0.0) {                                 /* lines 15-16: rate  */
            lr[j] = lr[j] * lr_inc;
            if (lr[j] > lr_max) lr[j] = lr_max;
        } else if (g * gprev[j] < 0.0) {
            lr[j] = lr[j] * lr_dec;
            if (lr[j] < lr_min) lr[j] = lr_min;
        }
        double step = ms[j] > 0.0 ? lr[j] * g / sqrt(ms[j]) : 0.0; /* line 17: step     */
        if (log_bw) {
            h[j] = exp(log(h[j]) - step);                         /* eq. 18     */
        } else {
            if (step > h[j] / 2.0) step = h[j] / 2.0;             /* positivity */
            h[j] = h[j] - step;
        }
        gprev[j] = g;
        acc[j] = 0.0;
    }
}

/* =====================================================================
 * Epanechnikov product kernel.  The paper names it as the
 * cheaper alternative ("a truncated second-degree
 * polynomial") but derives nothing for it.  Reading R14: the
 * 1-D kernel with bandwidth h is the density
 *     K_h(x) = 3 / (4 h) * (1 - (x/h)^2)   for |x| <= h,  0 otherwise,
 * i.e. h is the support half-width, and the d-dim kernel is the product over
 * dimensions (the product-kernel argument of P:L472).  Everything below is
 * the plain integral / derivative of that density: the 1-D box mass is
 * F((u-t)/h) - F((l-t)/h) with the CDF F(v) = (2 + 3v - v^3) / 4 on
 * [-1, 1] (0 below, 1 above), and d/dh of it is
 *     F'(v_u) (-v_u / h) - F'(v_l) (-v_l / h),   F'(v) = 3/4 (1 - v^2) on |v| < 1.
 * ===================================================================== */
static double epan_cdf(double v)
{
    if (v <= -1.0) return 0.0;
    if (v >= 1.0) return 1.0;
    return (2.0 + 3.0 * v - v * v * v) / 4.0;
}

static double epan_pdf01(double v) /* F'(v) */
{
    if (v <= -1.0 || v >= 1.0) return 0.0;
    return 0.75 * (1.0 - v * v);
}

/* 1-D mass of (l, u) for a point t; +-inf bounds give v = +-inf. */
static double epan_mass1(double t, double h, double l, double u)
{
    return epan_cdf((u - t) / h) - epan_cdf((l - t) / h);
}

static double epan_dmass1_dh(double t, double h, double l, double u)
{
    double vu = (u - t) / h, vl = (l - t) / h;
    double du = isinf(vu) ? 0.0 : epan_pdf01(vu) * (-vu / h);
    double dl = isinf(vl) ? 0.0 : epan_pdf01(vl) * (-vl / h);
    return du - dl;
}

/* p^(i)(Omega) for the Epanechnikov product kernel (eq. 10-11 with K_h). */
double oracle_epan_point_mass(const float *t, int32_t d, const double *h, const float *lo, const float *hi)
{
    double prod = 1.0;
    for (int32_t j = 0; j < d; ++j) prod *= epan_mass1((double)t[j], h[j], (double)lo[j], (double)hi[j]);
    return prod;
}

void oracle_epan_contributions(const float *sample, int64_t n, int32_t d, const double *h,
                               const float *lo, const float *hi, double *c_out)
{
    for (int64_t i = 0; i < n; ++i) c_out[i] = oracle_epan_point_mass(sample + i * d, d, h, lo, hi);
}

/* eq. (2) estimate and its h-gradient (product rule as in eq. 16) for q boxes. */
void oracle_epan_estimate_grad(const float *sample, int64_t n, int32_t d, const double *h,
                               const float *lo, const float *hi, int64_t q, double *est, double *dpdh)
{
    #pragma omp parallel for schedule(dynamic, 1)
    for (int64_t qq = 0; qq < q; ++qq) {
        const float *l = lo + qq * d, *u = hi + qq * d;
        double sum = 0.0, gsum[64];
        for (int32_t i = 0; i < d; ++i) gsum[i] = 0.0;
        for (int64_t j = 0; j < n; ++j) {
            const float *t = sample + j * d;
            sum += oracle_epan_point_mass(t, d, h, l, u);
            for (int32_t i = 0; i < d; ++i) {
                double prod = 1.0;
                for (int32_t k = 0; k < d; ++k) {
                    if (k == i) continue;
                    prod *= epan_mass1((double)t[k], h[k], (double)l[k], (double)u[k]);
                }
                gsum[i] += epan_dmass1_dh((double)t[i], h[i], (double)l[i], (double)u[i]) * prod;
            }
        }
        est[qq] = sum / (double)n;
        if (dpdh)
            for (int32_t i = 0; i < d; ++i) dpdh[qq * d + i] = gsum[i] / (double)n;
    }
}

/* tolerance scale: the derivative terms (both bounds) in absolute value */
void oracle_epan_grad_abs_scale(const float *sample, int64_t n, int32_t d, const double *h,
                                const float *lo, const float *hi, int64_t q, double *mabs)
{
    #pragma omp parallel for schedule(dynamic, 1)
    for (int64_t qq = 0; qq < q; ++qq) {
        const float *l = lo + qq * d, *u = hi + qq * d;
        double gsum[64];
        for (int32_t i = 0; i < d; ++i) gsum[i] = 0.0;
        for (int64_t j = 0; j < n; ++j) {
            const float *t = sample + j * d;
            for (int32_t i = 0; i < d; ++i) {
                double prod = 1.0;
                for (int32_t k = 0; k < d; ++k) {
                    if (k == i) continue;
                    prod *= epan_mass1((double)t[k], h[k], (double)l[k], (double)u[k]);
                }
                double vu = ((double)u[i] - (double)t[i]) / h[i], vl = ((double)l[i] - (double)t[i]) / h[i];
                double a = isinf(vu) ? 0.0 : fabs(epan_pdf01(vu) * vu / h[i]);
                double b = isinf(vl) ? 0.0 : fabs(epan_pdf01(vl) * vl / h[i]);
                gsum[i] += (a + b) * fabs(prod);
            }
        }
        for (int32_t i = 0; i < d; ++i) mabs[qq * d + i] = gsum[i] / (double)n;
    }
}

/* eq. (19)-(20) derivation for the Epanechnikov product kernel:
 * p_max = prod_j M_j(centre), thr = max_j p_max / M_j(centre) * M_j(face). */
double oracle_epan_empty_region_threshold(int32_t d, const double *h, const float *lo, const float *hi,
                                          double *pmax_out)
{
    double pmax = 1.0, best = 0.0;
    int disabled = 0;
    for (int32_t j = 0; j < d; ++j) {
        double w = (double)hi[j] - (double)lo[j];
        if (!(w > 0.0)) { disabled = 1; continue; }
        double centre = isinf(w) ? 1.0 : epan_cdf(w / (2.0 * h[j])) - epan_cdf(-w / (2.0 * h[j]));
        double face = isinf(w) ? 0.5 : epan_cdf(w / h[j]) - epan_cdf(0.0);
        pmax *= centre;
        double ratio = face / centre;
        if (ratio > best) best = ratio;
    }
    if (pmax_out) *pmax_out = disabled ? 0.0 : pmax;
    if (disabled || !(pmax > 0.0)) return INFINITY;
    return pmax * best;
}

/* =====================================================================
 * Reservoir sampling for insert-only workloads (Section 4.2, P:L189 / P:L248:
 * "the well-known reservoir sampling algorithm [43]" adds a newly inserted tuple
 * with probability |S|/|R|, replacing a random point).  Algorithm R, SURVEY.md
 * §8(c) O11: the a-th arriving tuple (a = 1, 2, ...; the first N arrivals fill
 * the sample) draws j uniformly from [0, a) and replaces slot j if j < N.
 * The random draw is a counter-based generator both sides implement from its
 * definition (random numbers the method draws):
 *   z = SplitMix64 finaliser of (seed + a * 0x9E3779B97F4A7C15),
 *   j = floor(z * a / 2^64)            (multiply-shift onto [0, a)).
 * ===================================================================== */
static uint64_t or_splitmix(uint64_t seed, uint64_t a)
{
    uint64_t z = seed + a * 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

/* uniform draw of arrival a in [0, a) */
int64_t oracle_reservoir_draw(uint64_t seed, int64_t a)
{
    return (int64_t)(((unsigned __int128)or_splitmix(seed, (uint64_t)a) * (unsigned __int128)(uint64_t)a) >> 64);
}

/* slot taken by each of k arrivals a = n_seen + 1 .. n_seen + k, or -1 (not sampled) */
void oracle_reservoir_slots(uint64_t seed, int64_t n_sample, int64_t n_seen, int64_t k, int64_t *slot_out)
{
    for (int64_t r = 0; r < k; ++r) {
        const int64_t a = n_seen + r + 1;
        if (a <= n_sample) { slot_out[r] = a - 1; continue; }   /* the first N arrivals fill the sample */
        const int64_t j = oracle_reservoir_draw(seed, a);
        slot_out[r] = j < n_sample ? j : -1;
    }
}

/* Run Algorithm R over arrivals 1..n_total: content[i] = id (1-based arrival) in slot i */
void oracle_reservoir_run(uint64_t seed, int64_t n_sample, int64_t n_total, int64_t *content)
{
    for (int64_t a = 1; a <= n_total; ++a) {
        if (a <= n_sample) { content[a - 1] = a; continue; }
        const int64_t j = oracle_reservoir_draw(seed, a);
        if (j < n_sample) content[j] = a;
    }
}
