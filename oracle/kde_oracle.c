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
 *      update is reconstructed from the prose P:L179-183, L561.
 *      PARITY UNPINNED by the paper (no listing, no trace).
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
double oracle_point_mass(const float *t, int32_t d, const double *h,
                         const float *lo, const float *hi)
{
    double prod = 1.0;
    for (int32_t j = 0; j < d; ++j) {
        double u = (double)hi[j], l = (double)lo[j], tj = (double)t[j];
        double diff = erf((u - tj) / (OR_SQRT2 * h[j])) - erf((l - tj) / (OR_SQRT2 * h[j]));
        prod *= diff;
    }
    return prod / pow(2.0, (double)d);
}

/* eq. (13) for every sample point of one query (the retained buffer). */
void oracle_contributions(const float *sample, int64_t n, int32_t d, const double *h,
                          const float *lo, const float *hi, double *c_out)
{
    for (int64_t i = 0; i < n; ++i)
        c_out[i] = oracle_point_mass(sample + i * d, d, h, lo, hi);
}

/* ---------------------------------------------------------------------
 * eq. (2): p_H(Omega) = (1/s) sum_i p^(i)(Omega), index order.
 * ------------------------------------------------------------------- */
void oracle_estimate(const float *sample, int64_t n, int32_t d, const double *h,
                     const float *lo, const float *hi, int64_t q, double *est)
{
    #pragma omp parallel for schedule(dynamic, 1)
    for (int64_t k = 0; k < q; ++k) {
        double sum = 0.0;
        for (int64_t i = 0; i < n; ++i)
            sum += oracle_point_mass(sample + i * d, d, h, lo + k * d, hi + k * d);
        est[k] = sum / (double)n;
    }
}

/* x * exp(-x^2 / (2 h^2)) with the limit value 0 for infinite x (R3). */
static double xexp(double x, double h)
{
    if (isinf(x)) return 0.0;
    return x * exp(-(x * x) / (2.0 * h * h));
}

/* ---------------------------------------------------------------------
 * eq. (17), written literally:
 *   dp/dh_i = sqrt2 / (sqrtpi h_i^2 2^d s) * sum_j [ (l_i - t_i) e^{-(l_i-t_i)^2/2h_i^2}
 *                                                - (u_i - t_i) e^{-(u_i-t_i)^2/2h_i^2} ]
 *             * prod_{k != i} [ erf((u_k - t_k)/(sqrt2 h_k)) - erf((l_k - t_k)/(sqrt2 h_k)) ]
 * Also returns the estimate (eq. 2) of the same query.  The product over
 * k != i is recomputed for every i (O(d^2)), exactly as written.
 * ------------------------------------------------------------------- */
void oracle_estimate_grad(const float *sample, int64_t n, int32_t d, const double *h,
                          const float *lo, const float *hi, int64_t q,
                          double *est, double *dpdh)
{
    #pragma omp parallel for schedule(dynamic, 1)
    for (int64_t qq = 0; qq < q; ++qq) {
        const float *l = lo + qq * d, *u = hi + qq * d;
        double sum = 0.0;
        double gsum[64];
        for (int32_t i = 0; i < d; ++i) gsum[i] = 0.0;
        for (int64_t j = 0; j < n; ++j) {
            const float *t = sample + j * d;
            sum += oracle_point_mass(t, d, h, l, u);
            for (int32_t i = 0; i < d; ++i) {
                double li = (double)l[i] - (double)t[i];
                double ui = (double)u[i] - (double)t[i];
                double bracket = xexp(li, h[i]) - xexp(ui, h[i]);
                double prod = 1.0;
                for (int32_t k = 0; k < d; ++k) {
                    if (k == i) continue;
                    prod *= erf(((double)u[k] - (double)t[k]) / (OR_SQRT2 * h[k]))
                          - erf(((double)l[k] - (double)t[k]) / (OR_SQRT2 * h[k]));
                }
                gsum[i] += bracket * prod;
            }
        }
        est[qq] = sum / (double)n;
        for (int32_t i = 0; i < d; ++i)
            dpdh[qq * d + i] = OR_SQRT2 / (OR_SQRTPI * h[i] * h[i] * pow(2.0, (double)d) * (double)n)
                               * gsum[i];
    }
}

/* Gradient magnitude scale used by the parity tolerance (test infrastructure,
 * not a paper quantity):
 *   m_ij = sqrt2 / (sqrtpi h_i^2 2^d s) * sum_j ( |(l_i - t_i) e^{..}| + |(u_i - t_i) e^{..}| )
 *                                             * | prod_{k != i} [...] |
 * i.e. eq. (17) with both terms of the bracket and every per-point term taken
 * in absolute value -- the condition-number scale of evaluating eq. (17) in
 * finite precision (the bracket cancels when both bounds give equal terms). */
void oracle_grad_abs_scale(const float *sample, int64_t n, int32_t d, const double *h,
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
                double li = (double)l[i] - (double)t[i];
                double ui = (double)u[i] - (double)t[i];
                double bracket = fabs(xexp(li, h[i])) + fabs(xexp(ui, h[i]));
                double prod = 1.0;
                for (int32_t k = 0; k < d; ++k) {
                    if (k == i) continue;
                    prod *= erf(((double)u[k] - (double)t[k]) / (OR_SQRT2 * h[k]))
                          - erf(((double)l[k] - (double)t[k]) / (OR_SQRT2 * h[k]));
                }
                gsum[i] += bracket * fabs(prod);
            }
        }
        for (int32_t i = 0; i < d; ++i)
            mabs[qq * d + i] = OR_SQRT2 / (OR_SQRTPI * h[i] * h[i] * pow(2.0, (double)d) * (double)n)
                               * gsum[i];
    }
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
