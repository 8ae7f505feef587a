/* c_api_example.c -- the C ABI used from plain C (no Python, no torch).
 *
 *   gcc -O2 -I include examples/c_api_example.c \
 *       -L paper_conf_sigmod_heimelkm15_b200 -lkde -Wl,-rpath,$PWD/paper_conf_sigmod_heimelkm15_b200 -o c_api_example
 *
 * Builds a model on a small synthetic sample (Scott bandwidth, eq. 3), estimates
 * a few boxes with gradients, evaluates the batch loss (eq. 5), runs one karma
 * pass and replaces the flagged points.  Exit code 0 on success. */
#include <math.h>
#include <stdio.h>
#include <stdlib.h>

#include "kde.h"

#define CHECK(x)                                                                         \
  do {                                                                                   \
    kde_status s_ = (x);                                                                 \
    if (s_ != KDE_OK && s_ != KDE_ETRUNC) {                                              \
      fprintf(stderr, "%s -> %s: %s\n", #x, kde_status_string(s_), kde_last_error());    \
      return 1;                                                                          \
    }                                                                                    \
  } while (0)

static float urand(unsigned *s) {
  *s = *s * 1664525u + 1013904223u;
  return (float)((*s >> 8) * (1.0 / 16777216.0));
}

int main(void) {
  enum { N = 10000, D = 3, Q = 4 };
  static float sample[N * D];
  unsigned seed = 12345u;
  for (int i = 0; i < N * D; ++i) sample[i] = 10.0f * urand(&seed) + 5.0f * urand(&seed);
  kde_model *m = NULL;
  CHECK(kde_create(sample, N, D, NULL, &m));
  double h[D];
  CHECK(kde_get_bandwidth(m, h));
  printf("Scott h = %.6f %.6f %.6f\n", h[0], h[1], h[2]);

  float lo[Q * D], hi[Q * D];
  for (int k = 0; k < Q; ++k)
    for (int j = 0; j < D; ++j) {
      lo[k * D + j] = 3.0f + k;
      hi[k * D + j] = 9.0f + k;
    }
  double est[Q], grad[Q * D];
  CHECK(kde_estimate_batch(m, lo, hi, Q, est, grad));
  for (int k = 0; k < Q; ++k) printf("box %d: p_hat = %.9f  dp/dh0 = %.3e\n", k, est[k], grad[k * D]);

  double truth[Q] = {0.2, 0.15, 0.1, 0.05}, loss, g[D];
  CHECK(kde_loss_and_grad(m, lo, hi, truth, Q, KDE_LOSS_SQUARED, 0.0, 1, &loss, g, NULL));
  printf("L2 loss = %.6e, dL/dln h = %.3e %.3e %.3e\n", loss, g[0], g[1], g[2]);

  kde_karma_params kp = {KDE_LOSS_ABSOLUTE, 1, 0.0, 4.0, 0.0, -1.0 / (N - 1)};
  int64_t idx[N], nflag = 0;
  CHECK(kde_set_retain(m, 1));
  CHECK(kde_estimate_batch(m, lo, hi, 1, est, NULL));
  CHECK(kde_karma_update(m, lo, hi, 0.0, &kp, idx, N, &nflag));
  printf("karma pass with true selectivity 0: %lld points flagged\n", (long long)nflag);
  if (nflag > 0) {
    float *rows = (float *)malloc(sizeof(float) * (size_t)nflag * D);
    for (int64_t r = 0; r < nflag * D; ++r) rows[r] = 20.0f + urand(&seed);
    CHECK(kde_replace_points(m, idx, rows, nflag, 0.0));
    free(rows);
  }
  double after;
  CHECK(kde_estimate_batch(m, lo, hi, 1, &after, NULL));
  printf("p_hat after replacement = %.9f (was %.9f)\n", after, est[0]);
  kde_destroy(m);
  return (isfinite(after) && after <= est[0]) ? 0 : 2;
}
