/* oracle.h — plain, slow, obviously-correct CPU oracle (fp64) for Vista's
 * feature-transfer workload (§3.2 Eqs. (1)-(4)).
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load liboracle.so.  The product path
 * (libvista.so) never links, loads or calls it, and the two share no code except
 * the seeded input generators in gen/ (which hold no method arithmetic).
 *
 * Layouts: activations NHWC fp64; conv weights OHWI [Cout][R][S][Cin/groups];
 * FC weights [Nout][K] with K in NHWC flatten order.  Parameter values come from
 * gen/vista_gen.h (vg_param) with this file's own architecture tables.
 *
 * Parity status of every exported function: see DESIGN.md §"Oracle pins".
 * Functions marked "parity unpinned" below have no pin independent of themselves.
 */
#ifndef VISTA_ORACLE_H
#define VISTA_ORACLE_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

enum { OR_ALEXNET = 0, OR_VGG16 = 1, OR_RESNET50 = 2 };
enum { OR_OK = 0, OR_ERR_ARG = 1, OR_ERR_DUP_KEY = 3 };

/* ---------- primitives (fp64, NHWC) ---------- */
int or_conv2d(const double* x, int N, int H, int W, int C, const double* w, int Cout, int R, int S,
              int stride, int pad, int groups, const double* bias, double* y);
int or_fc(const double* x, int N, int K, const double* w, int Nout, const double* bias, double* y);
int or_maxpool(const double* x, int N, int H, int W, int C, int k, int s, double* y);
int or_avgpool_global(const double* x, int N, int H, int W, int C, double* y);
int or_lrn(const double* x, int N, int H, int W, int C, double* y);
int or_batchnorm(const double* x, int64_t count, int C, const double* gamma, const double* beta,
                 const double* mean, const double* var, double eps, double* y);
int or_tap(const double* A, int N, int H, int W, int C, double* F);

/* ---------- CNN roster ---------- */
/* Tap ids: AlexNet 0 conv5, 1 fc6, 2 fc7, 3 fc8; VGG16 0 fc6, 1 fc7, 2 fc8;
 * ResNet50 0 conv4_6, 1 conv5_1, 2 conv5_2, 3 conv5_3, 4 fc.
 * info out[8]: H, W, C (activation at the tap; FC taps H=W=1), d (tap width),
 * cumulative MACs from pixels to the tap, cumulative MACs + bias adds,
 * number of taps, activation elements per image. */
int oracle_cnn_info(int cnn, int tap, int64_t* out);

/* Eq. (2) for every requested tap: F_t[i] = g_t(f^_t(x_i)) — a full fp64 forward
 * pass from pixels.  images uint8 NHWC [n,227,227,3].  F[t] (may be NULL for an
 * unrequested tap) receives double [n, d_t].  A[t] (may be NULL) receives the
 * full tap activation double [n, H_t*W_t*C_t] (NHWC).  nthreads 0 = all cores. */
int oracle_features(int cnn, uint64_t weight_seed, const uint8_t* images, int64_t n,
                    double** F, double** A, int nthreads);
/* Partial inference f^_{t0 -> t} (Def 3.7) from the stored
 * activation of tap t0 (A_in double [n, act(t0)]) through every later tap. */
int oracle_features_from(int cnn, uint64_t weight_seed, int t0, const double* A_in, int64_t n,
                         double** F, double** A, int nthreads);

/* ---------- Eq. (3): key-key join ---------- */
/* Emits (s, img_row) for every structured row s whose key matches an image key,
 * in ascending s.  is_test[p] = mix64(key ^ subseed(split_seed, 6)) % 5 == 0.
 * Capacity of the outputs: n_str.  Returns OR_ERR_DUP_KEY if either key column
 * is not a primary key. */
int oracle_join(const int64_t* img_keys, int64_t n_img, const int64_t* str_keys, int64_t n_str,
                uint64_t split_seed, int64_t* pair_str, int64_t* pair_img, uint8_t* is_test,
                int64_t* n_pairs);
/* ---------- Eq. (4): X'_l = [X, g_l(...)] ---------- */
int oracle_concat(const float* X, int d_s, const double* F, int d_l, const int64_t* pair_str,
                  const int64_t* pair_img, int64_t n_pairs, double* MM /* [n_pairs, d_s+d_l] */);

/* ---------- M = elastic-net logistic regression ---------- */
typedef struct {
  int32_t iters;       /* T (10) */
  int32_t power_iters; /* K = 20 */
  double lambda;       /* 0.01 */
  double alpha;        /* 0.5 */
} oracle_lr_cfg;
/* metrics out[10]: train_acc, test_acc, test_f1, n_train, n_test, tp, fp, tn, fn, eta */
int oracle_lr_train(const double* MM, int64_t n, int d, const uint8_t* y, const uint8_t* is_test,
                    const oracle_lr_cfg* cfg, double* w_out, double* b_out, double* loss_out,
                    double* lambda_hat_out, double* metrics_out);
/* step 2 of O6: standardisation statistics over train rows */
int oracle_lr_stats(const double* MM, int64_t n, int d, const uint8_t* is_test, double* mu, double* sigma,
                    double* inv);
/* smooth part of the objective at (w, b) in standardised space and its gradient */
int oracle_lr_objective(const double* MM, int64_t n, int d, const uint8_t* y, const uint8_t* is_test,
                        const double* mu, const double* inv, const double* w, double b, double lambda,
                        double alpha, double* f_out, double* grad_w, double* grad_b);
/* step 3 of O6: power iteration estimate of lambda_max((1/n)[X~,1]^T[X~,1]) */
int oracle_lr_power(const double* MM, int64_t n, int d, const uint8_t* is_test, const double* mu,
                    const double* inv, int K, double* lambda_out);
/* additive per-row sums of one gradient pass on raw rows (the quantity a rank
 * contributes to the allreduce): out[0..d) = sum r_p x_pj, out[d] = sum r_p,
 * out[d+1] = sum loss_p, over train rows, with z_p = b_hat + w_hat . x_p */
int oracle_lr_grad_sums(const double* MM, int64_t n, int d, const uint8_t* y, const uint8_t* is_test,
                        const double* w_hat, double b_hat, double* out);

#ifdef __cplusplus
}
#endif
#endif
