/* vista_gen.h — seeded synthetic-input generators (Foods/Amazon-shaped tables,
 * 227x227 images, random-init CNN parameters).
 *
 * This module is the ONLY code shared by the CUDA product path
 * (paper_conf_sigmod_nakandalak20_b200/libvista.so) and the CPU oracle
 * (oracle/liboracle.so).  It holds none of the method's arithmetic: no conv,
 * pooling, tap, join, concat or LR math — only counter-based random numbers and
 * the fixed data recipe of DESIGN.md §"Input recipe" (SURVEY.md §8d "Generator").
 *
 * Paper context: T_str(ID, X) and T_img(ID, I) (§3.2); Foods ~20k rows
 * x 130 structured features, Amazon ~200k rows x (price, 100-d title embedding,
 * 100-d PCA of categories) (§5); images resized to 227x227
 * (PAPER.md:364); pretrained weights replaced by seeded random init
 * (SURVEY.md §8c reading #11).
 *
 * Every function is deterministic in its arguments (no global state) and
 * thread-count independent.
 */
#ifndef VISTA_GEN_H
#define VISTA_GEN_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define VG_DEFAULT_SEED 0x5EED2020ULL
#define VG_IMG_H 227
#define VG_IMG_W 227
#define VG_IMG_C 3
#define VG_IMG_BYTES (227 * 227 * 3)

/* sub-seed stream ids: S_k = mix64(S ^ mix64(k)) */
enum { VG_S_KEY = 1, VG_S_IMG = 2, VG_S_STR = 3, VG_S_LAB = 4, VG_S_W = 5,
       VG_S_SPLIT = 6, VG_S_PERM = 7, VG_S_LAT = 8 };

/* structured-table kinds */
enum { VG_FOODS = 0, VG_AMAZON = 1 };

/* parameter tensor ids inside one parameterised layer */
enum { VG_T_WEIGHT = 0, VG_T_BIAS = 1, VG_T_BN_GAMMA = 2, VG_T_BN_BETA = 3,
       VG_T_BN_MEAN = 4, VG_T_BN_VAR = 5 };

uint64_t vg_mix64(uint64_t x);                 /* splitmix64 finaliser */
uint64_t vg_subseed(uint64_t S, uint64_t k);   /* mix64(S ^ mix64(k)) */
double   vg_u01(uint64_t h);                   /* (h >> 11) * 2^-53 in [0,1) */
double   vg_normal(uint64_t h);                /* Box-Muller N(0,1) from h, mix64(h) */
float    vg_bf16_round(double v);              /* fp64 -> fp32 (RNE) -> bf16 (RNE), returned as float */
void     vg_set_threads(int nthreads);         /* 0 = hardware concurrency */

/* key_r = mix64(S_key + r), r = r0 .. r0+n-1 (a bijection, so keys are unique) */
void vg_keys(uint64_t S, int64_t r0, int64_t n, int64_t* keys);
/* latent z in [-128, 127] carried by the image of this key */
int  vg_latent(uint64_t S, int64_t key);
/* uint8 NHWC [n, 227, 227, 3] pixels, integer-only recipe */
void vg_images(uint64_t S, const int64_t* keys, int64_t n, uint8_t* px);
/* structured features, fp32 [n, d_s] row-major, every value bf16-representable */
void vg_structured(uint64_t S, const int64_t* keys, int64_t n, int32_t d_s, int32_t kind, float* X);
/* binary labels {0,1}; depend on X[:, :5] and on the image latent */
void vg_labels(uint64_t S, const int64_t* keys, const float* X, int64_t n, int32_t d_s, uint8_t* y);
/* Structured-table row list: for the image table rows r = 0..N-1, returns the
 * image-row index r of each structured row, in structured-table order (a
 * Fisher-Yates permutation of the matched rows).  mismatch != 0 drops the rows
 * r % 100 == 99 and appends N/100 extra rows r in [N, N + N/100) that have no
 * image.  rows_out needs capacity N + N/100.  Returns the row count. */
int64_t vg_str_rows(uint64_t S, int64_t N, int32_t mismatch, int64_t* rows_out);

/* Random-init CNN parameters of parameterised layer `layer`, tensor `tensor`,
 * elements e = 0..n-1 (the caller fixes the element order):
 *   kind 0: mean + std * N(0,1)
 *   kind 1: mean + std * U[0,1)
 * round_bf16 != 0 rounds each value to bf16 (RNE) before returning it. */
void vg_param(uint64_t S, int32_t cnn, int32_t layer, int32_t tensor, int64_t n,
              int32_t kind, double mean, double std, int32_t round_bf16, double* out);
/* same values as vg_param(round_bf16=1) but returned as fp32 (exact) */
void vg_param_f32(uint64_t S, int32_t cnn, int32_t layer, int32_t tensor, int64_t n,
                  int32_t kind, double mean, double std, float* out);

#ifdef __cplusplus
}
#endif
#endif
