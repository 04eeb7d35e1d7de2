/* vista_gen.c — seeded synthetic-input generators.  See vista_gen.h.
 * Recipe: DESIGN.md §"Input recipe" (restates SURVEY.md §8d "Generator").
 * No method arithmetic lives here. */
#include "vista_gen.h"

#include <math.h>
#include <pthread.h>
#include <stdlib.h>
#include <string.h>
#include <unistd.h>

static int g_threads = 0;

void vg_set_threads(int nthreads) { g_threads = nthreads; }

static int n_threads(void) {
  if (g_threads > 0) return g_threads;
  long c = sysconf(_SC_NPROCESSORS_ONLN);
  return c > 0 ? (int)c : 1;
}

uint64_t vg_mix64(uint64_t x) {
  x += 0x9E3779B97F4A7C15ULL;
  x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ULL;
  x = (x ^ (x >> 27)) * 0x94D049BB133111EBULL;
  return x ^ (x >> 31);
}

uint64_t vg_subseed(uint64_t S, uint64_t k) { return vg_mix64(S ^ vg_mix64(k)); }

double vg_u01(uint64_t h) { return (double)(h >> 11) * (1.0 / 9007199254740992.0); }

double vg_normal(uint64_t h) {
  double u1 = 1.0 - vg_u01(h);            /* (0, 1] */
  double u2 = vg_u01(vg_mix64(h));
  return sqrt(-2.0 * log(u1)) * cos(6.283185307179586 * u2);
}

float vg_bf16_round(double v) {
  float f = (float)v;
  uint32_t u;
  memcpy(&u, &f, 4);
  if ((u & 0x7f800000u) == 0x7f800000u) return f; /* inf / nan unchanged */
  uint32_t lsb = (u >> 16) & 1u;
  u = (u + 0x7fffu + lsb) & 0xffff0000u;
  memcpy(&f, &u, 4);
  return f;
}

void vg_keys(uint64_t S, int64_t r0, int64_t n, int64_t* keys) {
  uint64_t sk = vg_subseed(S, VG_S_KEY);
  for (int64_t i = 0; i < n; ++i) keys[i] = (int64_t)vg_mix64(sk + (uint64_t)(r0 + i));
}

int vg_latent(uint64_t S, int64_t key) {
  uint64_t sl = vg_subseed(S, VG_S_LAT);
  return (int)(vg_mix64(sl ^ (uint64_t)key) >> 56) - 128;
}

/* ---- images: threads over images ---- */
typedef struct {
  uint64_t S;
  const int64_t* keys;
  int64_t n;
  uint8_t* px;
  int64_t next;
  pthread_mutex_t mu;
} img_job;

static void image_one(uint64_t s_img, int z, int64_t key, uint8_t* out) {
  uint64_t u = vg_mix64(s_img ^ (uint64_t)key);
  int f1 = 1 + (int)(u & 7u);
  int f2 = 1 + (int)((u >> 3) & 7u);
  int phi[3];
  for (int c = 0; c < 3; ++c) phi[c] = (int)((u >> (8 + 9 * c)) & 511u);
  for (int h = 0; h < VG_IMG_H; ++h)
    for (int w = 0; w < VG_IMG_W; ++w)
      for (int c = 0; c < 3; ++c) {
        int t = (h * f1 + w * f2 + phi[c]) % 454;
        int tri = abs(t - 227) - 113;
        uint64_t idx = (uint64_t)((h * VG_IMG_W + w) * 3 + c);
        int noise = (int)(vg_mix64(u ^ idx) & 63u) - 32;
        int p = 128 + (z * tri) / 128 + noise; /* C truncating division */
        if (p < 0) p = 0;
        if (p > 255) p = 255;
        out[idx] = (uint8_t)p;
      }
}

static void* image_worker(void* arg) {
  img_job* j = (img_job*)arg;
  uint64_t s_img = vg_subseed(j->S, VG_S_IMG);
  for (;;) {
    pthread_mutex_lock(&j->mu);
    int64_t i = j->next;
    j->next += 16;
    pthread_mutex_unlock(&j->mu);
    if (i >= j->n) break;
    int64_t e = i + 16 < j->n ? i + 16 : j->n;
    for (; i < e; ++i)
      image_one(s_img, vg_latent(j->S, j->keys[i]), j->keys[i], j->px + (size_t)i * VG_IMG_BYTES);
  }
  return NULL;
}

void vg_images(uint64_t S, const int64_t* keys, int64_t n, uint8_t* px) {
  img_job j;
  j.S = S; j.keys = keys; j.n = n; j.px = px; j.next = 0;
  pthread_mutex_init(&j.mu, NULL);
  int nt = n_threads();
  if (nt > 256) nt = 256;
  if ((int64_t)nt > n / 16 + 1) nt = (int)(n / 16 + 1);
  pthread_t th[256];
  for (int t = 1; t < nt; ++t) pthread_create(&th[t], NULL, image_worker, &j);
  image_worker(&j);
  for (int t = 1; t < nt; ++t) pthread_join(th[t], NULL);
  pthread_mutex_destroy(&j.mu);
}

void vg_structured(uint64_t S, const int64_t* keys, int64_t n, int32_t d_s, int32_t kind, float* X) {
  uint64_t ss = vg_subseed(S, VG_S_STR);
  for (int64_t i = 0; i < n; ++i) {
    uint64_t kh = vg_mix64((uint64_t)keys[i]);
    for (int32_t j = 0; j < d_s; ++j) {
      double v = vg_normal(vg_mix64(ss ^ kh ^ vg_mix64((uint64_t)j + 0x51ULL)));
      if (kind == VG_AMAZON && j > 100) v *= 1.0 / sqrt((double)(j - 100));
      X[(size_t)i * d_s + j] = vg_bf16_round(v);
    }
  }
}

void vg_labels(uint64_t S, const int64_t* keys, const float* X, int64_t n, int32_t d_s, uint8_t* y) {
  uint64_t sl = vg_subseed(S, VG_S_LAB);
  int m = d_s < 5 ? d_s : 5;
  for (int64_t i = 0; i < n; ++i) {
    double s = 0.0;
    for (int j = 0; j < m; ++j) s += (double)X[(size_t)i * d_s + j];
    double logit = 0.8 * s / sqrt(5.0) + 1.5 * (double)vg_latent(S, keys[i]) / 64.0;
    double p = 1.0 / (1.0 + exp(-logit));
    y[i] = vg_u01(vg_mix64(sl ^ (uint64_t)keys[i])) < p ? 1 : 0;
  }
}

int64_t vg_str_rows(uint64_t S, int64_t N, int32_t mismatch, int64_t* rows) {
  int64_t n = 0;
  for (int64_t r = 0; r < N; ++r)
    if (!mismatch || r % 100 != 99) rows[n++] = r;
  if (mismatch)
    for (int64_t r = N; r < N + N / 100; ++r) rows[n++] = r;
  uint64_t sp = vg_subseed(S, VG_S_PERM);
  for (int64_t i = n - 1; i > 0; --i) {
    int64_t j = (int64_t)(vg_mix64(sp ^ vg_mix64((uint64_t)i)) % (uint64_t)(i + 1));
    int64_t t = rows[i]; rows[i] = rows[j]; rows[j] = t;
  }
  return n;
}

static uint64_t param_stream(uint64_t S, int32_t cnn, int32_t layer, int32_t tensor) {
  uint64_t sw = vg_subseed(S, VG_S_W);
  return vg_mix64(sw ^ vg_mix64(((uint64_t)(uint32_t)cnn << 40) ^ ((uint64_t)(uint32_t)layer << 8) ^
                                (uint64_t)(uint32_t)tensor));
}

typedef struct {
  uint64_t st;
  int64_t n;
  int32_t kind;
  double mean, std;
  int32_t round_bf16;
  double* out;
  float* outf;
  int nt;
  int tid;
} param_job;

static void* param_worker(void* arg) {
  param_job* j = (param_job*)arg;
  int64_t per = (j->n + j->nt - 1) / j->nt;
  int64_t b = (int64_t)j->tid * per, e = b + per < j->n ? b + per : j->n;
  for (int64_t i = b; i < e; ++i) {
    uint64_t h = vg_mix64(j->st + (uint64_t)i);
    double r = j->kind == 0 ? vg_normal(h) : vg_u01(h);
    double v = j->mean + j->std * r;
    if (j->round_bf16 || j->outf) v = (double)vg_bf16_round(v);
    if (j->out) j->out[i] = v;
    if (j->outf) j->outf[i] = (float)v;
  }
  return NULL;
}

static void param_run(uint64_t S, int32_t cnn, int32_t layer, int32_t tensor, int64_t n, int32_t kind,
                      double mean, double std, int32_t round_bf16, double* out, float* outf) {
  int nt = n_threads();
  if (nt > 256) nt = 256;
  if (n < 65536) nt = 1;
  param_job jobs[256];
  pthread_t th[256];
  for (int t = 0; t < nt; ++t) {
    param_job j = {param_stream(S, cnn, layer, tensor), n, kind, mean, std, round_bf16, out, outf, nt, t};
    jobs[t] = j;
  }
  for (int t = 1; t < nt; ++t) pthread_create(&th[t], NULL, param_worker, &jobs[t]);
  param_worker(&jobs[0]);
  for (int t = 1; t < nt; ++t) pthread_join(th[t], NULL);
}

void vg_param(uint64_t S, int32_t cnn, int32_t layer, int32_t tensor, int64_t n, int32_t kind,
              double mean, double std, int32_t round_bf16, double* out) {
  param_run(S, cnn, layer, tensor, n, kind, mean, std, round_bf16, out, NULL);
}

void vg_param_f32(uint64_t S, int32_t cnn, int32_t layer, int32_t tensor, int64_t n, int32_t kind,
                  double mean, double std, float* out) {
  param_run(S, cnn, layer, tensor, n, kind, mean, std, 1, NULL, out);
}
