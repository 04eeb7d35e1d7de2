// internal.h — declarations shared by the product's translation units (never by the oracle).
#pragma once
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include <string>
#include <vector>

namespace vista {

typedef __nv_bfloat16 bf16;

// ---- error plumbing: every failing CUDA call becomes a VistaError with a message ----
struct VistaError {
  int status;
  std::string msg;
};
[[noreturn]] void fail(int status, const std::string& msg);
#define VCHECK(x)                                                                                     \
  do {                                                                                                \
    cudaError_t e_ = (x);                                                                             \
    if (e_ != cudaSuccess) ::vista::fail(5, std::string(#x) + ": " + cudaGetErrorString(e_));        \
  } while (0)

// every kernel launch of the library is counted (bench.py reports gpu_launches from it)
void count_launch();
#define LAUNCHED()                      \
  do {                                  \
    VCHECK(cudaGetLastError());         \
    ::vista::count_launch();            \
  } while (0)

// ---- conv / FC layer on the tcgen05 implicit-GEMM kernel ----
// GEMM view per group g: M = N*Ho*Wo output pixels, N = Cg_out, K = R*S*Cg_in,
// A[m, k] = x[n, ho*st - pad + r, wo*st - pad + s, g*Cg_in + c] with k = (r*S + s)*Cg_in + c,
// B[n, k] = w[g*Cg_out + n][k] (padded to Kp, a multiple of 64), D in TMEM (fp32).
struct ConvLayer {
  int Cin = 0, Cout = 0, R = 1, S = 1, stride = 1, pad = 0, groups = 1;  // Cin: channels as stored (padded)
  int Cg_in = 0, Cg_out = 0, K = 0, Kp = 0, BN = 128;
  bool relu = false;
  bool row_mode = false;     // Cin = 8, S <= 8: one k-block per filter row, k = r*64 + s*8 + c
  bool rowview = false;      // stride-1 unpadded conv with S*Cin == 64: one output row per 128-row tile,
                             // A rows = overlapping 128-byte windows of one input row (tiled TMA)
  int K_alg = 0;             // algorithmic reduction length R*S*Cin_real/groups (FLOP accounting)
  bf16* w = nullptr;         // [Cout][Kp]
  float* scale = nullptr;    // [Cout]
  float* shift = nullptr;    // [Cout]
  CUtensorMap tmap_w;        // box {64, BN}, SWIZZLE_128B
  CUtensorMap tmap_w_half;   // box {64, BN / 2}: per-CTA half of a k-block multicast to a CTA pair
};

// Builds the padded weight matrix on the device (from OHWI bf16 on the host, Cin_real <= Cin),
// scale/shift, and the TMA descriptor.
void conv_layer_init(ConvLayer& L, const std::vector<uint16_t>& w_ohwi_bf16, int Cin_real,
                     const std::vector<float>& scale, const std::vector<float>& shift);
void conv_layer_free(ConvLayer& L);
// y[N,Ho,Wo,Cout] = act(scale * conv(x) + shift (+ res)).
// tapf (optional): fp32-bit accumulator [N][4][Cout] (zeroed by the caller) receiving the fused tap
// (2x2-grid maxima); returns false if the tap could not be fused (caller runs launch_tap instead).
bool conv_forward(const ConvLayer& L, const bf16* x, int N, int H, int W, const bf16* res, bf16* y,
                  cudaStream_t st, unsigned int* tapf = nullptr);
// closing 1x1 conv of a projection unit with the projection shortcut in its K loop (conv_tc.cu):
// L = the concatenated layer ([Cout][Kb + Cx] weights, see conv_cat_forward), b [N,Ho,Wo,Kb], x [N,Hx,Wx,Cx]
void conv_cat_forward(const ConvLayer& L, int Cx, const bf16* b, const bf16* x, int N, int Hx, int Wx, int stride,
                      bf16* y, cudaStream_t st);
bool make_rowview_tmap(CUtensorMap* m, const void* x, int N, int H, int W, int C, int Wo);
// N-D bf16 tiled tensor map, 128B swizzle, out-of-bounds elements read as zero
bool make_nd_tmap(CUtensorMap* m, const void* ptr, int rank, const uint64_t* dims, const uint64_t* strides,
                  const uint32_t* box, int swizzle_bytes = 128);  // 128, 32 or 0
// 3x3 / 1 / pad 1 conv with Cin = Cout = 64 and W <= 62 (ResNet res2) issued input-row-major with N = 192
// MMAs (conv3x3_rows.cu), bit-identical to the conv_tc halo path; VISTA_ROWCONV=0 disables it
bool rowconv3x3_supported(const ConvLayer& L, int H, int W);
void rowconv3x3_forward(const ConvLayer& L, const bf16* x, int N, int H, int W, bf16* y, cudaStream_t st);
bool make_plain_tmap(CUtensorMap* m, const void* ptr, int cols, int rows);
// Two chained 1x1 convs of consecutive ResNet units (res_chain.cu): out = ReLU(BN_c(b * Wc) + res) and
// a_next = ReLU(BN_a(out * Wa)) in one kernel, bit-identical to two conv_forward calls.
// La == nullptr: the closing conv alone (no chained opening conv, a_next unused)
bool res_chain_supported(const ConvLayer& Lc, const ConvLayer* La);
void res_chain_forward(const ConvLayer& Lc, const ConvLayer* La, const bf16* b, const bf16* res, bf16* out,
                       bf16* a_next, int N, int H, int W, cudaStream_t st);
// ResNet50 stem: conv1 (s2d row view) + BN + ReLU + pool1 3x3/2 in one kernel (conv1_pool.cu):
// x bf16 [N, 117, 117, 16] space-to-depth input -> y bf16 [N, 56, 56, 64], bit-identical to
// conv_forward + launch_maxpool.
bool conv1_pool_supported(const ConvLayer& L, int H, int W);
void conv1_pool_forward(const ConvLayer& L, const bf16* x, int N, bf16* y, cudaStream_t st);
// F bf16 [n, 4C] <- fp32 tap accumulator (exact: the maxima are bf16 values)
void launch_tap_finalize(const unsigned int* tapf, int64_t count, bf16* F, cudaStream_t st);
inline int conv_out_dim(int H, int k, int s, int p) { return (H + 2 * p - k) / s + 1; }

// ---- fp32 check mode (reading R23): SIMT FFMA conv / FC with fp32 storage ----
struct ConvLayerF32 {
  int Cin = 0, Cout = 0, R = 1, S = 1, stride = 1, pad = 0, groups = 1;
  int Cg_in = 0, Cg_out = 0, K = 0;
  bool relu = false;
  float* w = nullptr;  // [Cout][K]
  float* scale = nullptr;
  float* shift = nullptr;
};
void conv_layer_init_f32(ConvLayerF32& L, const std::vector<float>& w_ohwi, int Cin_real,
                         const std::vector<float>& scale, const std::vector<float>& shift);
void conv_layer_free_f32(ConvLayerF32& L);
void conv_forward_f32(const ConvLayerF32& L, const float* x, int N, int H, int W, const float* res, float* y,
                      cudaStream_t st);
void launch_ingest_f32(const uint8_t* px, int64_t n, float* y, cudaStream_t st);
void launch_ingest_s2d_f32(const uint8_t* px, int64_t n, float* y, cudaStream_t st);
void launch_maxpool_f32(const float* x, int N, int H, int W, int C, int k, int s, float* y, cudaStream_t st);
void launch_lrn_f32(const float* x, int N, int H, int W, int C, float* y, cudaStream_t st);
void launch_avgpool_f32(const float* x, int N, int H, int W, int C, float* y, cudaStream_t st);
void launch_tap_f32(const float* A, int64_t N, int H, int W, int C, float* F, cudaStream_t st);
void launch_concat_f32(const float* X, int d_s, int ds_pad, const float* F, int d_l, const int32_t* pair_str,
                       const int32_t* pair_img, const uint8_t* labels, int64_t n_pairs, int ld, float* MM,
                       uint8_t* y, cudaStream_t st);

// ---- SIMT kernels (memory-bound) ----
void launch_ingest(const uint8_t* px, int64_t n, bf16* y, cudaStream_t st);
void launch_ingest_s2d(const uint8_t* px, int64_t n, bf16* y, cudaStream_t st);
void launch_maxpool(const bf16* x, int N, int H, int W, int C, int k, int s, bf16* y, cudaStream_t st);
void launch_lrn(const bf16* x, int N, int H, int W, int C, bf16* y, cudaStream_t st);
void launch_avgpool(const bf16* x, int N, int H, int W, int C, bf16* y, cudaStream_t st);
void launch_tap(const bf16* A, int64_t N, int H, int W, int C, bf16* F, cudaStream_t st);

// ---- join (Eq. 3) + concat (Eq. 4) ----
struct JoinResult {
  int64_t n_pairs = 0, n_train = 0;
  int dup = 0;
};
// pair_str / pair_img: device int32 [n_str]; rows [0,n_train) train, then test, each in T_str order.
JoinResult join_keys(const int64_t* d_img_keys, int64_t n_img, const int64_t* d_str_keys, int64_t n_str,
                     uint64_t split_subseed, int32_t* d_pair_str, int32_t* d_pair_img, cudaStream_t st);
// bad: device int, OR-ed with 1 when a joined X value is not bf16-representable
void launch_concat(const float* X, int d_s, int ds_pad, const bf16* F, int d_l, const int32_t* pair_str,
                   const int32_t* pair_img, const uint8_t* labels, int64_t n_pairs, int ld, bf16* MM,
                   uint8_t* y, int* bad, cudaStream_t st);

// ---- LR (M) ----
struct LRWork;  // device scratch for one layer
struct LRResult {
  std::vector<double> w;  // [ld] standardised-space weights (pad columns 0)
  double b = 0;
  std::vector<double> loss;
  double lambda_hat = 0, eta = 0;
  int64_t n_train = 0, n_test = 0, tp = 0, fp = 0, tn = 0, fn = 0, train_ok = 0;
};
typedef void (*allreduce_fn)(double* d_buf, int64_t count, cudaStream_t st, void* user);
// asynchronous single-rank training: lr_train enqueues everything on st, copies the results into `pinned`
// (caller-owned pinned host memory of lr_async_bytes(ld, iters)) and records `done`; lr_collect waits for
// it and assembles the LRResult
struct LRAsync {
  void* pinned = nullptr;
  size_t bytes = 0;
  cudaEvent_t done = nullptr;
  int64_t n_rows = 0, n_train = 0;
  int ld = 0, iters = 0;
};
size_t lr_async_bytes(int ld, int iters);
LRResult lr_collect(const LRAsync& a);
LRResult lr_train(const bf16* MM, const uint8_t* y, int64_t n_rows, int64_t n_train, int ld,
                  const uint8_t* real_col_mask_host, int iters, int power_iters, double lambda, double alpha,
                  allreduce_fn allreduce, void* ar_user, cudaStream_t st, LRAsync* async = nullptr,
                  int grid_cap = 0);  // grid_cap > 0: at most that many CTAs per pass (layers trained side by side)
// fp32 check mode: the same passes over fp32 rows (ld a multiple of 8)
LRResult lr_train_f32(const float* MM, const uint8_t* y, int64_t n_rows, int64_t n_train, int ld,
                      const uint8_t* real_col_mask_host, int iters, int power_iters, double lambda, double alpha,
                      allreduce_fn allreduce, void* ar_user, cudaStream_t st);

// ---- second downstream model: 3-layer MLP (reading R30), mlp.cu ----
typedef void (*allreduce_f32_fn)(float* d_buf, int64_t count, cudaStream_t st, void* user);
struct MLPResult {
  std::vector<double> loss;            // mean train loss before each of the T steps
  std::vector<float> W1, b1, W2, b2, w3;  // final weights; W1 [h][d] over the real columns
  float b3 = 0;
  int64_t n_train = 0, n_test = 0, tp = 0, fp = 0, tn = 0, fn = 0, train_ok = 0;
};
// gemm on the tcgen05 kernel (conv_tc.cu): y[m, n] = act(scale[n] * sum_k A[m, k] B[n, k] + shift[n])
void gemm_tn(const bf16* A, int64_t M, int K, int lda, const bf16* B, int N, int ldb, const float* scale,
             const float* shift, bool relu, void* y, bool out_f32, cudaStream_t st, int prof_cls);
// W1p_0 / W2_0 / w3_0: device fp32 initial weights (W1 in the padded [h][roundup(ld, 64)] column layout of MM_k)
MLPResult mlp_train(const bf16* MM, const uint8_t* y, int64_t n_rows, int64_t n_train, int ld,
                    const std::vector<int>& real_cols, const float* W1p_0, const float* W2_0, const float* w3_0,
                    int h, int iters, double lr, bool want_weights, allreduce_fn ar64, allreduce_f32_fn ar32,
                    void* ar_user, cudaStream_t st);

// ---- profiling hooks (class ids as in vista.h vista_profile) ----
struct Profiler;
extern thread_local Profiler* g_prof;
void prof_begin(cudaStream_t st);
void prof_end(cudaStream_t st, int cls, double flops, double bytes, const char* label = nullptr);
bool prof_labels();  // true when per-launch records are logged (VISTA_PROF_LOG)

int num_sms();
// cudaFuncAttributeMaxDynamicSharedMemorySize = bytes for fn on the current device (once per device)
void ensure_smem_attr(const void* fn, int bytes);
void set_sm_budget(int n);  // per-thread grid cap for persistent launches (0 = all SMs)

}  // namespace vista
