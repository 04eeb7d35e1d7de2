/* vista.h — C-ABI of libvista.so: the B200 (sm_100a) hot path of Vista's Staged
 * feature-transfer plan (Nakandala & Kumar, SIGMOD 2020).
 *
 * The workload (§3.2, Eqs. (1)-(4)):
 *     for every l in L:  T'_img,l = Apply(g_l o f^_l) to T_img            (2)
 *                        T'_l     = T_str |><|_ID T'_img,l                 (3)
 *                        train M on X'_l = [X, g_l(f^_l(I))]               (4)
 * executed with the Staged logical plan (Fig 5E): each
 * image goes through the CNN once, the full activation of tapped layer l_k stays
 * resident in HBM and is the input of the partial inference f^_{l_k -> l_k+1}
 * (Def 3.7).  g_l max-pools conv layers to a 2x2 grid of the
 * same depth and flattens (PAPER.md:369 footnote 4, Def 3.5);
 * M = logistic regression, elastic net alpha = 0.5, lambda = 0.01
 * (PAPER.md:433-434).  API input groups follow PAPER.md:171-172 §3.3: system
 * environment, CNN f and |L|, downstream M, tables T_str / T_img.
 *
 * Conventions (all entry points):
 *  - extern "C", never throw, return vista_status (VISTA_OK = 0).  On error the
 *    detail is in vista_last_error(ctx) (ctx NULL = last error of this thread).
 *  - Callers own every array they pass; nothing is retained after a call returns
 *    unless stated.  The ctx owns all device memory it allocates.
 *  - "device or host" pointers are auto-detected with cudaPointerGetAttributes.
 *  - One ctx per GPU and process; a ctx is not thread-safe.
 *  - Order: vista_plan -> vista_transfer -> vista_train(k)*.  vista_train before
 *    vista_transfer returns VISTA_ERR_STATE.
 *  - There is no CPU fallback: without a usable sm_100 device every compute call
 *    returns VISTA_ERR_CUDA.
 */
#ifndef VISTA_H
#define VISTA_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  VISTA_OK = 0,
  VISTA_ERR_INVALID_ARG = 1,
  VISTA_ERR_NO_PLAN = 2,   /* infeasible within the HBM budget (Alg. 1 "throw") */
  VISTA_ERR_DUP_KEY = 3,   /* ID is not a primary key */
  VISTA_ERR_STATE = 4,     /* call order violated */
  VISTA_ERR_CUDA = 5,      /* CUDA error, or no sm_100 device */
  VISTA_ERR_NCCL = 6,
  VISTA_ERR_OOM = 7
} vista_status;

/* CNN roster ("AlexNet [46], VGG16 [61], and ResNet50 [37]") */
typedef enum { VISTA_ALEXNET = 0, VISTA_VGG16 = 1, VISTA_RESNET50 = 2 } vista_cnn;

/* Tap (feature layer) ids per CNN, ascending depth:
 *   AlexNet : 0 conv5, 1 fc6, 2 fc7, 3 fc8          (|L| = 4)
 *   VGG16   : 0 fc6, 1 fc7, 2 fc8                   (|L| = 3)
 *   ResNet50: 0 conv4_6, 1 conv5_1, 2 conv5_2, 3 conv5_3, 4 fc   (top 5 layers) */
enum { VISTA_ALEXNET_CONV5 = 0, VISTA_ALEXNET_FC6 = 1, VISTA_ALEXNET_FC7 = 2, VISTA_ALEXNET_FC8 = 3 };
enum { VISTA_VGG16_FC6 = 0, VISTA_VGG16_FC7 = 1, VISTA_VGG16_FC8 = 2 };
enum { VISTA_RESNET50_CONV4_6 = 0, VISTA_RESNET50_CONV5_1 = 1, VISTA_RESNET50_CONV5_2 = 2,
       VISTA_RESNET50_CONV5_3 = 3, VISTA_RESNET50_FC = 4 };

/* Logical plans (Fig 5): STAGED (Fig 5E, the default), EAGER (Fig 5C: one pass
 * over the images taps every layer of L), LAZY (Fig 5A: one pass from the pixels per layer). */
typedef enum { VISTA_PLAN_STAGED = 0, VISTA_PLAN_EAGER = 1, VISTA_PLAN_LAZY = 2 } vista_plan_kind;
/* Arithmetic of the CNN and of M.
 * VISTA_BF16: bf16 operands on the tcgen05 tensor cores, fp32 accumulate, RNE to bf16 at layer
 *   boundaries; MM_k is bf16 (the product path).
 * VISTA_F32: the fp32 check mode (north_star: "1e-4 in the fp32 check mode"; reading R23): fp32
 *   storage and fp32 FFMA accumulation everywhere, MM_k is fp32.  Every buffer below documented as
 *   "bf16" is then float32. */
typedef enum { VISTA_BF16 = 0, VISTA_F32 = 1 } vista_dtype;

/* Downstream M (reading R17 in DESIGN.md) */
typedef struct {
  int32_t iters;        /* T proximal-gradient iterations; paper: 10 */
  int32_t power_iters;  /* K power iterations for the step size; default 20 */
  double lambda;        /* regularisation, 0.01 */
  double alpha;         /* elastic-net mixing, 0.5 */
  uint64_t split_seed;  /* test row iff mix64(key ^ subseed(split_seed, 6)) % 5 == 0 (20 %) */
} vista_lr_cfg;

/* System environment (PAPER.md:171 first input group) */
typedef struct {
  int32_t rank, world;       /* this process's rank among `world` GPU processes */
  const uint8_t* nccl_uid;   /* 128-byte ncclUniqueId (broadcast by the caller), NULL iff world == 1 */
  int32_t device;            /* CUDA device ordinal */
  uint64_t hbm_budget_bytes; /* 0 = free HBM - 4 GiB reserve */
  vista_dtype dtype;
  vista_plan_kind plan;
  void* stream;              /* cudaStream_t to run on (e.g. torch's current stream); NULL = own stream */
  int32_t micro_batch;       /* images per micro-batch of the first stage; 0 = planner's choice */
  /* Caller-supplied collective, used instead of NCCL when world > 1 and nccl_uid == NULL (e.g. a gloo
   * process group, or ranks that share one GPU, which NCCL refuses).  In-place SUM allreduce of `count`
   * elements of HOST memory across the `world` ranks; dtype 0 = float64, 1 = float32.  Every rank calls
   * it the same number of times with the same counts.  Returns 0 on success (non-zero -> VISTA_ERR_NCCL).
   * The library copies the device partials to the host, calls it, and copies the sums back. */
  int32_t (*allreduce)(void* host_buf, int64_t count, int32_t dtype, void* user);
  void* allreduce_user;      /* passed through to allreduce */
} vista_sys_cfg;

typedef struct vista_ctx vista_ctx;

/* What the planner decided (S6 of SURVEY.md §8a; Eqs. 5, 6, 16 analogues). */
typedef struct {
  int32_t n_layers;          /* |L| */
  int32_t tap[8];            /* tap id of layer k */
  int32_t d_l[8];            /* tap width of layer k */
  int32_t ld[8];             /* row stride (elements) of the multimodal buffer MM_k */
  int32_t micro_batch[8];    /* images per micro-batch of stage k */
  int64_t act_bytes[8];      /* bytes of the resident activation A_k (all local images) */
  int64_t peak_bytes_pred;   /* predicted peak device bytes of vista_transfer */
  int64_t weight_bytes;      /* resident CNN parameters */
  int32_t d_s, ds_pad;       /* structured width and its padded width in MM_k */
  int64_t chunk_images;      /* Staged: images per chunk (== n_images_local unless the budget forces chunking) */
  /* Measured (0 before the first vista_transfer): weight_bytes + the high-water mark of the device memory
   * pool's in-use bytes over the last vista_transfer / vista_transfer_from_base (every buffer the library
   * allocates during a transfer comes from that pool), and the same with the pool's reserved bytes. */
  int64_t peak_bytes_meas;
  int64_t peak_reserved_meas;
  /* The last transfer ran its CNN part (S0-S3 + taps) as one CUDA graph: 0 no, 1 captured, 2 replayed;
   * cnn_graph_kernels = kernels in that graph. */
  int32_t cnn_graph;
  int32_t cnn_graph_kernels;
} vista_plan_info_t;

/* Borrowed view of layer k's outputs on this rank (valid until vista_destroy or the
 * next vista_transfer).  All pointers are device pointers. */
typedef struct {
  void* mm;                /* bf16 (f32 in VISTA_F32) [rows, ld]: columns [0,d_s) = X, [d_s,ds_pad) = 0, [ds_pad, ds_pad+d_l) = F_k, rest 0 */
  int64_t rows;            /* joined rows on this rank: [0, n_train) train, [n_train, rows) test */
  int64_t n_train;
  int32_t ld, d_s, ds_pad, d_l;
  const int32_t* pair_str; /* [rows] structured-table row of MM row p */
  const int32_t* pair_img; /* [rows] local image row of MM row p */
  const uint8_t* labels;   /* [rows] y of MM row p */
  void* features;          /* bf16 [n_images_local, d_l]: F_k = g_k(f^_k(I)) per local image */
  void* activation;        /* bf16 NHWC full activation A_k (NULL once freed by the Staged plan) */
} vista_buffer;

/* Per-layer training results (identical on every rank). */
typedef struct {
  double loss[64];      /* mean logistic loss at each of the first min(T, 64) iterations */
  double lambda_hat;    /* power-iteration estimate of lambda_max */
  double eta;           /* step size 1/L */
  double train_acc, test_acc, test_f1;  /* percent */
  int64_t n_train, n_test, tp, fp, tn, fn;
} vista_metrics;

/* vista_plan(cnn, {L}, |T|, |I|, model) — north star signature.
 *   layers: tap ids in ascending depth (n_layers of them), or layers == NULL and n_top > 0
 *           for the top-|L| layers "starting from the top most layer".
 *   n_str_rows / n_str_feats: |T_str| rows and d_s (X in R^{d_s}).
 *   n_images_local: images this rank will pass to vista_transfer.
 *   weight_seed: seed of the random-init CNN parameters (pretrained weights, PAPER.md:365,
 *           are replaced by seeded random init: DESIGN.md reading R11).
 * Generates and uploads the weights, plans micro-batches and residency within the HBM
 * budget (VISTA_ERR_NO_PLAN if even the smallest plan does not fit), allocates. */
vista_status vista_plan(vista_cnn cnn, const int32_t* layers, int32_t n_layers, int32_t n_top,
                        int64_t n_str_rows, int32_t n_str_feats, int64_t n_images_local,
                        const vista_lr_cfg* model, const vista_sys_cfg* sys, uint64_t weight_seed,
                        vista_ctx** out);
vista_status vista_plan_info(const vista_ctx* ctx, vista_plan_info_t* out);

/* vista_transfer(images, structured, keys) -> per-layer multimodal feature buffers.
 *   images:     uint8 NHWC [n_images_local, 227, 227, 3] (host or device)
 *   image_keys: int64 [n_images_local] (host or device), unique
 *   structured: float32 [n_str_rows, d_s] row-major, values bf16-representable (host or device); a
 *               joined row holding a value with any of its low 16 bits set -> VISTA_ERR_INVALID_ARG
 *               (bf16 path; MM_k stores X in bf16, so such a value could not be kept exactly)
 *   str_keys:   int64 [n_str_rows], unique (host or device)
 *   labels:     uint8 {0,1} [n_str_rows] (host or device)
 * Runs the join once (Eq. 3; broadcast join: T_str is whole on every rank),
 * then stage k = 1..|L|: f^_{l_k-1 -> l_k} from the resident A_{k-1}, tap g_{l_k}, concat
 * (Eq. 4) into MM_k.  Synchronises the stream before returning. */
vista_status vista_transfer(vista_ctx* ctx, const uint8_t* images, const int64_t* image_keys,
                            const float* structured, const int64_t* str_keys, const uint8_t* labels);
vista_status vista_features(const vista_ctx* ctx, int32_t k, vista_buffer* out);

/* ---- Pre-materialised base layer (App. B) ----
 * "a base layer can [be] pre-materialized before hand for later use of exploring other layers"
 * (PAPER.md:714-716); "for the other layers partial CNN inference is performed starting from the
 * base layer".  The base layer is the FIRST requested layer L[0] of the plan.
 *
 * vista_base_shape: out4 = {H, W, C, bytes per element} of one image's base activation A_{L[0]}
 *   (FC layer: H = W = 1, C = d); elements are bf16 (2 bytes), fp32 (4) in VISTA_F32.
 * vista_materialize: base_out <- A_{L[0]} of the n_images_local images, NHWC [n, H, W, C] in the
 *   context's element type: inference from pixels through L[0] only, over the planner's chunks.
 *   images as in vista_transfer.  base_out: caller-owned host (pinned or pageable) or device
 *   buffer of n_images_local * H * W * C elements.  Does not change the vista_features state.
 * vista_transfer_from_base: vista_transfer with the CNN started at the stored base layer: no
 *   inference below L[0]; F_0 = g_{L[0]}(base); A_{L[k]} = f^_{L[0] -> L[k]}(base) for k >= 1
 *   (Def 3.7 partial inference); join, concat and MM_k as vista_transfer.  base: host or device,
 *   the layout vista_materialize writes (read only; a device base is read in place).  Results are
 *   bit-identical to vista_transfer from the pixels the base was materialised from, under every plan:
 *   Staged (stored A_k reused), Eager (one pass base -> all of L) and Lazy ("Lazy-5 with Pre-mat",
 *   one pass from the stored base per layer, recomputing everything above it). */
vista_status vista_base_shape(const vista_ctx* ctx, int64_t* out4);
vista_status vista_materialize(vista_ctx* ctx, const uint8_t* images, void* base_out);
vista_status vista_transfer_from_base(vista_ctx* ctx, const void* base, const int64_t* image_keys,
                                      const float* structured, const int64_t* str_keys, const uint8_t* labels);

/* S4 key join on its own (Eq. (3); broadcast join PAPER.md:279), the kernels
 * vista_transfer runs once per transfer: inner equi-join of the image keys with the structured keys,
 * output pairs (structured row, image row) of the matched rows, train rows first then test rows, each
 * in T_str order (reading R14/R16; test iff mix64(key ^ subseed(split_seed, 6)) % 5 == 0).
 *   img_keys int64 [n_img], str_keys int64 [n_str]: DEVICE pointers, unique keys.
 *   pair_str, pair_img: DEVICE int32 [n_str] (caller-owned), rows [0, *n_pairs) written.
 *   n_pairs, n_train: HOST int64 out.
 * Errors: VISTA_ERR_DUP_KEY if either key column has a duplicate; VISTA_ERR_INVALID_ARG for a key equal
 * to INT64_MIN (the empty-slot marker) or NULL pointers.  Synchronises `stream` before returning. */
vista_status vista_join(const int64_t* img_keys, int64_t n_img, const int64_t* str_keys, int64_t n_str,
                        uint64_t split_seed, int32_t* pair_str, int32_t* pair_img, int64_t* n_pairs,
                        int64_t* n_train, void* stream);

/* vista_train(layer) -> weights / accuracy.  Collective over the `world` ranks (all must call
 * with the same k): per-rank partial sums are combined by an fp64 NCCL allreduce.
 *   weights_out: caller-owned double[d_s + d_l + 1] or NULL: w in standardised space for the
 *                d_s + d_l real columns, then the bias b. */
vista_status vista_train(vista_ctx* ctx, int32_t k, double* weights_out, vista_metrics* out);

/* vista_run: the whole Staged plan (Fig 5E: "train M" on every branch of the inference path)
 * in one call = vista_transfer + vista_train(k) for every layer k (S6 of SURVEY.md §8a).
 * Arguments as vista_transfer; weights_out: NULL or n_layers caller-owned pointers, each NULL or a
 * double[d_s + d_l(k) + 1] as vista_train's; out: NULL or vista_metrics[n_layers].
 * Schedule: M of layer k on a second stream as soon as MM_k exists, beside the partial inference of stage k+1
 * (VISTA_OVERLAP=0: after the transfer, layer by layer); results bit-identical to vista_transfer followed by
 * vista_train(k) for k = 0 .. n_layers-1.  VISTA_LR_BATCH=1 (one rank, bf16): the M of every layer side by side
 * after the transfer, each layer's passes on its own stream with a share of the SMs proportional to its bytes
 * (the same algorithm over fewer CTAs per layer: equal up to the fp32 grouping of the per-CTA partial sums,
 * weights within 2e-4 normwise in the tests).  world > 1 and the fp32 check mode train after the transfer,
 * layer by layer.  Collective like vista_train. */
vista_status vista_run(vista_ctx* ctx, const uint8_t* images, const int64_t* image_keys, const float* structured,
                       const int64_t* str_keys, const uint8_t* labels, double* const* weights_out,
                       vista_metrics* out);

/* ---- second downstream model M: 3-layer MLP ----
 * "train a 3-layer MLP (each hidden layer has 1024 units) for 10 iterations using distributed
 * TF/Horovod".  Reading R30: on the rows of MM_k (the d = d_s + d_l real
 * columns, z-scored with the train statistics of O6 step 2), h1 = ReLU(W1 x + b1), h2 = ReLU(W2 h1 + b2), z = w3 . h2 + b3, mean logistic loss over the
 * train rows, `iters` full-batch gradient-descent steps of size `lr`; initial W1 ~ N(0, 2/d),
 * W2 ~ N(0, 2/h), w3 ~ N(0, 1/h) drawn by the seeded generator (model id 3) and rounded to bf16, biases 0.
 * GEMMs on the tcgen05 tensor cores (bf16 operands, fp32 accumulation), fp32 master weights; data
 * parallel over ranks: one fp32 NCCL allreduce of the gradient sums per step.  Collective (all ranks,
 * same k and cfg).  weights_out (caller-owned, may be NULL): float[h*d + h + h*h + h + h + 1] =
 * W1 [h][d], b1, W2 [h][h], b2, w3, b3.  metrics: loss[t] before step t, train/test accuracy, F1,
 * eta = lr.  Errors: VISTA_ERR_STATE before vista_transfer, VISTA_ERR_INVALID_ARG for hidden != 1024
 * or the fp32 check mode. */
typedef struct {
  int32_t hidden;  /* units per hidden layer, 1024; 0 = 1024 */
  int32_t iters;   /* gradient steps, 10; 0 = 10 */
  double lr;       /* step size; 0 = 0.01 */
  uint64_t seed;   /* initial-weight seed */
} vista_mlp_cfg;
vista_status vista_train_mlp(vista_ctx* ctx, int32_t k, const vista_mlp_cfg* cfg, float* weights_out,
                             vista_metrics* out);

void vista_destroy(vista_ctx* ctx);
const char* vista_status_str(vista_status s);
const char* vista_last_error(const vista_ctx* ctx);

/* Image-row shard of `rank` among `world` ranks: [floor(r N / G), floor((r+1) N / G)).
 * Host-only (no GPU needed). */
void vista_shard_range(int64_t n, int32_t rank, int32_t world, int64_t* begin, int64_t* end);

/* 128-byte ncclUniqueId for vista_sys_cfg.nccl_uid (call on rank 0, broadcast the bytes). */
vista_status vista_nccl_unique_id(uint8_t* out128);

/* Per-kernel-class device time accumulated since the last reset when profiling is on
 * (CUDA events around every launch on the ctx stream; adds launch gaps, so bench.py
 * uses it only in a separate instrumented step).  classes: 0 conv/fc tensor-core GEMM,
 * 1 tap, 2 pools/cvt/lrn, 3 join, 4 concat, 5 LR passes, 6 LR small kernels.
 * ms[c], launches[c], flops[c] (algorithmic FLOPs, conv class), bytes[c] (algorithmic bytes),
 * roof_ms[c] = sum over the class's launches of max(flops / peak FLOP/s, bytes / peak B/s): the time
 * each launch would take at the roofline of vista_set_roofline's peaks (0 until they are set). */
typedef struct {
  double ms[8];
  int64_t launches[8];
  double flops[8];
  double bytes[8];
  double roof_ms[8];
} vista_profile;  /* classes: 0 conv/FC/GEMM (tcgen05), 1 tap, 2 pool/convert/LRN, 3 join, 4 concat, 5 LR pass,
                     6 LR small, 7 MLP (its tcgen05 GEMMs, transposes, head, update) */
vista_status vista_set_profiling(vista_ctx* ctx, int32_t on);
/* Peaks for vista_profile.roof_ms: dense tensor TFLOP/s and HBM GB/s (e.g. MEASURED_PEAKS.json). */
vista_status vista_set_roofline(vista_ctx* ctx, double tflops, double gbps);
/* Number of kernels this process has launched through libvista.so so far (all ctxs). */
int64_t vista_kernel_launches(void);
vista_status vista_get_profile(vista_ctx* ctx, vista_profile* out, int32_t reset);

/* ---------------- kernel-level entry points (for parity tests of single ops) ----------------
 * Device pointers only; run on `stream` (NULL = legacy default) and synchronise before
 * returning.  They allocate and free their own scratch.
 *
 * vista_conv2d: y = act(scale * conv(x, w) + shift (+ residual)) in bf16 NHWC on the tcgen05
 *   implicit-GEMM kernel (Def 3.3 TensorOp; BN/bias epilogue, reading R12).
 *   x bf16 [N,H,W,C] (C % 8 == 0), w bf16 OHWI [Cout,R,S,C/groups], scale/shift fp32 [Cout],
 *   residual bf16 [N,Ho,Wo,Cout] or NULL, relu 0/1, y bf16 [N,Ho,Wo,Cout]. */
vista_status vista_conv2d(const void* x, int32_t N, int32_t H, int32_t W, int32_t C, const void* w,
                          int32_t Cout, int32_t R, int32_t S, int32_t stride, int32_t pad, int32_t groups,
                          const float* scale, const float* shift, const void* residual, int32_t relu,
                          void* y, void* stream);
/* The same conv with ReLU and the tap g_l (PAPER.md:369 fn 4) fused into its epilogue: y as in
 * vista_conv2d (groups 1, relu 1) and F bf16 [N, 4*Cout] = 2x2-grid maxima of y (NHWC flatten).
 * VISTA_ERR_INVALID_ARG when the shape cannot take the fused path (short-K TMA epilogue, Ho*Wo >= 43). */
vista_status vista_conv2d_tap(const void* x, int32_t N, int32_t H, int32_t W, int32_t C, const void* w, int32_t Cout,
                              int32_t R, int32_t S, int32_t stride, int32_t pad, const float* scale,
                              const float* shift, const void* residual, void* y, void* F, void* stream);
/* g_l on a conv activation: A bf16 [N,H,W,C] -> F bf16 [N,4C] (2x2 grid max, NHWC flatten). */
vista_status vista_tap(const void* A, int32_t N, int32_t H, int32_t W, int32_t C, void* F, void* stream);
/* unpadded max pool k/s, bf16 NHWC */
vista_status vista_maxpool(const void* x, int32_t N, int32_t H, int32_t W, int32_t C, int32_t k, int32_t s,
                           void* y, void* stream);
/* AlexNet LRN (Caffe constants), bf16 NHWC */
vista_status vista_lrn(const void* x, int32_t N, int32_t H, int32_t W, int32_t C, void* y, void* stream);
/* global average pool bf16 [N,H,W,C] -> bf16 [N,C] */
vista_status vista_avgpool(const void* x, int32_t N, int32_t H, int32_t W, int32_t C, void* y, void* stream);
/* ingest: uint8 NHWC [N,227,227,3] -> bf16 NHWC [N,227,227,8], x = (p - 128) / 128, channels 3..7 = 0 */
vista_status vista_ingest(const uint8_t* px, int32_t N, void* y, void* stream);

#ifdef __cplusplus
}
#endif
#endif
