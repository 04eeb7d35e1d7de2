// join.cu — S4 of SURVEY.md §8a: the key-key join T_str |><|_ID T'_img,l (Eq. (3),
// PAPER.md:146) as a broadcast hash join (T_str replicated on every rank, a local hash
// table on the join key), then the concatenation X'_l = [X, F_l]
// (Eq. (4)) into the bf16 multimodal buffer MM_l.
//
// Output order (reading R14/R16): pairs (str_row, img_row) of the matched structured
// rows, train rows first then test rows, each in T_str order — a stable partition, so the
// result is unique and independent of thread scheduling.  Integer work: bit-exact.
#include "internal.h"
#include "ptx.cuh"

namespace vista {

constexpr unsigned long long kEmpty = 0x8000000000000000ULL;  // INT64_MIN marks an empty slot

__device__ __forceinline__ uint64_t dmix64(uint64_t x) {  // splitmix64 finaliser
  x += 0x9E3779B97F4A7C15ULL;
  x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ULL;
  x = (x ^ (x >> 27)) * 0x94D049BB133111EBULL;
  return x ^ (x >> 31);
}

// open addressing, linear probing; value written after the CAS wins the slot
__global__ void hash_build_kernel(const int64_t* __restrict__ keys, int64_t n, unsigned long long* tkeys,
                                  int32_t* tvals, uint64_t mask, int* flags) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const unsigned long long k = (unsigned long long)keys[i];
    if (k == kEmpty) {
      atomicOr(flags, 2);
      continue;
    }
    uint64_t h = dmix64(k) & mask;
    for (;;) {
      const unsigned long long prev = atomicCAS(&tkeys[h], kEmpty, k);
      if (prev == kEmpty) {
        if (tvals) tvals[h] = (int32_t)i;
        break;
      }
      if (prev == k) {
        atomicOr(flags, 1);  // duplicate key: ID is not a primary key
        break;
      }
      h = (h + 1) & mask;
    }
  }
}

// match[s] = image row of structured row s or -1; cls[s] = 0 unmatched, 1 train, 2 test
__global__ void hash_probe_kernel(const int64_t* __restrict__ keys, int64_t n, const unsigned long long* tkeys,
                                  const int32_t* tvals, uint64_t mask, uint64_t split_ss, int32_t* match,
                                  uint8_t* cls) {
  for (int64_t s = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; s < n; s += (int64_t)gridDim.x * blockDim.x) {
    const unsigned long long k = (unsigned long long)keys[s];
    uint64_t h = dmix64(k) & mask;
    int32_t row = -1;
    for (;;) {
      const unsigned long long t = tkeys[h];
      if (t == kEmpty) break;
      if (t == k) {
        row = tvals[h];
        break;
      }
      h = (h + 1) & mask;
    }
    match[s] = row;
    cls[s] = row < 0 ? 0 : ((dmix64(k ^ split_ss) % 5ull) == 0 ? 2 : 1);
  }
}

constexpr int kScanBlock = 1024;
void fill_u64(unsigned long long* p, uint64_t n, unsigned long long v, cudaStream_t st);

// per-block counts of train / test matches
__global__ void count_kernel(const uint8_t* __restrict__ cls, int64_t n, int32_t* counts /*[2][nblk]*/, int nblk) {
  __shared__ int s_tr[32], s_te[32];
  const int64_t i = blockIdx.x * (int64_t)kScanBlock + threadIdx.x;
  const uint8_t c = i < n ? cls[i] : 0;
  const unsigned btr = __ballot_sync(0xffffffffu, c == 1), bte = __ballot_sync(0xffffffffu, c == 2);
  const int w = threadIdx.x >> 5;
  if ((threadIdx.x & 31) == 0) {
    s_tr[w] = __popc(btr);
    s_te[w] = __popc(bte);
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    int a = 0, b = 0;
    for (int j = 0; j < kScanBlock / 32; ++j) {
      a += s_tr[j];
      b += s_te[j];
    }
    counts[blockIdx.x] = a;
    counts[nblk + blockIdx.x] = b;
  }
}

// exclusive scan of the block counts (single block, sequential chunks) -> offsets; totals at [2*nblk]
__global__ void scan_counts_kernel(int32_t* counts, int nblk, int64_t* totals) {
  if (threadIdx.x != 0 || blockIdx.x != 0) return;
  int64_t a = 0, b = 0;
  for (int j = 0; j < nblk; ++j) {
    const int32_t ca = counts[j], cb = counts[nblk + j];
    counts[j] = (int32_t)a;
    counts[nblk + j] = (int32_t)b;
    a += ca;
    b += cb;
  }
  totals[0] = a;  // n_train
  totals[1] = b;  // n_test
}

__global__ void scatter_kernel(const uint8_t* __restrict__ cls, const int32_t* __restrict__ match, int64_t n,
                               const int32_t* offs, int nblk, const int64_t* totals, int32_t* pair_str,
                               int32_t* pair_img) {
  __shared__ int s_tr[32], s_te[32];
  const int64_t i = blockIdx.x * (int64_t)kScanBlock + threadIdx.x;
  const uint8_t c = i < n ? cls[i] : 0;
  const unsigned btr = __ballot_sync(0xffffffffu, c == 1), bte = __ballot_sync(0xffffffffu, c == 2);
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (lane == 0) {
    s_tr[w] = __popc(btr);
    s_te[w] = __popc(bte);
  }
  __syncthreads();
  if (c == 0) return;
  int before = 0;
  const int* arr = c == 1 ? s_tr : s_te;
  for (int j = 0; j < w; ++j) before += arr[j];
  const unsigned lanemask = (1u << lane) - 1u;
  before += __popc((c == 1 ? btr : bte) & lanemask);
  const int64_t pos = c == 1 ? (int64_t)offs[blockIdx.x] + before : totals[0] + offs[nblk + blockIdx.x] + before;
  pair_str[pos] = (int32_t)i;
  pair_img[pos] = match[i];
}

JoinResult join_keys(const int64_t* img_keys, int64_t n_img, const int64_t* str_keys, int64_t n_str,
                     uint64_t split_ss, int32_t* pair_str, int32_t* pair_img, cudaStream_t st) {
  JoinResult res;
  if (n_img > INT32_MAX || n_str > INT32_MAX) fail(1, "join: more than 2^31 rows");
  uint64_t cap = 1024;
  while (cap < 2 * (uint64_t)(n_img > n_str ? n_img : n_str)) cap <<= 1;
  const int nblk = (int)((n_str + kScanBlock - 1) / kScanBlock);
  // one scratch allocation: image table, structured-key table (dup check), match, cls, counts, flags, totals
  size_t off = 0;
  auto carve = [&](size_t bytes) { size_t o = off; off += (bytes + 255) & ~(size_t)255; return o; };
  const size_t o_tk = carve(cap * 8), o_tv = carve(cap * 4), o_sk = carve(cap * 8), o_match = carve(n_str * 4 + 4),
               o_cls = carve(n_str + 1), o_cnt = carve((size_t)2 * nblk * 4 + 8), o_flags = carve(16),
               o_tot = carve(16);
  uint8_t* scratch = nullptr;
  VCHECK(cudaMallocAsync(&scratch, off, st));
  auto* tk = reinterpret_cast<unsigned long long*>(scratch + o_tk);
  auto* tv = reinterpret_cast<int32_t*>(scratch + o_tv);
  auto* sk = reinterpret_cast<unsigned long long*>(scratch + o_sk);
  auto* match = reinterpret_cast<int32_t*>(scratch + o_match);
  auto* cls = scratch + o_cls;
  auto* cnt = reinterpret_cast<int32_t*>(scratch + o_cnt);
  auto* flags = reinterpret_cast<int*>(scratch + o_flags);
  auto* tot = reinterpret_cast<int64_t*>(scratch + o_tot);
  fill_u64(tk, cap, kEmpty, st);
  fill_u64(sk, cap, kEmpty, st);
  VCHECK(cudaMemsetAsync(flags, 0, 16, st));
  const int threads = 256;
  auto grid = [&](int64_t n) {
    int64_t b = (n + threads - 1) / threads;
    int64_t cap2 = (int64_t)num_sms() * 16;
    return (int)(b < 1 ? 1 : (b > cap2 ? cap2 : b));
  };
  prof_begin(st);
  hash_build_kernel<<<grid(n_img), threads, 0, st>>>(img_keys, n_img, tk, tv, cap - 1, flags);
  LAUNCHED();
  hash_build_kernel<<<grid(n_str), threads, 0, st>>>(str_keys, n_str, sk, nullptr, cap - 1, flags);
  LAUNCHED();
  hash_probe_kernel<<<grid(n_str), threads, 0, st>>>(str_keys, n_str, tk, tv, cap - 1, split_ss, match, cls);
  LAUNCHED();
  if (nblk > 0) {
    count_kernel<<<nblk, kScanBlock, 0, st>>>(cls, n_str, cnt, nblk);
    LAUNCHED();
  }
  scan_counts_kernel<<<1, 32, 0, st>>>(cnt, nblk, tot);
  LAUNCHED();
  if (nblk > 0) {
    scatter_kernel<<<nblk, kScanBlock, 0, st>>>(cls, match, n_str, cnt, nblk, tot, pair_str, pair_img);
    LAUNCHED();
  }
  prof_end(st, 3, 0, 8.0 * (n_img + 2.0 * n_str) + 16.0 * (n_img + n_str) + 8.0 * n_str);
  int64_t h_tot[2];
  int h_flags;
  VCHECK(cudaMemcpyAsync(h_tot, tot, 16, cudaMemcpyDeviceToHost, st));
  VCHECK(cudaMemcpyAsync(&h_flags, flags, 4, cudaMemcpyDeviceToHost, st));
  VCHECK(cudaFreeAsync(scratch, st));
  VCHECK(cudaStreamSynchronize(st));
  res.n_train = h_tot[0];
  res.n_pairs = h_tot[0] + h_tot[1];
  res.dup = h_flags;
  return res;
}

__global__ void fill_u64_kernel(unsigned long long* p, uint64_t n, unsigned long long v) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
    p[i] = v;
}
void fill_u64(unsigned long long* p, uint64_t n, unsigned long long v, cudaStream_t st) {
  uint64_t b = (n + 255) / 256;
  if (b > (uint64_t)num_sms() * 16) b = (uint64_t)num_sms() * 16;
  fill_u64_kernel<<<(unsigned)(b ? b : 1), 256, 0, st>>>(p, n, v);
  LAUNCHED();
}

// ---- concat (Eq. (4)): one warp per MM row, 16-byte stores ----
// MM[p] = [bf16(X[s_p, 0..d_s)), 0 .. ds_pad, F[i_p, 0..d_l), 0 .. ld];  y[p] = labels[s_p].
// X values must be bf16-representable (include/vista.h precondition), so the conversion is exact; a value
// with any of its low 16 bits set sets *bad (vista_transfer then fails with VISTA_ERR_INVALID_ARG).
__global__ void concat_kernel(const float* __restrict__ X, int d_s, int ds_pad, const bf16* __restrict__ F, int d_l,
                              const int32_t* __restrict__ pair_str, const int32_t* __restrict__ pair_img,
                              const uint8_t* __restrict__ labels, int64_t n, int ld, bf16* __restrict__ MM,
                              uint8_t* __restrict__ y, int* __restrict__ bad) {
  const int lane = threadIdx.x & 31;
  const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
  for (int64_t p = blockIdx.x * (int64_t)(blockDim.x >> 5) + (threadIdx.x >> 5); p < n; p += warps) {
    const int32_t s = pair_str[p], i = pair_img[p];
    bf16* row = MM + (size_t)p * ld;
    const float* xs = X + (size_t)s * d_s;
    for (int c8 = lane; c8 * 8 < ds_pad; c8 += 32) {
      float f[8];
      uint32_t low = 0;
#pragma unroll
      for (int j = 0; j < 8; ++j) {
        const int c = c8 * 8 + j;
        f[j] = c < d_s ? xs[c] : 0.0f;
        low |= __float_as_uint(f[j]) & 0xffffu;
      }
      if (low) atomicOr(bad, 1);
      uint4 v;
      v.x = pack_bf16x2(f[0], f[1]);
      v.y = pack_bf16x2(f[2], f[3]);
      v.z = pack_bf16x2(f[4], f[5]);
      v.w = pack_bf16x2(f[6], f[7]);
      *reinterpret_cast<uint4*>(row + c8 * 8) = v;
    }
    const uint4* fs = reinterpret_cast<const uint4*>(F + (size_t)i * d_l);
    uint4* dst = reinterpret_cast<uint4*>(row + ds_pad);
    for (int c8 = lane; c8 < d_l / 8; c8 += 32) dst[c8] = __ldg(fs + c8);
    for (int c = ds_pad + d_l + lane * 8; c < ld; c += 256) *reinterpret_cast<uint4*>(row + c) = make_uint4(0, 0, 0, 0);
    if (lane == 0) y[p] = labels[s];
  }
}

// fp32 check mode (reading R23): the same layout with fp32 elements, one warp per row
__global__ void concat_f32_kernel(const float* __restrict__ X, int d_s, int ds_pad, const float* __restrict__ F,
                                  int d_l, const int32_t* __restrict__ pair_str, const int32_t* __restrict__ pair_img,
                                  const uint8_t* __restrict__ labels, int64_t n, int ld, float* __restrict__ MM,
                                  uint8_t* __restrict__ y) {
  const int lane = threadIdx.x & 31;
  const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
  for (int64_t p = blockIdx.x * (int64_t)(blockDim.x >> 5) + (threadIdx.x >> 5); p < n; p += warps) {
    const int32_t s = pair_str[p], i = pair_img[p];
    float* row = MM + (size_t)p * ld;
    for (int c = lane; c < ld; c += 32) {
      float v = 0.f;
      if (c < d_s) v = X[(size_t)s * d_s + c];
      else if (c >= ds_pad && c < ds_pad + d_l) v = F[(size_t)i * d_l + (c - ds_pad)];
      row[c] = v;
    }
    if (lane == 0) y[p] = labels[s];
  }
}

void launch_concat_f32(const float* X, int d_s, int ds_pad, const float* F, int d_l, const int32_t* pair_str,
                       const int32_t* pair_img, const uint8_t* labels, int64_t n_pairs, int ld, float* MM,
                       uint8_t* y, cudaStream_t st) {
  if (n_pairs <= 0) return;
  int64_t blocks = (n_pairs + 7) / 8;
  const int64_t cap = (int64_t)num_sms() * 8;
  if (blocks > cap) blocks = cap;
  prof_begin(st);
  concat_f32_kernel<<<(int)blocks, 256, 0, st>>>(X, d_s, ds_pad, F, d_l, pair_str, pair_img, labels, n_pairs, ld, MM,
                                                 y);
  LAUNCHED();
  prof_end(st, 4, 0, (double)n_pairs * (4.0 * d_s + 4.0 * d_l + 4.0 * ld + 9));
}

void launch_concat(const float* X, int d_s, int ds_pad, const bf16* F, int d_l, const int32_t* pair_str,
                   const int32_t* pair_img, const uint8_t* labels, int64_t n_pairs, int ld, bf16* MM, uint8_t* y,
                   int* bad, cudaStream_t st) {
  if (n_pairs <= 0) return;
  int64_t blocks = (n_pairs + 7) / 8;
  const int64_t cap = (int64_t)num_sms() * 8;
  if (blocks > cap) blocks = cap;
  prof_begin(st);
  concat_kernel<<<(int)blocks, 256, 0, st>>>(X, d_s, ds_pad, F, d_l, pair_str, pair_img, labels, n_pairs, ld, MM, y,
                                             bad);
  LAUNCHED();
  prof_end(st, 4, 0, (double)n_pairs * (4.0 * d_s + 2.0 * d_l + 2.0 * ld + 9));
}

}  // namespace vista
