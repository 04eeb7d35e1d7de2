// oracle.cpp — plain fp64 CPU oracle for Vista's feature-transfer workload.
//
// TEST INFRASTRUCTURE ONLY (see oracle.h).  Shares no code with the CUDA path;
// only the seeded input generators of gen/ are common.
//
// What it computes is the *plain definition* the Staged plan must reproduce
// exactly: "All approaches ... yield identical downstream models" (PAPER.md:388
// §5.2).  For every image and tapped layer l: F_l = g_l(f^_l(x)) by a full
// forward pass (Eq. (2)), the key-key join (Eq. (3)), the
// concatenation X'_l = [X, F_l] (Eq. (4)), then M = elastic-net
// logistic regression trained on X'_l by the full-batch
// proximal-gradient reading of SURVEY.md §8c O6 / DESIGN.md reading R17.
#include "oracle.h"

#include <algorithm>
#include <atomic>
#include <cmath>
#include <cstring>
#include <map>
#include <memory>
#include <mutex>
#include <thread>
#include <unordered_map>
#include <unordered_set>
#include <vector>

extern "C" {
#include "../gen/vista_gen.h"
}

namespace {

// ------------------------------------------------------------------------
// MAC accounting for the roster pins (AlexNet fc7 721 MFLOPS,
// fc8 725 MFLOPS).  Set by the dry run of the architecture code below.
// ------------------------------------------------------------------------
struct Count {
  bool dry = false;
  double macs = 0, bias_adds = 0;
};
thread_local Count* g_count = nullptr;

inline int out_dim(int H, int k, int s, int p) { return (H + 2 * p - k) / s + 1; }

}  // namespace

// ===================== primitives (fp64, NHWC) =====================

// Convolution, Def 3.3/3.4 TensorOp; direct sum with zero
// padding: y[h,w,o] = b[o] + sum_{r,s,c in grp(o)} x[h*st-pad+r, w*st-pad+s, c] W[o,r,s,c].
extern "C" int or_conv2d(const double* x, int N, int H, int W, int C, const double* w, int Cout, int R,
                         int S, int stride, int pad, int groups, const double* bias, double* y) {
  if (groups < 1 || C % groups || Cout % groups || stride < 1) return OR_ERR_ARG;
  const int Ho = out_dim(H, R, stride, pad), Wo = out_dim(W, S, stride, pad);
  const int Cg = C / groups, Cog = Cout / groups;
  if (g_count) {
    g_count->macs += (double)N * Ho * Wo * Cout * R * S * Cg;
    if (bias) g_count->bias_adds += (double)N * Ho * Wo * Cout;
    if (g_count->dry) return OR_OK;
  }
  for (int n = 0; n < N; ++n)
    for (int ho = 0; ho < Ho; ++ho)
      for (int wo = 0; wo < Wo; ++wo)
        for (int o = 0; o < Cout; ++o) {
          const int g = o / Cog;
          double acc = bias ? bias[o] : 0.0;
          for (int r = 0; r < R; ++r) {
            const int hi = ho * stride - pad + r;
            if (hi < 0 || hi >= H) continue;
            for (int s = 0; s < S; ++s) {
              const int wi = wo * stride - pad + s;
              if (wi < 0 || wi >= W) continue;
              const double* xp = x + (((size_t)n * H + hi) * W + wi) * C + (size_t)g * Cg;
              const double* wp = w + (((size_t)o * R + r) * S + s) * Cg;
              for (int c = 0; c < Cg; ++c) acc += xp[c] * wp[c];
            }
          }
          y[(((size_t)n * Ho + ho) * Wo + wo) * Cout + o] = acc;
        }
  return OR_OK;
}

// Fully connected layer: y = W x + b (a perceptron layer).
extern "C" int or_fc(const double* x, int N, int K, const double* w, int Nout, const double* bias, double* y) {
  if (g_count) {
    g_count->macs += (double)N * K * Nout;
    if (bias) g_count->bias_adds += (double)N * Nout;
    if (g_count->dry) return OR_OK;
  }
  for (int n = 0; n < N; ++n)
    for (int o = 0; o < Nout; ++o) {
      double acc = bias ? bias[o] : 0.0;
      const double* xp = x + (size_t)n * K;
      const double* wp = w + (size_t)o * K;
      for (int k = 0; k < K; ++k) acc += xp[k] * wp[k];
      y[(size_t)n * Nout + o] = acc;
    }
  return OR_OK;
}

// Max pooling, unpadded, window k stride s ("pooling subsamples").
extern "C" int or_maxpool(const double* x, int N, int H, int W, int C, int k, int s, double* y) {
  const int Ho = out_dim(H, k, s, 0), Wo = out_dim(W, k, s, 0);
  if (g_count && g_count->dry) return OR_OK;
  for (int n = 0; n < N; ++n)
    for (int ho = 0; ho < Ho; ++ho)
      for (int wo = 0; wo < Wo; ++wo)
        for (int c = 0; c < C; ++c) {
          double m = -INFINITY;
          for (int r = 0; r < k; ++r)
            for (int q = 0; q < k; ++q) {
              const int hi = ho * s + r, wi = wo * s + q;
              if (hi < H && wi < W) m = std::max(m, x[(((size_t)n * H + hi) * W + wi) * C + c]);
            }
          y[(((size_t)n * Ho + ho) * Wo + wo) * C + c] = m;
        }
  return OR_OK;
}

// Global average pooling (ResNet50 [37] before fc): y[c] = (1/HW) sum_hw x[h,w,c].
extern "C" int or_avgpool_global(const double* x, int N, int H, int W, int C, double* y) {
  if (g_count && g_count->dry) return OR_OK;
  for (int n = 0; n < N; ++n)
    for (int c = 0; c < C; ++c) {
      double acc = 0;
      for (int i = 0; i < H * W; ++i) acc += x[((size_t)n * H * W + i) * C + c];
      y[(size_t)n * C + c] = acc / (double)(H * W);
    }
  return OR_OK;
}

// Local response normalisation of AlexNet [46] (reading R3, Caffe/bvlc
// constants): y_c = x_c / (1 + (alpha/n) sum_{c'=c-2..c+2} x_c'^2)^beta,
// alpha/n = 2e-5 (alpha 1e-4, n 5), beta 0.75, k 1.
extern "C" int or_lrn(const double* x, int N, int H, int W, int C, double* y) {
  if (g_count && g_count->dry) return OR_OK;
  for (int64_t p = 0; p < (int64_t)N * H * W; ++p) {
    const double* xp = x + (size_t)p * C;
    double* yp = y + (size_t)p * C;
    for (int c = 0; c < C; ++c) {
      double ss = 0;
      for (int d = std::max(0, c - 2); d <= std::min(C - 1, c + 2); ++d) ss += xp[d] * xp[d];
      yp[c] = xp[c] / std::pow(1.0 + 2e-5 * ss, 0.75);
    }
  }
  return OR_OK;
}

// Batch normalisation in inference form (ResNet50 [37]; reading R12):
// y = gamma (x - mu) / sqrt(var + eps) + beta, per channel (last dim).
extern "C" int or_batchnorm(const double* x, int64_t count, int C, const double* gamma, const double* beta,
                            const double* mean, const double* var, double eps, double* y) {
  if (g_count && g_count->dry) return OR_OK;
  for (int64_t p = 0; p < count; ++p)
    for (int c = 0; c < C; ++c) {
      const size_t i = (size_t)p * C + c;
      y[i] = gamma[c] * (x[i] - mean[c]) / std::sqrt(var[c] + eps) + beta[c];
    }
  return OR_OK;
}

// Tap g_l (Def 3.5, with the pooling of footnote 4, PAPER.md:369:
// "Filter width and stride for max pooling are set to reduce the feature tensor
// to a 2 x 2 grid of the same depth"), reading R7: R_0 = [0, ceil(H/2)),
// R_1 = [ceil(H/2), H), likewise W; flatten NHWC: F[(2i+j)C + c] = max A[h,w,c].
extern "C" int or_tap(const double* A, int N, int H, int W, int C, double* F) {
  const int h2 = (H + 1) / 2, w2 = (W + 1) / 2;
  for (int n = 0; n < N; ++n)
    for (int i = 0; i < 2; ++i)
      for (int j = 0; j < 2; ++j)
        for (int c = 0; c < C; ++c) {
          double m = -INFINITY;
          for (int h = i ? h2 : 0; h < (i ? H : h2); ++h)
            for (int w = j ? w2 : 0; w < (j ? W : w2); ++w)
              m = std::max(m, A[(((size_t)n * H + h) * W + w) * C + c]);
          F[(size_t)n * 4 * C + (2 * i + j) * C + c] = m;
        }
  return OR_OK;
}

// ===================== CNN roster =====================
namespace {

struct Act {
  int H = 0, W = 0, C = 0;
  std::vector<double> v;
  size_t size() const { return (size_t)H * W * C; }
};

struct Layer {  // one parameterised layer (conv or fc) with its bias / BN
  int Cout = 0, R = 1, S = 1, Cin = 0, groups = 1, stride = 1, pad = 0;
  std::vector<double> w, bias, gamma, beta, mean, var;
};

struct Net {
  int cnn = 0;
  std::vector<Layer> L;
  int n_taps = 0;
};

// Parameter recipe (reading R11): He-normal N(0, 2/fan_in) weights,
// RNE-rounded to bf16; AlexNet/VGG biases N(0, 0.01^2) -> bf16; ResNet BN
// gamma N(1, 0.1^2) (last BN of a branch and projection BN: N(0.2, 0.02^2)),
// beta N(0, 0.05^2), mean N(0, 0.05^2), var 1 + 0.2 U[0,1); fc bias N(0, 0.01^2).
Layer make_layer(uint64_t seed, int cnn, int id, int Cout, int R, int S, int Cin, int groups, int stride,
                 int pad, bool has_bias, int bn_kind /*0 none, 1 normal, 2 branch-last*/) {
  Layer l;
  l.Cout = Cout; l.R = R; l.S = S; l.Cin = Cin; l.groups = groups; l.stride = stride; l.pad = pad;
  const int64_t fan_in = (int64_t)R * S * (Cin / groups);
  const int64_t nw = (int64_t)Cout * fan_in;
  l.w.resize(nw);
  vg_param(seed, cnn, id, VG_T_WEIGHT, nw, 0, 0.0, std::sqrt(2.0 / (double)fan_in), 1, l.w.data());
  if (has_bias) {
    l.bias.resize(Cout);
    vg_param(seed, cnn, id, VG_T_BIAS, Cout, 0, 0.0, 0.01, 1, l.bias.data());
  }
  if (bn_kind) {
    l.gamma.resize(Cout); l.beta.resize(Cout); l.mean.resize(Cout); l.var.resize(Cout);
    if (bn_kind == 2)
      vg_param(seed, cnn, id, VG_T_BN_GAMMA, Cout, 0, 0.2, 0.02, 0, l.gamma.data());
    else
      vg_param(seed, cnn, id, VG_T_BN_GAMMA, Cout, 0, 1.0, 0.1, 0, l.gamma.data());
    vg_param(seed, cnn, id, VG_T_BN_BETA, Cout, 0, 0.0, 0.05, 0, l.beta.data());
    vg_param(seed, cnn, id, VG_T_BN_MEAN, Cout, 0, 0.0, 0.05, 0, l.mean.data());
    vg_param(seed, cnn, id, VG_T_BN_VAR, Cout, 1, 1.0, 0.2, 0, l.var.data());
  }
  return l;
}

// Architectures of SURVEY.md §8c c.1 (readings R1-R6).  When `seed_ok`
// is false only the shapes are built (dry run for MAC counts).
Net build_net(int cnn, uint64_t seed, bool with_weights) {
  Net net;
  net.cnn = cnn;
  auto add = [&](int Cout, int R, int S, int Cin, int groups, int stride, int pad, bool bias, int bn) {
    const int id = (int)net.L.size();
    if (with_weights) {
      net.L.push_back(make_layer(seed, cnn, id, Cout, R, S, Cin, groups, stride, pad, bias, bn));
    } else {
      Layer l;
      l.Cout = Cout; l.R = R; l.S = S; l.Cin = Cin; l.groups = groups; l.stride = stride; l.pad = pad;
      if (bias) l.bias.assign(Cout, 0.0);
      net.L.push_back(l);
    }
  };
  if (cnn == OR_ALEXNET) {  // grouped two-tower AlexNet [46] at 227 (reading R2)
    add(96, 11, 11, 3, 1, 4, 0, true, 0);      // 0 conv1
    add(256, 5, 5, 96, 2, 1, 2, true, 0);      // 1 conv2
    add(384, 3, 3, 256, 1, 1, 1, true, 0);     // 2 conv3
    add(384, 3, 3, 384, 2, 1, 1, true, 0);     // 3 conv4
    add(256, 3, 3, 384, 2, 1, 1, true, 0);     // 4 conv5
    add(4096, 1, 1, 9216, 1, 1, 0, true, 0);   // 5 fc6
    add(4096, 1, 1, 4096, 1, 1, 0, true, 0);   // 6 fc7
    add(1000, 1, 1, 4096, 1, 1, 0, true, 0);   // 7 fc8
    net.n_taps = 4;
  } else if (cnn == OR_VGG16) {  // configuration D of [61] at 227
    const int cfg[13] = {64, 64, 128, 128, 256, 256, 256, 512, 512, 512, 512, 512, 512};
    int cin = 3;
    for (int i = 0; i < 13; ++i) {
      add(cfg[i], 3, 3, cin, 1, 1, 1, true, 0);
      cin = cfg[i];
    }
    add(4096, 1, 1, 25088, 1, 1, 0, true, 0);  // 13 fc6
    add(4096, 1, 1, 4096, 1, 1, 0, true, 0);   // 14 fc7
    add(1000, 1, 1, 4096, 1, 1, 0, true, 0);   // 15 fc8
    net.n_taps = 3;
  } else if (cnn == OR_RESNET50) {  // ResNet50 v1 [37] at 227 (reading R4)
    add(64, 7, 7, 3, 1, 2, 3, false, 1);  // 0 conv1
    const int mids[4] = {64, 128, 256, 512}, units[4] = {3, 4, 6, 3};
    int cin = 64;
    for (int st = 0; st < 4; ++st) {
      const int mid = mids[st], out = 4 * mid;
      for (int u = 0; u < units[st]; ++u) {
        const int stride = (u == 0 && st > 0) ? 2 : 1;
        add(mid, 1, 1, cin, 1, stride, 0, false, 1);  // a
        add(mid, 3, 3, mid, 1, 1, 1, false, 1);       // b
        add(out, 1, 1, mid, 1, 1, 0, false, 2);       // c
        if (u == 0) add(out, 1, 1, cin, 1, stride, 0, false, 2);  // projection
        cin = out;
      }
    }
    add(1000, 1, 1, 2048, 1, 1, 0, true, 0);  // 53 fc
    net.n_taps = 5;
  }
  return net;
}

// --- per-image layer applications (N = 1) ---
Act conv(const Act& x, const Layer& l) {
  Act y;
  y.H = out_dim(x.H, l.R, l.stride, l.pad);
  y.W = out_dim(x.W, l.S, l.stride, l.pad);
  y.C = l.Cout;
  y.v.resize(y.size());
  or_conv2d(x.v.data(), 1, x.H, x.W, x.C, l.w.data(), l.Cout, l.R, l.S, l.stride, l.pad, l.groups,
            l.bias.empty() ? nullptr : l.bias.data(), y.v.data());
  return y;
}
Act fc(const Act& x, const Layer& l) {  // flatten NHWC (reading R8) then W x + b
  Act y;
  y.H = 1; y.W = 1; y.C = l.Cout;
  y.v.resize(l.Cout);
  or_fc(x.v.data(), 1, (int)x.size(), l.w.data(), l.Cout, l.bias.empty() ? nullptr : l.bias.data(), y.v.data());
  return y;
}
void bn(Act& x, const Layer& l) {
  or_batchnorm(x.v.data(), (int64_t)x.H * x.W, x.C, l.gamma.data(), l.beta.data(), l.mean.data(), l.var.data(),
               1e-5, x.v.data());
}
void relu(Act& x) {
  if (g_count && g_count->dry) return;
  for (double& e : x.v) e = e > 0 ? e : 0;
}
Act lrn(const Act& x) {
  Act y = x;
  or_lrn(x.v.data(), 1, x.H, x.W, x.C, y.v.data());
  return y;
}
Act maxpool(const Act& x, int k, int s) {
  Act y;
  y.H = out_dim(x.H, k, s, 0); y.W = out_dim(x.W, k, s, 0); y.C = x.C;
  y.v.resize(y.size());
  or_maxpool(x.v.data(), 1, x.H, x.W, x.C, k, s, y.v.data());
  return y;
}
Act avgpool(const Act& x) {
  Act y;
  y.H = 1; y.W = 1; y.C = x.C;
  y.v.resize(x.C);
  or_avgpool_global(x.v.data(), 1, x.H, x.W, x.C, y.v.data());
  return y;
}

// ResNet bottleneck unit: a = ReLU(BN(1x1_s(x))); b = ReLU(BN(3x3(a)));
// c = BN(1x1(b)); sc = BN(1x1_s(x)) on unit 1 else x; out = ReLU(c + sc).
Act resunit(const Act& x, const Net& net, int id, bool proj) {
  Act a = conv(x, net.L[id]); bn(a, net.L[id]); relu(a);
  Act b = conv(a, net.L[id + 1]); bn(b, net.L[id + 1]); relu(b);
  Act c = conv(b, net.L[id + 2]); bn(c, net.L[id + 2]);
  if (proj) {
    Act p = conv(x, net.L[id + 3]); bn(p, net.L[id + 3]);
    if (!(g_count && g_count->dry))
      for (size_t i = 0; i < c.v.size(); ++i) c.v[i] += p.v[i];
  } else if (!(g_count && g_count->dry)) {
    for (size_t i = 0; i < c.v.size(); ++i) c.v[i] += x.v[i];
  }
  relu(c);
  return c;
}

// Block t maps the activation of tap t-1 (pixels for t = 0) to the activation of
// tap t.  Staged execution (Fig 5E) chains these blocks; the
// oracle uses the same chain for eager and lazy, so staged == eager == lazy.
Act run_block(const Net& net, int t, const Act& x) {
  if (net.cnn == OR_ALEXNET) {
    if (t == 0) {
      Act y = conv(x, net.L[0]); relu(y); y = lrn(y); y = maxpool(y, 3, 2);
      y = conv(y, net.L[1]); relu(y); y = lrn(y); y = maxpool(y, 3, 2);
      y = conv(y, net.L[2]); relu(y);
      y = conv(y, net.L[3]); relu(y);
      y = conv(y, net.L[4]); relu(y);
      return y;  // conv5 13x13x256
    }
    if (t == 1) { Act y = maxpool(x, 3, 2); y = fc(y, net.L[5]); relu(y); return y; }
    if (t == 2) { Act y = fc(x, net.L[6]); relu(y); return y; }
    return fc(x, net.L[7]);  // fc8 logits (reading R6)
  }
  if (net.cnn == OR_VGG16) {
    if (t == 0) {
      const int pool_after[13] = {0, 1, 0, 1, 0, 0, 1, 0, 0, 1, 0, 0, 1};
      Act y = x;
      for (int i = 0; i < 13; ++i) {
        y = conv(y, net.L[i]); relu(y);
        if (pool_after[i]) y = maxpool(y, 2, 2);
      }
      y = fc(y, net.L[13]); relu(y);
      return y;  // fc6
    }
    if (t == 1) { Act y = fc(x, net.L[14]); relu(y); return y; }
    return fc(x, net.L[15]);
  }
  // ResNet50
  if (t == 0) {
    Act y = conv(x, net.L[0]); bn(y, net.L[0]); relu(y); y = maxpool(y, 3, 2);
    int id = 1;
    const int units[3] = {3, 4, 6};
    for (int st = 0; st < 3; ++st)
      for (int u = 0; u < units[st]; ++u) {
        y = resunit(y, net, id, u == 0);
        id += (u == 0) ? 4 : 3;
      }
    return y;  // conv4_6: 14x14x1024
  }
  if (t >= 1 && t <= 3) {
    const int id = 1 + (3 * 3 + 1) + (4 * 3 + 1) + (6 * 3 + 1) + (t == 1 ? 0 : 4 + 3 * (t - 2));
    return resunit(x, net, id, t == 1);  // conv5_t: 7x7x2048
  }
  Act y = avgpool(x);
  return fc(y, net.L[53]);  // fc (Fig 8 "fc_6", 1000-d per Table 2)
}

Act preprocess(const uint8_t* px) {  // reading R10: x = (p - 128) / 128
  Act x;
  x.H = VG_IMG_H; x.W = VG_IMG_W; x.C = 3;
  x.v.resize(x.size());
  for (size_t i = 0; i < x.size(); ++i) x.v[i] = ((double)px[i] - 128.0) / 128.0;
  return x;
}

void tap_features(const Act& a, double* F) {  // g_t; FC taps are the identity
  if (a.H == 1 && a.W == 1) {
    std::memcpy(F, a.v.data(), a.size() * sizeof(double));
  } else {
    or_tap(a.v.data(), 1, a.H, a.W, a.C, F);
  }
}

std::mutex g_net_mu;
std::map<std::pair<int, uint64_t>, std::shared_ptr<Net>> g_nets;

std::shared_ptr<Net> get_net(int cnn, uint64_t seed) {
  std::lock_guard<std::mutex> lk(g_net_mu);
  auto key = std::make_pair(cnn, seed);
  auto it = g_nets.find(key);
  if (it != g_nets.end()) return it->second;
  auto p = std::make_shared<Net>(build_net(cnn, seed, true));
  g_nets[key] = p;
  return p;
}

struct TapShape {
  int H, W, C, d;
  double macs, macs_bias;
};

std::vector<TapShape> dry_shapes(int cnn) {
  Net net = build_net(cnn, 0, false);
  Count cnt;
  cnt.dry = true;
  g_count = &cnt;
  std::vector<TapShape> out;
  Act x;
  x.H = VG_IMG_H; x.W = VG_IMG_W; x.C = 3;
  for (int t = 0; t < net.n_taps; ++t) {
    x = run_block(net, t, x);
    const bool is_fc = x.H == 1 && x.W == 1;
    out.push_back({x.H, x.W, x.C, is_fc ? x.C : 4 * x.C, cnt.macs, cnt.macs + cnt.bias_adds});
  }
  g_count = nullptr;
  return out;
}

int resolve_threads(int nthreads, int64_t n) {
  int nt = nthreads > 0 ? nthreads : (int)std::thread::hardware_concurrency();
  if (nt < 1) nt = 1;
  if ((int64_t)nt > n) nt = (int)std::max<int64_t>(n, 1);
  return nt;
}

int run_images(int cnn, uint64_t seed, int t0, const uint8_t* images, const double* A_in, int64_t n,
               double** F, double** A, int nthreads) {
  if (cnn < 0 || cnn > 2) return OR_ERR_ARG;
  auto net = get_net(cnn, seed);
  auto shapes = dry_shapes(cnn);
  const int T = net->n_taps;
  if (t0 < -1 || t0 >= T) return OR_ERR_ARG;
  int last = -1;
  for (int t = t0 + 1; t < T; ++t)
    if ((F && F[t]) || (A && A[t])) last = t;
  std::atomic<int64_t> next(0);
  auto worker = [&]() {
    for (;;) {
      const int64_t i = next.fetch_add(1);
      if (i >= n) break;
      Act x;
      if (t0 < 0) {
        x = preprocess(images + (size_t)i * VG_IMG_BYTES);
      } else {
        const TapShape& s = shapes[t0];
        x.H = s.H; x.W = s.W; x.C = s.C;
        x.v.assign(A_in + (size_t)i * x.size(), A_in + (size_t)(i + 1) * x.size());
      }
      for (int t = t0 + 1; t <= last; ++t) {
        x = run_block(*net, t, x);
        if (F && F[t]) tap_features(x, F[t] + (size_t)i * shapes[t].d);
        if (A && A[t]) std::memcpy(A[t] + (size_t)i * x.size(), x.v.data(), x.size() * sizeof(double));
      }
    }
  };
  const int nt = resolve_threads(nthreads, n);
  std::vector<std::thread> th;
  for (int k = 1; k < nt; ++k) th.emplace_back(worker);
  worker();
  for (auto& t : th) t.join();
  return OR_OK;
}

}  // namespace

extern "C" int oracle_cnn_info(int cnn, int tap, int64_t* out) {
  if (cnn < 0 || cnn > 2) return OR_ERR_ARG;
  auto s = dry_shapes(cnn);
  if (tap < 0 || tap >= (int)s.size()) return OR_ERR_ARG;
  out[0] = s[tap].H; out[1] = s[tap].W; out[2] = s[tap].C; out[3] = s[tap].d;
  out[4] = (int64_t)std::llround(s[tap].macs);
  out[5] = (int64_t)std::llround(s[tap].macs_bias);
  out[6] = (int64_t)s.size();
  out[7] = (int64_t)s[tap].H * s[tap].W * s[tap].C;
  return OR_OK;
}

extern "C" int oracle_features(int cnn, uint64_t weight_seed, const uint8_t* images, int64_t n, double** F,
                               double** A, int nthreads) {
  return run_images(cnn, weight_seed, -1, images, nullptr, n, F, A, nthreads);
}

extern "C" int oracle_features_from(int cnn, uint64_t weight_seed, int t0, const double* A_in, int64_t n,
                                    double** F, double** A, int nthreads) {
  if (t0 < 0) return OR_ERR_ARG;
  return run_images(cnn, weight_seed, t0, nullptr, A_in, n, F, A, nthreads);
}

// ===================== Eq. (3) join, Eq. (4) concat =====================

// T'_l = T_str |><|_ID T'_img,l: inner key-key equi-join, ID a primary key on
// both sides, built as the broadcast join's local hash table
// (PAPER.md:279).  Output in T_str row order (reading R14); the 80/20 split of
// PAPER.md:389 is a hash of the key (reading R16).
extern "C" int oracle_join(const int64_t* img_keys, int64_t n_img, const int64_t* str_keys, int64_t n_str,
                           uint64_t split_seed, int64_t* pair_str, int64_t* pair_img, uint8_t* is_test,
                           int64_t* n_pairs) {
  std::unordered_map<int64_t, int64_t> table;
  table.reserve((size_t)n_img * 2);
  for (int64_t i = 0; i < n_img; ++i)
    if (!table.emplace(img_keys[i], i).second) return OR_ERR_DUP_KEY;
  std::unordered_set<int64_t> seen;
  seen.reserve((size_t)n_str * 2);
  const uint64_t ss = vg_subseed(split_seed, VG_S_SPLIT);
  int64_t p = 0;
  for (int64_t s = 0; s < n_str; ++s) {
    if (!seen.insert(str_keys[s]).second) return OR_ERR_DUP_KEY;
    auto it = table.find(str_keys[s]);
    if (it == table.end()) continue;
    pair_str[p] = s;
    pair_img[p] = it->second;
    is_test[p] = (vg_mix64((uint64_t)str_keys[s] ^ ss) % 5u) == 0 ? 1 : 0;
    ++p;
  }
  *n_pairs = p;
  return OR_OK;
}

// X'_l = [X, g_l(f^_l(I))] (Eq. (4)): structured first, then the tap.
extern "C" int oracle_concat(const float* X, int d_s, const double* F, int d_l, const int64_t* pair_str,
                             const int64_t* pair_img, int64_t n_pairs, double* MM) {
  const int d = d_s + d_l;
  for (int64_t p = 0; p < n_pairs; ++p) {
    for (int j = 0; j < d_s; ++j) MM[(size_t)p * d + j] = (double)X[(size_t)pair_str[p] * d_s + j];
    for (int j = 0; j < d_l; ++j) MM[(size_t)p * d + d_s + j] = F[(size_t)pair_img[p] * d_l + j];
  }
  return OR_OK;
}

// ===================== M: elastic-net logistic regression (O6) =====================
namespace {

double softplus(double z) { return z > 0 ? z + std::log1p(std::exp(-z)) : std::log1p(std::exp(z)); }
double sigmoid(double z) { return z >= 0 ? 1.0 / (1.0 + std::exp(-z)) : std::exp(z) / (1.0 + std::exp(z)); }

}  // namespace

// O6 step 2: mu_j = mean over train rows, sigma_j = population std (two-pass),
// keep_j = sigma_j > 1e-12, inv_j = keep_j ? 1/sigma_j : 0.
extern "C" int oracle_lr_stats(const double* MM, int64_t n, int d, const uint8_t* is_test, double* mu,
                               double* sigma, double* inv) {
  int64_t nt = 0;
  std::vector<double> s(d, 0.0), q(d, 0.0);
  for (int64_t p = 0; p < n; ++p) {
    if (is_test && is_test[p]) continue;
    ++nt;
    for (int j = 0; j < d; ++j) s[j] += MM[(size_t)p * d + j];
  }
  if (nt == 0) return OR_ERR_ARG;
  for (int j = 0; j < d; ++j) mu[j] = s[j] / (double)nt;
  for (int64_t p = 0; p < n; ++p) {
    if (is_test && is_test[p]) continue;
    for (int j = 0; j < d; ++j) {
      const double e = MM[(size_t)p * d + j] - mu[j];
      q[j] += e * e;
    }
  }
  for (int j = 0; j < d; ++j) {
    sigma[j] = std::sqrt(q[j] / (double)nt);
    inv[j] = sigma[j] > 1e-12 ? 1.0 / sigma[j] : 0.0;
  }
  return OR_OK;
}

// f(w, b) = (1/n) sum_p [log(1 + e^{z_p}) - y_p z_p] + (lambda (1 - alpha) / 2) ||w||^2,
// z_p = b + sum_j w_j x~_pj; the smooth part whose gradient O6 step 5 uses.
extern "C" int oracle_lr_objective(const double* MM, int64_t n, int d, const uint8_t* y, const uint8_t* is_test,
                                   const double* mu, const double* inv, const double* w, double b, double lambda,
                                   double alpha, double* f_out, double* grad_w, double* grad_b) {
  int64_t nt = 0;
  double f = 0, gb = 0;
  std::vector<double> g(d, 0.0);
  for (int64_t p = 0; p < n; ++p) {
    if (is_test && is_test[p]) continue;
    ++nt;
    double z = b;
    for (int j = 0; j < d; ++j) z += w[j] * (MM[(size_t)p * d + j] - mu[j]) * inv[j];
    const double r = sigmoid(z) - (double)y[p];
    f += softplus(z) - (double)y[p] * z;
    for (int j = 0; j < d; ++j) g[j] += r * (MM[(size_t)p * d + j] - mu[j]) * inv[j];
    gb += r;
  }
  if (nt == 0) return OR_ERR_ARG;
  double w2 = 0;
  for (int j = 0; j < d; ++j) w2 += w[j] * w[j];
  *f_out = f / (double)nt + 0.5 * lambda * (1.0 - alpha) * w2;
  for (int j = 0; j < d; ++j) grad_w[j] = g[j] / (double)nt + lambda * (1.0 - alpha) * w[j];
  *grad_b = gb / (double)nt;
  return OR_OK;
}

// O6 step 3: K power iterations on (1/n)[X~, 1]^T [X~, 1] from v0 = 1/sqrt(d+1):
// u = X~ v_{1:d} + v_{d+1}; q = (1/n)[X~^T u; sum u]; lambda = ||q||; v = q / lambda.
extern "C" int oracle_lr_power(const double* MM, int64_t n, int d, const uint8_t* is_test, const double* mu,
                               const double* inv, int K, double* lambda_out) {
  int64_t nt = 0;
  for (int64_t p = 0; p < n; ++p)
    if (!(is_test && is_test[p])) ++nt;
  if (nt == 0) return OR_ERR_ARG;
  std::vector<double> v(d + 1, 1.0 / std::sqrt((double)(d + 1))), q(d + 1);
  double lam = 0;
  for (int k = 0; k < K; ++k) {
    std::fill(q.begin(), q.end(), 0.0);
    for (int64_t p = 0; p < n; ++p) {
      if (is_test && is_test[p]) continue;
      double u = v[d];
      for (int j = 0; j < d; ++j) u += (MM[(size_t)p * d + j] - mu[j]) * inv[j] * v[j];
      for (int j = 0; j < d; ++j) q[j] += u * (MM[(size_t)p * d + j] - mu[j]) * inv[j];
      q[d] += u;
    }
    double nrm = 0;
    for (int j = 0; j <= d; ++j) {
      q[j] /= (double)nt;
      nrm += q[j] * q[j];
    }
    lam = std::sqrt(nrm);
    if (lam == 0) break;
    for (int j = 0; j <= d; ++j) v[j] = q[j] / lam;
  }
  *lambda_out = lam;
  return OR_OK;
}

extern "C" int oracle_lr_grad_sums(const double* MM, int64_t n, int d, const uint8_t* y, const uint8_t* is_test,
                                   const double* w_hat, double b_hat, double* out) {
  std::fill(out, out + d + 2, 0.0);
  for (int64_t p = 0; p < n; ++p) {
    if (is_test && is_test[p]) continue;
    double z = b_hat;
    for (int j = 0; j < d; ++j) z += w_hat[j] * MM[(size_t)p * d + j];
    const double r = sigmoid(z) - (double)y[p];
    for (int j = 0; j < d; ++j) out[j] += r * MM[(size_t)p * d + j];
    out[d] += r;
    out[d + 1] += softplus(z) - (double)y[p] * z;
  }
  return OR_OK;
}

// O6 in full: stats -> step size 1/L with L = 0.25 * 1.05 * lambda_hat + lambda (1 - alpha)
// -> T proximal-gradient (ISTA) steps from w = 0, b = 0 (bias unregularised) -> eval
// (predict 1 iff z >= 0; accuracy and F1, the paper's metric).
extern "C" int oracle_lr_train(const double* MM, int64_t n, int d, const uint8_t* y, const uint8_t* is_test,
                               const oracle_lr_cfg* cfg, double* w_out, double* b_out, double* loss_out,
                               double* lambda_hat_out, double* metrics_out) {
  std::vector<double> mu(d), sigma(d), inv(d);
  int rc = oracle_lr_stats(MM, n, d, is_test, mu.data(), sigma.data(), inv.data());
  if (rc) return rc;
  double lam_hat = 0;
  oracle_lr_power(MM, n, d, is_test, mu.data(), inv.data(), cfg->power_iters, &lam_hat);
  const double L = 0.25 * 1.05 * lam_hat + cfg->lambda * (1.0 - cfg->alpha);
  const double eta = 1.0 / L;
  std::vector<double> w(d, 0.0), g(d);
  double b = 0;
  for (int t = 0; t < cfg->iters; ++t) {
    double f, gb;
    oracle_lr_objective(MM, n, d, y, is_test, mu.data(), inv.data(), w.data(), b, cfg->lambda, cfg->alpha, &f,
                        g.data(), &gb);
    double w2 = 0;
    for (int j = 0; j < d; ++j) w2 += w[j] * w[j];
    loss_out[t] = f - 0.5 * cfg->lambda * (1.0 - cfg->alpha) * w2;  // logistic part only
    const double thr = eta * cfg->lambda * cfg->alpha;
    for (int j = 0; j < d; ++j) {
      const double v = w[j] - eta * g[j];
      w[j] = (v > 0 ? 1.0 : (v < 0 ? -1.0 : 0.0)) * std::max(std::fabs(v) - thr, 0.0);
    }
    b -= eta * gb;
  }
  int64_t tp = 0, fp = 0, tn = 0, fn = 0, tr_ok = 0, n_tr = 0, n_te = 0;
  for (int64_t p = 0; p < n; ++p) {
    double z = b;
    for (int j = 0; j < d; ++j) z += w[j] * (MM[(size_t)p * d + j] - mu[j]) * inv[j];
    const int pred = z >= 0 ? 1 : 0;
    if (is_test && is_test[p]) {
      ++n_te;
      if (pred && y[p]) ++tp;
      else if (pred && !y[p]) ++fp;
      else if (!pred && !y[p]) ++tn;
      else ++fn;
    } else {
      ++n_tr;
      tr_ok += pred == y[p];
    }
  }
  for (int j = 0; j < d; ++j) w_out[j] = w[j];
  *b_out = b;
  *lambda_hat_out = lam_hat;
  metrics_out[0] = n_tr ? 100.0 * (double)tr_ok / (double)n_tr : 0.0;
  metrics_out[1] = n_te ? 100.0 * (double)(tp + tn) / (double)n_te : 0.0;
  metrics_out[2] = (2 * tp + fp + fn) ? 100.0 * 2.0 * (double)tp / (double)(2 * tp + fp + fn) : 0.0;
  metrics_out[3] = (double)n_tr;
  metrics_out[4] = (double)n_te;
  metrics_out[5] = (double)tp;
  metrics_out[6] = (double)fp;
  metrics_out[7] = (double)tn;
  metrics_out[8] = (double)fn;
  metrics_out[9] = eta;
  return OR_OK;
}
