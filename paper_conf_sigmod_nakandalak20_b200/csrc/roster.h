// roster.h — the product's CNN roster (§3.2 "AlexNet [46], VGG16 [61], and
// ResNet50 [37]"; layer sets PAPER.md:365) as executable op lists per stage.
//
// Block / stage t maps the activation of tap t-1 (raw pixels for t = 0) to the full
// activation of tap t: partial CNN inference f^_{l(t-1) -> l(t)} (Def 3.7).
// The Staged plan (Fig 5E) runs the blocks in order, keeping A_t resident in HBM.
#pragma once
#include <cstdint>
#include <vector>

namespace vista {

enum OpKind { OP_INGEST = 0, OP_CONV = 1, OP_MAXPOOL = 2, OP_LRN = 3, OP_AVGPOOL = 4, OP_INGEST_S2D = 5 };

// ResNet50 conv1 (7x7 stride 2 pad 3 on 3 channels) runs as a 4x4 stride-1 conv on a 2x2
// space-to-depth input: [117, 117, 16] with channel c' = (dy*2 + dx)*3 + ch (12..15 zero) holding
// pixel (2*h2 + dy - 3, 2*w2 + dx - 3); the filter tap (r, s) = (2a + dy, 2b + dx), r, s < 7.
constexpr int kS2dHW = 117, kS2dC = 16;
enum BufId { BUF_IN = 0, BUF_OUT = 1, BUF_T0 = 2, NUM_BUFS = 7 };  // T0..T4 = scratch slots 2..6

struct LayerSpec {  // one parameterised layer (conv or fc); id = generator layer id
  int id;
  int Cin_real, Cin, Cout, R, S, stride, pad, groups;
  bool bias;      // conv/fc bias (AlexNet, VGG16, ResNet fc)
  int bn_kind;    // 0 none, 1 BN, 2 BN closing a residual branch / projection
  bool relu;      // ReLU in the epilogue
  bool s2d = false;  // executed on the space-to-depth input (see kS2dHW)
};

struct OpDesc {
  OpKind kind;
  int in, out, res;  // buffer ids (res = -1: none)
  int layer;         // index into NetDesc::layers for OP_CONV
  int k, s;          // pool window / stride
  int H, W, C;       // input shape per image
  int Ho, Wo, Co;    // output shape per image
};

struct StageDesc {
  std::vector<OpDesc> ops;
  int outH, outW, outC;             // A_t per image
  bool fc_tap;                      // tap is an FC layer (g = identity)
  int d_tap;                        // tap width
  int64_t in_elems, out_elems;      // per image (in: uint8 pixels for t = 0)
  int64_t slot_elems[NUM_BUFS];     // per-image elements each scratch slot must hold
  double macs;                      // MACs per image of this stage
};

struct NetDesc {
  int cnn;
  std::vector<LayerSpec> layers;
  std::vector<StageDesc> stages;
};

NetDesc build_roster(int cnn);

}  // namespace vista
