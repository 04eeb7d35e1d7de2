// roster.cpp — op lists of AlexNet / VGG16 / ResNet50 at 227x227, staged at
// the taps of PAPER.md:365 (readings R1-R6).  Convs carry their epilogue (bias or
// BN, ReLU, residual) so every conv is one tensor-core launch.
#include <algorithm>
#include <cstring>

#include "internal.h"
#include "roster.h"

namespace vista {

namespace {

struct Shape {
  int H = 0, W = 0, C = 0;
};

struct Builder {
  NetDesc net;
  StageDesc cur;
  Shape shp[NUM_BUFS];

  void begin_stage(Shape in, int64_t in_elems) {
    cur = StageDesc();
    cur.in_elems = in_elems;
    for (auto& s : shp) s = Shape();
    shp[BUF_IN] = in;
    std::fill(cur.slot_elems, cur.slot_elems + NUM_BUFS, 0);
    cur.macs = 0;
  }
  void set_out(int buf, Shape s) {
    shp[buf] = s;
    cur.slot_elems[buf] = std::max<int64_t>(cur.slot_elems[buf], (int64_t)s.H * s.W * s.C);
  }
  int layer(int Cin_real, int Cin, int Cout, int R, int S, int stride, int pad, int groups, bool bias, int bn,
            bool relu) {
    LayerSpec l{(int)net.layers.size(), Cin_real, Cin, Cout, R, S, stride, pad, groups, bias, bn, relu};
    net.layers.push_back(l);
    return l.id;
  }
  // conv (or fc when the input is flattened: R = S = 1 on a 1x1xK view)
  void conv(int in, int out, int res, int Cout, int R, int stride, int pad, int groups, bool bias, int bn, bool relu,
            int Cin_real = -1) {
    Shape s = shp[in];
    if (Cin_real < 0) Cin_real = s.C;
    const int id = layer(Cin_real, s.C, Cout, R, R, stride, pad, groups, bias, bn, relu);
    OpDesc op{OP_CONV, in, out, res, id, 0, 0, s.H, s.W, s.C, conv_out_dim(s.H, R, stride, pad),
              conv_out_dim(s.W, R, stride, pad), Cout};
    cur.macs += (double)op.Ho * op.Wo * Cout * R * R * (Cin_real / groups);
    cur.ops.push_back(op);
    set_out(out, Shape{op.Ho, op.Wo, Cout});
  }
  void fc(int in, int out, int Cout, bool relu) {
    Shape s = shp[in];
    const int K = s.H * s.W * s.C;  // NHWC flatten (reading R8)
    shp[in] = Shape{1, 1, K};
    conv(in, out, -1, Cout, 1, 1, 0, 1, true, 0, relu);
  }
  void pool(int in, int out, int k, int s) {
    Shape x = shp[in];
    OpDesc op{OP_MAXPOOL, in, out, -1, -1, k, s, x.H, x.W, x.C, (x.H - k) / s + 1, (x.W - k) / s + 1, x.C};
    cur.ops.push_back(op);
    set_out(out, Shape{op.Ho, op.Wo, x.C});
  }
  void lrn(int in, int out) {
    Shape x = shp[in];
    cur.ops.push_back(OpDesc{OP_LRN, in, out, -1, -1, 0, 0, x.H, x.W, x.C, x.H, x.W, x.C});
    set_out(out, x);
  }
  void avgpool(int in, int out) {
    Shape x = shp[in];
    cur.ops.push_back(OpDesc{OP_AVGPOOL, in, out, -1, -1, 0, 0, x.H, x.W, x.C, 1, 1, x.C});
    set_out(out, Shape{1, 1, x.C});
  }
  void ingest(int out) {  // uint8 NHWC3 -> bf16 NHWC8
    cur.ops.push_back(OpDesc{OP_INGEST, BUF_IN, out, -1, -1, 0, 0, 227, 227, 3, 227, 227, 8});
    set_out(out, Shape{227, 227, 8});
  }
  // ResNet conv1 = 7x7/2 pad 3 on the raw image, executed as 4x4/1 on the space-to-depth input
  void ingest_s2d_conv1(int tmp, int out, int Cout) {
    cur.ops.push_back(OpDesc{OP_INGEST_S2D, BUF_IN, tmp, -1, -1, 0, 0, 227, 227, 3, kS2dHW, kS2dHW, kS2dC});
    set_out(tmp, Shape{kS2dHW, kS2dHW, kS2dC});
    const int id = layer(3, 3, Cout, 7, 7, 2, 3, 1, false, 1, true);
    net.layers[id].s2d = true;
    const int Ho = conv_out_dim(227, 7, 2, 3);  // 114 = 117 - 4 + 1
    OpDesc op{OP_CONV, tmp, out, -1, id, 0, 0, kS2dHW, kS2dHW, kS2dC, Ho, Ho, Cout};
    cur.macs += (double)Ho * Ho * Cout * 7 * 7 * 3;
    cur.ops.push_back(op);
    set_out(out, Shape{Ho, Ho, Cout});
  }
  void end_stage() {
    Shape o = shp[BUF_OUT];
    cur.outH = o.H;
    cur.outW = o.W;
    cur.outC = o.C;
    cur.fc_tap = o.H == 1 && o.W == 1;
    cur.d_tap = cur.fc_tap ? o.C : 4 * o.C;
    cur.out_elems = (int64_t)o.H * o.W * o.C;
    cur.slot_elems[BUF_IN] = cur.slot_elems[BUF_OUT] = 0;
    net.stages.push_back(cur);
  }
  // ResNet bottleneck unit: a = ReLU(BN(1x1_s(x))); b = ReLU(BN(3x3(a))); [p = BN(1x1_s(x))];
  // out = ReLU(BN(1x1(b)) + (p or x)) — the add and ReLU fused into the c conv's epilogue.
  void resunit(int in, int out, int mid, int stride, bool proj, int ta, int tb, int tp) {
    const int cin = shp[in].C;
    conv(in, ta, -1, mid, 1, stride, 0, 1, false, 1, true);
    conv(ta, tb, -1, mid, 3, 1, 1, 1, false, 1, true);
    // generator layer order is a, b, c, proj (SURVEY.md/oracle numbering): create c before proj
    const int c_id = layer(mid, mid, 4 * mid, 1, 1, 1, 0, 1, false, 2, true);
    int res = in;
    if (proj) {
      Shape s = shp[in];
      const int p_id = layer(cin, cin, 4 * mid, 1, 1, stride, 0, 1, false, 2, false);
      OpDesc op{OP_CONV, in, tp, -1, p_id, 0, 0, s.H, s.W, s.C, conv_out_dim(s.H, 1, stride, 0),
                conv_out_dim(s.W, 1, stride, 0), 4 * mid};
      cur.macs += (double)op.Ho * op.Wo * op.Co * cin;
      cur.ops.push_back(op);
      set_out(tp, Shape{op.Ho, op.Wo, op.Co});
      res = tp;
    }
    Shape sb = shp[tb];
    OpDesc op{OP_CONV, tb, out, res, c_id, 0, 0, sb.H, sb.W, sb.C, sb.H, sb.W, 4 * mid};
    cur.macs += (double)sb.H * sb.W * 4 * mid * mid;
    cur.ops.push_back(op);
    set_out(out, Shape{sb.H, sb.W, 4 * mid});
  }
};

const int T0 = BUF_T0, T1 = BUF_T0 + 1, T2 = BUF_T0 + 2, T3 = BUF_T0 + 3, T4 = BUF_T0 + 4;

}  // namespace

NetDesc build_roster(int cnn) {
  Builder b;
  b.net.cnn = cnn;
  const Shape px{227, 227, 3};
  const int64_t px_elems = 227 * 227 * 3;
  if (cnn == 0) {  // AlexNet, grouped two-tower [46] (reading R2), LRN (R3)
    b.begin_stage(px, px_elems);
    b.ingest(T0);
    b.conv(T0, T1, -1, 96, 11, 4, 0, 1, true, 0, true, 3);
    b.lrn(T1, T2);
    b.pool(T2, T0, 3, 2);
    b.conv(T0, T1, -1, 256, 5, 1, 2, 2, true, 0, true);
    b.lrn(T1, T2);
    b.pool(T2, T0, 3, 2);
    b.conv(T0, T1, -1, 384, 3, 1, 1, 1, true, 0, true);
    b.conv(T1, T2, -1, 384, 3, 1, 1, 2, true, 0, true);
    b.conv(T2, BUF_OUT, -1, 256, 3, 1, 1, 2, true, 0, true);  // conv5
    b.end_stage();
    b.begin_stage(Shape{13, 13, 256}, 13 * 13 * 256);
    b.pool(BUF_IN, T0, 3, 2);
    b.fc(T0, BUF_OUT, 4096, true);  // fc6
    b.end_stage();
    b.begin_stage(Shape{1, 1, 4096}, 4096);
    b.fc(BUF_IN, BUF_OUT, 4096, true);  // fc7
    b.end_stage();
    b.begin_stage(Shape{1, 1, 4096}, 4096);
    b.fc(BUF_IN, BUF_OUT, 1000, false);  // fc8 logits (reading R6)
    b.end_stage();
  } else if (cnn == 1) {  // VGG16 configuration D [61]
    b.begin_stage(px, px_elems);
    b.ingest(T0);
    const int cfg[13] = {64, 64, 128, 128, 256, 256, 256, 512, 512, 512, 512, 512, 512};
    const int pool_after[13] = {0, 1, 0, 1, 0, 0, 1, 0, 0, 1, 0, 0, 1};
    int cur = T0;
    for (int i = 0; i < 13; ++i) {
      int nxt = cur == T0 ? T1 : T0;
      b.conv(cur, nxt, -1, cfg[i], 3, 1, 1, 1, true, 0, true, i == 0 ? 3 : -1);
      cur = nxt;
      if (pool_after[i]) {
        nxt = cur == T0 ? T1 : T0;
        b.pool(cur, nxt, 2, 2);
        cur = nxt;
      }
    }
    b.fc(cur, BUF_OUT, 4096, true);  // fc6
    b.end_stage();
    b.begin_stage(Shape{1, 1, 4096}, 4096);
    b.fc(BUF_IN, BUF_OUT, 4096, true);  // fc7
    b.end_stage();
    b.begin_stage(Shape{1, 1, 4096}, 4096);
    b.fc(BUF_IN, BUF_OUT, 1000, false);  // fc8
    b.end_stage();
  } else {  // ResNet50 v1 [37] (reading R4): pool1 unpadded, stride on the first 1x1
    b.begin_stage(px, px_elems);
    b.ingest_s2d_conv1(T0, T1, 64);
    b.pool(T1, T2, 3, 2);
    int cur = T2;
    const int mids[3] = {64, 128, 256}, units[3] = {3, 4, 6};
    for (int st = 0; st < 3; ++st)
      for (int u = 0; u < units[st]; ++u) {
        const bool last = st == 2 && u == units[st] - 1;
        const int out = last ? BUF_OUT : (cur == T2 ? T4 : T2);
        b.resunit(cur, out, mids[st], (u == 0 && st > 0) ? 2 : 1, u == 0, T0, T1, T3);
        cur = out;
      }
    b.end_stage();  // conv4_6
    for (int u = 0; u < 3; ++u) {  // conv5_1 .. conv5_3
      b.begin_stage(u == 0 ? Shape{14, 14, 1024} : Shape{7, 7, 2048}, u == 0 ? 14 * 14 * 1024 : 7 * 7 * 2048);
      b.resunit(BUF_IN, BUF_OUT, 512, u == 0 ? 2 : 1, u == 0, T0, T1, T3);
      b.end_stage();
    }
    b.begin_stage(Shape{7, 7, 2048}, 7 * 7 * 2048);
    b.avgpool(BUF_IN, T0);
    b.fc(T0, BUF_OUT, 1000, false);  // fc ("fc_6" of Fig 8)
    b.end_stage();
  }
  return b.net;
}

}  // namespace vista
