"""Time single conv launch classes of the ResNet50 stage-1 micro-batch through vista_conv2d
(CUDA events around the kernel only: the layer object is built once, outside the timed loop)
and print TF/s, HBM GB/s (algorithmic bytes) per shape.  Run under ncu with -k regex:conv_tc
for a focused capture:  python tools/layer_probe.py [name ...]"""
import sys
import time

import torch

sys.path.insert(0, ".")
from paper_conf_sigmod_nakandalak20_b200 import vista as V  # noqa: E402

B = 1024
# name: (H, W, Cin, Cout, R, stride, pad, residual, N)
SHAPES = {
    "c4_res": (14, 14, 256, 1024, 1, 1, 0, True, B),
    "c2_res": (56, 56, 64, 256, 1, 1, 0, True, B),
    "c3_res": (28, 28, 128, 512, 1, 1, 0, True, B),
    "c5_res": (7, 7, 512, 2048, 1, 1, 0, True, B),
    "a2_3x3": (56, 56, 64, 64, 3, 1, 1, False, B),
    "a3_3x3": (28, 28, 128, 128, 3, 1, 1, False, B),
    "a4_3x3": (14, 14, 256, 256, 3, 1, 1, False, B),
    "r2_1x1": (56, 56, 256, 64, 1, 1, 0, False, B),
    "r4_1x1": (14, 14, 1024, 256, 1, 1, 0, False, B),
}


def main():
    names = sys.argv[1:] or list(SHAPES)
    reps = 20
    for nm in names:
        H, W, C, Co, R, s, p, res, N = SHAPES[nm]
        g = torch.Generator(device="cuda").manual_seed(0)
        x = (torch.randn((N, H, W, C), device="cuda", generator=g) * 0.5).to(torch.bfloat16)
        w = (torch.randn((Co, R, R, C), device="cuda", generator=g) / (R * R * C) ** 0.5).to(torch.bfloat16)
        sc = torch.ones(Co, device="cuda")
        sh = torch.zeros(Co, device="cuda")
        Ho = (H + 2 * p - R) // s + 1
        r = (torch.randn((N, Ho, Ho, Co), device="cuda", generator=g)).to(torch.bfloat16) if res else None
        y = torch.empty((N, Ho, Ho, Co), dtype=torch.bfloat16, device="cuda")
        st = torch.cuda.current_stream()
        for _ in range(3):
            V.vista_conv2d(x, w, sc, sh, stride=s, pad=p, residual=r, relu=True, y=y, stream=st.cuda_stream)
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        for _ in range(reps):
            V.vista_conv2d(x, w, sc, sh, stride=s, pad=p, residual=r, relu=True, y=y, stream=st.cuda_stream)
        torch.cuda.synchronize()
        wall = (time.perf_counter() - t0) / reps
        M = N * Ho * Ho
        fl = 2.0 * M * Co * R * R * C
        by = (N * H * W * C + M * Co * (2 if res else 1)) * 2 + Co * R * R * C * 2
        print(f"{nm:8s} wall/call {wall * 1e3:7.3f} ms  (incl. host layer build)  GFLOP {fl / 1e9:8.1f}  "
              f"MB {by / 1e6:8.1f}", flush=True)


if __name__ == "__main__":
    main()
