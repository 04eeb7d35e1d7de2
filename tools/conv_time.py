"""Device time (CUDA events) of one conv shape through vista_conv2d, repeated; prints TF/s.
usage: python tools/conv_time.py N H W C Cout k stride pad [reps] [residual 0/1]"""
import sys
sys.path.insert(0, ".")
import torch
from paper_conf_sigmod_nakandalak20_b200 import vista as V
N, H, W, C, Co, k, s, p = (int(a) for a in sys.argv[1:9])
reps = int(sys.argv[9]) if len(sys.argv) > 9 else 20
g = torch.Generator(device="cuda").manual_seed(0)
x = (torch.randn((N, H, W, C), device="cuda", generator=g) * 0.5).to(torch.bfloat16)
w = (torch.randn((Co, k, k, C), device="cuda", generator=g) / (k * k * C) ** 0.5).to(torch.bfloat16)
sc, sh = torch.ones(Co, device="cuda"), torch.zeros(Co, device="cuda")
Ho = (H + 2 * p - k) // s + 1
y = torch.empty((N, Ho, Ho, Co), dtype=torch.bfloat16, device="cuda")
res = torch.randn((N, Ho, Ho, Co), device="cuda", generator=g).to(torch.bfloat16) if len(sys.argv) > 10 and sys.argv[10] == "1" else None
st = torch.cuda.current_stream()

for _ in range(3):
    V.vista_conv2d(x, w, sc, sh, stride=s, pad=p, residual=res, relu=True, y=y, stream=st.cuda_stream)
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record(st)
for _ in range(reps):
    V.vista_conv2d(x, w, sc, sh, stride=s, pad=p, residual=res, relu=True, y=y, stream=st.cuda_stream)
e1.record(st)
torch.cuda.synchronize()
ms = e0.elapsed_time(e1) / reps
fl = 2.0 * N * Ho * Ho * Co * k * k * C
print(f"N{N} H{H} C{C}->{Co} k{k}: {ms:.3f} ms/call (incl. host setup between launches), {fl / ms / 1e9:.0f} TF/s")
