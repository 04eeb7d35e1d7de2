"""Measure B200 HBM read-only / write-only / copy bandwidth with torch kernels (context for the roofline)."""
import torch
n = 4 << 30  # 8 GiB bf16
a = torch.empty(n, dtype=torch.bfloat16, device="cuda")
b = torch.empty(n, dtype=torch.bfloat16, device="cuda")
a.fill_(1.0)
def t(f, reps=5):
    f(); torch.cuda.synchronize()
    s, e = torch.cuda.Event(True), torch.cuda.Event(True)
    best = 1e9
    for _ in range(reps):
        s.record(); f(); e.record(); torch.cuda.synchronize(); best = min(best, s.elapsed_time(e))
    return best
bytes_ = n * 2
w = t(lambda: b.fill_(2.0)); print("write-only fill_ GB/s", bytes_ / w / 1e6)
r = t(lambda: a.sum()); print("read-only sum GB/s", bytes_ / r / 1e6)
c = t(lambda: b.copy_(a)); print("copy (r+w) GB/s", 2 * bytes_ / c / 1e6)
