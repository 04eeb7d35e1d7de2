import sys
import numpy as np
import torch
sys.path.insert(0, ".")
from paper_conf_sigmod_nakandalak20_b200 import vista_conv2d
rng = np.random.default_rng(0)
N = int(sys.argv[1]) if len(sys.argv) > 1 else 24
x = torch.from_numpy(rng.standard_normal((N, 28, 28, 128)).astype(np.float32)).to(torch.bfloat16).cuda()
w = torch.from_numpy((rng.standard_normal((128, 3, 3, 128)) * 0.04).astype(np.float32)).to(torch.bfloat16).cuda()
sc = torch.ones(128).cuda()
sh = torch.zeros(128).cuda()
y = vista_conv2d(x, w, sc, sh, 1, 1, 1, relu=True)
torch.cuda.synchronize()
print("done", y.float().abs().mean().item())
