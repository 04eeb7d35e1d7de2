"""Dump MM_k (bf16 bits) of small synthetic workloads to gpurun_out/ for offline analysis."""
import sys; sys.path.insert(0, '.')
import numpy as np, torch, gen
from paper_conf_sigmod_nakandalak20_b200 import Vista
for cnn, taps, n, d_s in ((0, [0, 1], 800, 8), (2, [3, 4], 600, 130)):
    tab = gen.make_tables(n, d_s)
    v = Vista(cnn, layers=taps, n_str_rows=n, d_s=d_s, n_images_local=n, iters=2, split_seed=5, weight_seed=11)
    v.transfer(tab.images, tab.img_keys, tab.X, tab.str_keys, tab.labels)
    for k in range(len(taps)):
        f = v.features(k)
        np.savez(f"gpurun_out/mm_{cnn}_{k}.npz", mm=f["mm"].view(torch.int16).cpu().numpy(),
                 labels=f["labels"].cpu().numpy(), n_train=f["n_train"], d_s=f["d_s"], ds_pad=f["ds_pad"], d_l=f["d_l"])
    v.close()
