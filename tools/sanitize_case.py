"""Small end-to-end cases for compute-sanitizer (memcheck / racecheck / synccheck / initcheck):
every conv A-operand mode, the fused stem, the residual chains, projection units, weight multicast,
the tap, join, concat, and both LR paths (fused cooperative tail and the reduce/update kernels).

usage: python tools/sanitize_case.py <case>   cases: resnet, resnet_mc, resnet_run, alexnet, vgg, lr_unfused, mlp"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import gen  # noqa: E402
from paper_conf_sigmod_nakandalak20_b200 import Vista  # noqa: E402


def run(cnn, taps, n, d_s, mlp=False, **kw):
    tab = gen.make_tables(n, d_s, mismatch=True)
    v = Vista(cnn, layers=taps, n_str_rows=len(tab.str_keys), d_s=d_s, n_images_local=n, iters=2, power_iters=3,
              split_seed=5, weight_seed=11, **kw)
    v.transfer(tab.images, tab.img_keys, tab.X, tab.str_keys, tab.labels)
    for k in range(len(taps)):
        f = v.features(k)
        v.train(k, d_s + f["d_l"])
        if mlp and k == len(taps) - 1:
            v.train_mlp(k, d_s + f["d_l"], iters=2, want_weights=False)
    v.close()


if __name__ == "__main__":
    case = sys.argv[1]
    if case == "resnet":          # stem, chains (MID 64 / 128), projection units, halo / im2col 3x3, res4/res5, fc
        run(2, [0, 1, 2, 3, 4], 5, 16, micro_batch=5)
    elif case == "resnet_mc":     # 2-CTA weight multicast engages at >= 74 pair tiles
        os.environ["VISTA_MC"] = "1"
        run(2, [0, 4], 160, 8, micro_batch=160)
    elif case == "alexnet":       # cp.async gather A modes (conv1 / conv2), LRN, pools, fc
        run(0, [0, 1, 2, 3], 6, 8)
    elif case == "vgg":           # padded row view (conv1_1), row-segment halo tiles, fc6 from 25088
        run(1, [0, 1, 2], 2, 8)
    elif case == "lr_unfused":    # partials -> reduce -> update kernels (the world > 1 path on one rank)
        os.environ["VISTA_LR_FUSED"] = "0"
        run(0, [1, 2], 40, 8)
    elif case == "resnet_run":    # vista_run: every layer's LR side by side (cooperative grids on five streams, PDL)
        tab = gen.make_tables(7, 16, mismatch=True)
        v = Vista(2, layers=[0, 1, 2, 3, 4], n_str_rows=len(tab.str_keys), d_s=16, n_images_local=7, iters=2,
                  power_iters=3, split_seed=5, weight_seed=11, micro_batch=7)
        d = [16 + 0] * 5
        v.transfer(tab.images, tab.img_keys, tab.X, tab.str_keys, tab.labels)
        d = [16 + v.features(k)["d_l"] for k in range(5)]
        v.run(tab.images, tab.img_keys, tab.X, tab.str_keys, tab.labels, d)
        v.close()
    elif case == "mlp":
        run(0, [2], 40, 8, mlp=True)
    else:
        raise SystemExit("unknown case " + case)
    print("case", case, "ok")
