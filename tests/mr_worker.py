"""One rank of the world-2 library test (tests/test_gpu_multirank.py).

Runs the product's real collective path: vista_plan(world = 2) with a caller-supplied allreduce
(vista_sys_cfg.allreduce) backed by a gloo process group, because both ranks share the one GPU of
the test box (NCCL refuses two ranks on one device).  Every LR pass (stats, K power iterations,
T gradient steps, eval) and every MLP step goes through that hook.  Writes its results to
<out>/rank<r>.npz.

usage: python tests/mr_worker.py <out_dir> <n_images_global> <rank0_images> <mlp 0/1>
(rank / world / master address from the torchrun-style environment)
"""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    out, N, n0, mlp = sys.argv[1], int(sys.argv[2]), int(sys.argv[3]), int(sys.argv[4])
    tag = sys.argv[5] if len(sys.argv) > 5 else ""
    rank, world = int(os.environ["RANK"]), int(os.environ["WORLD_SIZE"])
    import torch
    import torch.distributed as dist

    import gen
    from paper_conf_sigmod_nakandalak20_b200 import Vista, torch_dist_allreduce
    torch.cuda.set_device(0)
    if world > 1:
        dist.init_process_group("gloo")
    # rank 0 owns image rows [0, n0), rank 1 owns [n0, N) (n0 = N: rank 1 has no images, no train rows)
    r0, n_img = (0, n0) if rank == 0 else (n0, N - n0)
    tab = gen.make_tables(N, 8, mismatch=True, r0=r0, n_img=n_img)
    taps = [0, 1, 2]
    v = Vista(0, layers=taps, n_str_rows=len(tab.str_keys), d_s=8, n_images_local=n_img, iters=10, split_seed=5,
              weight_seed=11, rank=rank, world=world, allreduce=torch_dist_allreduce() if world > 1 else None)
    v.transfer(tab.images, tab.img_keys, tab.X, tab.str_keys, tab.labels)
    res = {}
    for k in range(len(taps)):
        f = v.features(k)
        d = 8 + f["d_l"]
        w, b, met = v.train(k, d)
        res[f"w{k}"] = np.append(w, b)
        res[f"loss{k}"] = np.array(met["loss"][:10])
        res[f"met{k}"] = np.array([met["lambda_hat"], met["n_train"], met["n_test"], met["tp"], met["fp"], met["tn"],
                                   met["fn"]], dtype=np.float64)
        res[f"pair_str{k}"] = f["pair_str"].cpu().numpy()
        res[f"pair_img{k}"] = f["pair_img"].cpu().numpy() + r0  # global image rows
        res[f"mm{k}"] = f["mm"].view(torch.int16).cpu().numpy()
        res[f"n_train{k}"] = np.array([f["n_train"]])
        if mlp and k == 1:
            P, mm = v.train_mlp(k, d, iters=3, seed=3)
            res["mlp_W1"] = P["W1"]
            res["mlp_W2"] = P["W2"]
            res["mlp_w3"] = P["w3"]
            res["mlp_loss"] = np.array(mm["loss"][:3])
            res["mlp_met"] = np.array([mm["n_train"], mm["n_test"], mm["tp"], mm["fp"], mm["tn"], mm["fn"]], np.float64)
    v.close()
    np.savez(os.path.join(out, f"rank{rank}{tag}.npz"), **res)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
