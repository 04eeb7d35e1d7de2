"""bench.py — images/sec and end-to-end seconds of Staged k-layer feature transfer + per-layer LR
(BASELINE.json metric) on N B200s, one process per GPU.

Workload (BASELINE.json configs[1], the config the metric is quoted on that fits one GPU):
ResNet50 top-5 layers {conv4_6, conv5_1, conv5_2, conv5_3, fc}, Foods-shaped table:
20,000 synthetic 227x227 images and 130 structured features per GPU (weak scaling: the global
image table has 20,000 x N rows, the structured table is replicated on every rank), LR
T = 10, K = 20 power iterations.

One step = vista_transfer (join, 5 stages of partial inference, taps, concat) + vista_train(k)
for every layer k.  `value` is measured with all inputs resident in HBM; `e2e` repeats the
step through the same C-ABI with pinned HOST inputs (H2D inside the timed region) and the
trained weights read back to the host.  Inputs (3.1 GB of pixels per GPU) exceed the 126 MB L2.

--impl reference times the CPU oracle (oracle/, fp64, the box's host cores) on a bounded sample
of the same workload; it is the only other place bench.py executes oracle code.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "images/sec and end-to-end s for staged k-layer transfer+LR at 1/2/4/8 B200"
CONFIGS = {
    # name: (cnn, taps, images per GPU, d_s, table kind, LR T)
    "resnet50_top5_foods20k": (2, [0, 1, 2, 3, 4], 20000, 130, 0, 10),
    "alexnet_c1": (0, [0, 1, 2], 16, 8, 0, 5),
    "vgg16_fc678_amazon": (1, [0, 1, 2], 200000, 201, 1, 10),
    "resnet50_top5_amazon200k": (2, [0, 1, 2, 3, 4], 200000, 201, 1, 10),
}
DEFAULT = "resnet50_top5_foods20k"
TAP_NAMES = [["conv5", "fc6", "fc7", "fc8"], ["fc6", "fc7", "fc8"], ["conv4_6", "conv5_1", "conv5_2", "conv5_3", "fc"]]


def workload_config(name, world, n_img=None):
    """The `config` object both arms print (same workload, same keys)."""
    cnn, taps, n_default, d_s, kind, T = CONFIGS[name]
    n_img = n_img or n_default
    return {"workload": name, "images_per_gpu": n_img, "global_images": n_img * world,
            "taps": [TAP_NAMES[cnn][t] for t in taps], "d_s": d_s, "table": ["foods", "amazon"][kind],
            "lr_iters": T, "power_iters": 20, "plan": "staged",
            "parallelism": f"dp{world} (image shards, fp64 NCCL allreduce in LR)",
            "l2": "inputs larger than L2 (pixels %.2f GB/GPU)" % (n_img * 227 * 227 * 3 / 1e9)}


def env_int(k, d):
    try:
        return int(os.environ.get(k, d))
    except ValueError:
        return d


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled every 200 ms during the timed region."""

    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, device):
        self.device = device
        self.rows = []
        self.proc = None
        self.thread = None

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.device), f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "200"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except Exception:
            self.proc = None
            return
        self.thread = threading.Thread(target=self._read, daemon=True)
        self.thread.start()

    def _read(self):
        for line in self.proc.stdout:
            parts = [p.strip() for p in line.split(",")]
            if len(parts) >= 9:
                self.rows.append(parts)

    def stop(self):
        if self.proc is not None:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()
        if self.thread is not None:
            self.thread.join(timeout=2)
        return self.summary()

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"], "samples": 0}

        def num(x):
            try:
                return float(x)
            except ValueError:
                return None
        sm = [num(r[1]) for r in self.rows if num(r[1]) is not None]
        mx = [num(r[2]) for r in self.rows if num(r[2]) is not None]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in self.rows for i in range(4) if r[5 + i].lower() == "active"})
        pw = [num(r[3]) for r in self.rows if num(r[3]) is not None]
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "sm_mhz_min": min(sm) if sm else None, "reasons": reasons, "samples": len(self.rows),
                "power_w_max": max(pw) if pw else None, "power_w_median": statistics.median(pw) if pw else None}


def peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        return None


def ncu_traffic():
    """dram bytes per launch of the dominant kernel from the committed `ncu --set full` summary."""
    try:
        s = json.load(open(os.path.join(ROOT, "profiles", "ncu_summary.json")))
        return s.get("dominant", {}).get("dram_bytes_per_launch")
    except Exception:
        return None


def cpu_model():
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except Exception:
        pass
    return "unknown"


def oracle_sample(cfg_name, budget_s=20.0, nthreads=0):
    """The fp64 CPU oracle, as it stands, on a bounded sample of the workload: the full forward pass
    from pixels through every tap of S images (Eq. (2)), join + concat, and LR (O6) on the sample's
    rows.  Returns (images/s, seconds, images, threads, description)."""
    import numpy as np

    import gen
    import oracle
    cnn, taps, n_img, d_s, kind, T = CONFIGS[cfg_name]
    cores = nthreads or os.cpu_count() or 1
    # two images per host thread: ~10-15 s of fp64 work for ResNet50 whatever the core count
    S = max(1, min(2 * cores, n_img))
    tab = gen.make_tables(S, d_s, kind=kind)
    t0 = time.perf_counter()
    F, _ = oracle.features(cnn, 1, tab.images, taps=taps, nthreads=cores)
    ps, pi, te = oracle.join(tab.img_keys, tab.str_keys, 5)
    for t in taps:
        MM = oracle.concat(tab.X, F[t], ps, pi)
        te2 = te.copy()
        if te2.all():
            te2[0] = 0
        oracle.lr_train(MM, tab.labels[ps], te2, iters=T)
    dt = time.perf_counter() - t0
    desc = (f"{S} of {n_img} images per GPU: fp64 forward pass from pixels through taps {taps} "
            f"(oracle.features), join, concat and LR T={T}, K=20 on the sample's rows")
    return S / dt, dt, S, cores, desc


def run_reference(args):
    """--impl reference: the CPU oracle on a bounded sample per step (rank 0 only)."""
    rank = env_int("RANK", 0)
    world = env_int("WORLD_SIZE", 1)
    if rank != 0:
        return 0
    times = []
    for i in range(args.warmup + args.steps):
        v, dt, S, cores, desc = oracle_sample(args.config)
        if i >= args.warmup:
            times.append((S, dt))
    S_tot = sum(s for s, _ in times)
    T_tot = sum(t for _, t in times)
    value = S_tot / T_tot
    cnn, taps, n_img, d_s, kind, T = CONFIGS[args.config]
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": "images/s", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1000.0 * T_tot / max(len(times), 1),
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64",
        "data": "synthetic", "config": workload_config(args.config, world),
        "cpu_baseline": {"value": value, "unit": "images/s", "cores": os.cpu_count(), "kind": "oracle",
                         "sample": desc, "cpu_model": cpu_model()},
        "e2e": {"value": value, "unit": "images/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
        "gpu_launches": 0,
    }
    print(json.dumps(line), flush=True)
    return 0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default=DEFAULT, choices=sorted(CONFIGS))
    ap.add_argument("--e2e-steps", type=int, default=5)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--images", type=int, default=0, help="override images per GPU (debug only)")
    ap.add_argument("--micro-batch", type=int, default=0, help="stage-1 micro-batch (0 = planner)")
    ap.add_argument("--from-base", action="store_true",
                    help="App. B: materialise the first requested layer once (untimed, reported as materialize_s) "
                         "and time vista_transfer_from_base + train instead of the transfer from pixels")
    ap.add_argument("--model", default="lr", choices=["lr", "mlp"],
                    help="downstream model M per layer: lr (the product, PAPER.md:378) or the 3-layer MLP "
                         "(PAPER.md:383, vista_train_mlp, 10 steps)")
    ap.add_argument("--plan", default="staged", choices=["staged", "eager", "lazy"],
                    help="logical plan (Fig 5): staged is the product; eager / lazy for config 4 comparisons")
    ap.add_argument("--api", default="run", choices=["run", "split"],
                    help="run: vista_run (M of layer k on a second stream beside stage k+1, S6); split: "
                         "vista_transfer then vista_train(k) per layer")
    ap.add_argument("--dry-run", action="store_true",
                    help="print the launch command (torchrun re-exec for --gpus N > 1) and exit")
    args = ap.parse_args()
    if args.gpus > 1 and "RANK" not in os.environ:
        # one process per GPU: re-exec this command under torchrun (the driver may also launch us that way)
        port = env_int("MASTER_PORT", 29500 + os.getpid() % 1000)
        cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
               "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__)] + sys.argv[1:]
        if args.dry_run:
            print(json.dumps({"launch": cmd}))
            return 0
        sys.stdout.flush()
        os.execv(sys.executable, cmd)
    if args.dry_run:
        print(json.dumps({"launch": None, "rank": env_int("RANK", 0), "world": env_int("WORLD_SIZE", 1)}))
        return 0
    if "RANK" in os.environ and env_int("WORLD_SIZE", 1) != args.gpus:
        print(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={env_int('WORLD_SIZE', 1)}; using WORLD_SIZE",
              file=sys.stderr)
    if args.impl == "reference":
        return run_reference(args)

    import numpy as np
    import torch
    import torch.distributed as dist

    import gen
    from paper_conf_sigmod_nakandalak20_b200 import Vista, vista_nccl_unique_id

    rank, world = env_int("RANK", 0), env_int("WORLD_SIZE", 1)
    local = env_int("LOCAL_RANK", 0)
    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    cnn, taps, n_img, d_s, kind, T = CONFIGS[args.config]
    if args.images:
        n_img = args.images
    N_global = n_img * world
    # ---- synthetic inputs: this rank's image shard + the whole structured table ----
    t0 = time.time()
    tab = gen.make_tables(N_global, d_s, kind=kind, r0=rank * n_img, n_img=n_img)
    gen_s = time.time() - t0
    dev = torch.device("cuda", local)
    d_px = torch.from_numpy(tab.images).to(dev)
    d_ik = torch.from_numpy(tab.img_keys).to(dev)
    d_X = torch.from_numpy(tab.X).to(dev)
    d_sk = torch.from_numpy(tab.str_keys).to(dev)
    d_y = torch.from_numpy(tab.labels).to(dev)
    h_px = torch.from_numpy(tab.images).pin_memory()
    h_ik = torch.from_numpy(tab.img_keys).pin_memory()
    h_X = torch.from_numpy(tab.X).pin_memory()
    h_sk = torch.from_numpy(tab.str_keys).pin_memory()
    h_y = torch.from_numpy(tab.labels).pin_memory()
    h2d_bytes = sum(t.numel() * t.element_size() for t in (h_px, h_ik, h_X, h_sk, h_y))
    uid = None
    if world > 1:
        obj = [vista_nccl_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        uid = obj[0]
    stream = torch.cuda.current_stream(dev)
    v = Vista(cnn, layers=taps, n_str_rows=len(tab.str_keys), d_s=d_s, n_images_local=n_img, iters=T,
              power_iters=20, split_seed=5, weight_seed=1, rank=rank, world=world, nccl_uid=uid, device=local,
              stream=stream.cuda_stream, micro_batch=args.micro_batch, plan=args.plan)
    info = v.plan_info()
    d_tot = [d_s + d for d in info["d_l"]]
    materialize_s = None
    if args.from_base:
        H, W, C, _ = v.base_shape()
        d_base = torch.empty((n_img, H, W, C), dtype=torch.bfloat16, device=dev)
        torch.cuda.synchronize(dev)
        t0 = time.time()
        v.materialize(d_px, d_base)
        materialize_s = time.time() - t0
        h_base = torch.empty((n_img, H, W, C), dtype=torch.bfloat16).pin_memory()
        h_base.copy_(d_base)
        h2d_bytes += h_base.numel() * 2 - h_px.numel()

    def step(host=False):
        if args.from_base:
            if host:
                v.transfer_from_base(h_base, h_ik, h_X, h_sk, h_y)
            else:
                v.transfer_from_base(d_base, d_ik, d_X, d_sk, d_y)
        elif args.api == "run" and args.model == "lr":
            if host:
                return v.run(h_px, h_ik, h_X, h_sk, h_y, d_tot)
            return v.run(d_px, d_ik, d_X, d_sk, d_y, d_tot, want_weights=False)
        elif host:
            v.transfer(h_px, h_ik, h_X, h_sk, h_y)
        else:
            v.transfer(d_px, d_ik, d_X, d_sk, d_y)
        out = []
        for k in range(len(taps)):
            if args.model == "mlp":
                P, met = v.train_mlp(k, d_tot[k], iters=10, seed=3, want_weights=host)
                out.append((None, None, met))
            else:
                out.append(v.train(k, d_tot[k]))
        return out

    def barrier():
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize(dev)

    step_ms = {}

    def timed(nsteps, host=False):
        barrier()
        evs = [torch.cuda.Event(enable_timing=True) for _ in range(nsteps + 1)]
        evs[0].record(stream)
        res = None
        for i in range(nsteps):
            res = step(host)
            evs[i + 1].record(stream)
        barrier()
        ms = evs[0].elapsed_time(evs[-1])
        step_ms["e2e" if host else "device"] = [round(evs[i].elapsed_time(evs[i + 1]), 2) for i in range(nsteps)]
        if world > 1:
            t = torch.tensor([ms], device=dev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            ms = float(t.item())
        return ms, res

    # the clock sampler (nvidia-smi) starts before the warm-up: its NVML start-up stalls the GPU for a
    # few hundred ms, which must not land inside the timed region
    sampler = ClockSampler(local)
    sampler.start()
    for _ in range(args.warmup):
        step()
    sampler.rows.clear()  # keep only samples of the timed region
    l0 = v_launches()
    ms, res = timed(args.steps)
    launches = v_launches() - l0
    clocks = sampler.stop()
    ms_step = ms / args.steps
    value = N_global / (ms_step / 1000.0)
    # ---- e2e: host inputs through the C-ABI, weights back to the host ----
    peak_meas = None
    graph_info = {"cnn_graph": v.plan_info()["cnn_graph"], "kernels": v.plan_info()["cnn_graph_kernels"]}
    if args.e2e_steps > 0:
        step(host=True)  # untimed warm-up of the host-input path (sizes its per-chunk pixel buffer)
        pinfo = v.plan_info()  # pool high-water mark of that transfer from host pixels vs the prediction
        graph_info = {"cnn_graph": pinfo["cnn_graph"], "kernels": pinfo["cnn_graph_kernels"]}
        peak_meas = {"pred": pinfo["peak_bytes_pred"], "meas": pinfo["peak_bytes_meas"],
                     "reserved": pinfo["peak_reserved_meas"],
                     "meas_over_pred": pinfo["peak_bytes_meas"] / max(pinfo["peak_bytes_pred"], 1)}
        e2e_ms, _ = timed(args.e2e_steps, host=True)
        e2e_step = e2e_ms / args.e2e_steps
    else:  # profiling runs only (no e2e number)
        e2e_ms, e2e_step = 0.0, float("nan")
    d2h = (sum((d + 1) * 8 for d in d_tot) if args.model == "lr"
           else sum(4 * (1024 * d + 3 * 1024 + 1024 * 1024 + 1) for d in d_tot)) + len(taps) * 8 * 80
    # ---- instrumented step: per-kernel-class device time (CUDA events on the launch stream) ----
    pk = peaks()
    tensor_peak = pk.get("bf16_tflops_sustained") if pk else None
    peak_src = "MEASURED_PEAKS.json bf16_tflops_sustained (kernel timed inside a long step)"
    if tensor_peak is None:
        tensor_peak, peak_src = 1400.0, "fallback B200_PROFILING.md sustained ~1.4 PFLOP/s"
    hbm_peak = pk.get("hbm_gbs") if pk else None
    hbm_src = "MEASURED_PEAKS.json hbm_gbs (copy, read+write bytes)"
    if hbm_peak is None:
        hbm_peak, hbm_src = 7700.0, "fallback B200_PROFILING.md nominal 7.7 TB/s"
    v.set_profiling(True)
    v.set_roofline(tensor_peak, hbm_peak)
    # three instrumented steps, the one with the median conv-class time reported (one step's per-class sums move by
    # ~2 % with the power-capped clock)
    profs = []
    for _ in range(1 if os.environ.get("VISTA_PROF_LOG") else 3):  # (a per-launch log holds exactly one step)
        v.profile(reset=True)
        step()
        profs.append(v.profile(reset=True))
    v.set_profiling(False)
    profs.sort(key=lambda q: q["conv_fc_tcgen05"]["ms"])
    prof = profs[len(profs) // 2]
    conv = prof["conv_fc_tcgen05"]
    achieved = conv["flops"] / (conv["ms"] / 1000.0) / 1e12 if conv["ms"] > 0 else None
    total_prof_ms = sum(p["ms"] for p in prof.values())
    roof = {
        "kernel": "conv_tc_kernel (tcgen05 implicit-GEMM conv/FC, all launches of one step)",
        "bound": "tensor", "achieved": achieved, "peak": tensor_peak, "unit": "TFLOP/s",
        "frac": (achieved / tensor_peak) if achieved else None, "traffic": ncu_traffic(),
        "peak_source": peak_src, "launches_per_step": conv["launches"],
        "share_of_step": conv["ms"] / total_prof_ms if total_prof_ms else None,
        "algorithmic_flops_per_step": conv["flops"],
        # north_star's roofline: per launch the slower of its FLOPs at tensor peak and its algorithmic bytes
        # at HBM bandwidth, summed over the launches, divided by their measured time
        "mixed": {
            "conv_frac": (conv["roof_ms"] / conv["ms"]) if conv["ms"] > 0 else None,
            "conv_roof_ms": conv["roof_ms"], "conv_ms": conv["ms"],
            "step_frac": (sum(p["roof_ms"] for p in prof.values()) / total_prof_ms) if total_prof_ms else None,
            "tensor_peak_tflops": tensor_peak, "hbm_peak_gbs": hbm_peak, "hbm_peak_source": hbm_src,
        },
    }
    breakdown = {k: {"ms": round(p["ms"], 3), "launches": p["launches"],
                     "gbps": (p["bytes"] / (p["ms"] / 1000.0) / 1e9) if p["ms"] > 0 and p["bytes"] else None}
                 for k, p in prof.items() if p["launches"]}
    if "lr_pass" in breakdown and breakdown["lr_pass"]["launches"] == 1:
        breakdown["lr_pass"]["note"] = ("vista_run trains every layer side by side (one stream per layer): one record = the "
                                        "whole LR phase from fork to join; gbps = algorithmic pass bytes / that span")
    # ---- LR results of the last timed step (sanity, identical on all ranks) ----
    accs = [round(r[2]["test_acc"], 2) for r in res]
    cpu = None
    if rank == 0 and not args.no_cpu_baseline:
        try:
            cv, cdt, cS, ccores, cdesc = oracle_sample(args.config)
            cpu = {"value": cv, "unit": "images/s", "cores": ccores, "kind": "oracle", "sample": cdesc,
                   "seconds": cdt, "cpu_model": cpu_model()}
        except Exception as e:  # the baseline must never break the GPU number
            cpu = {"value": None, "unit": "images/s", "cores": os.cpu_count(), "kind": "oracle",
                   "sample": f"failed: {e}"}
    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": "images/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_step, "end_to_end_s": ms_step / 1000.0,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "bf16",
            "data": "synthetic",
            "config": dict(workload_config(args.config, world, n_img), micro_batch=info["micro_batch"],
                           plan=args.plan + ("+prematerialized_base" if args.from_base else ""),
                           model=("mlp_1024x1024x1_T10" if args.model == "mlp" else "elastic_net_lr_T%d" % T),
                           api=("vista_run" if args.api == "run" and args.model == "lr" and not args.from_base
                                else "vista_transfer+vista_train"),
                           peak_bytes_pred=info["peak_bytes_pred"], peak_bytes=peak_meas,
                           **({"base_layer": TAP_NAMES[cnn][taps[0]], "materialize_s": round(materialize_s, 3)}
                              if args.from_base else {})),
            "roofline": roof,
            "cpu_baseline": cpu,
            "e2e": {"value": N_global / (e2e_step / 1000.0), "unit": "images/s", "ms_per_step": e2e_step,
                    "h2d_bytes_per_step": h2d_bytes, "d2h_bytes_per_step": d2h,
                    "note": ("vista_run with pinned host inputs (H2D per stage-1 micro-batch inside the step), every "
                             "layer's trained weights and metrics read back" if args.api == "run" else
                             "vista_transfer with pinned host inputs + vista_train weights to host")},
            "gpu_launches": launches,
            "cuda_graph": graph_info,
            "clocks": clocks,
            "breakdown_ms": breakdown,
            "test_acc_per_layer": accs,
            "input_gen_s": round(gen_s, 1),
            "step_ms": step_ms,
        }
        print(json.dumps(line), flush=True)
    v.close()
    if world > 1:
        dist.destroy_process_group()
    return 0


def v_launches():
    from paper_conf_sigmod_nakandalak20_b200.vista import lib
    import ctypes
    f = lib().vista_kernel_launches
    f.restype = ctypes.c_int64
    return int(f())


if __name__ == "__main__":
    sys.exit(main())
