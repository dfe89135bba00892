#!/usr/bin/env python
"""Naive-EKF vs FEKF on the B200.  Prints one JSON line per measurement.

1. Kalman level (`--kalman`): the water-64 filter (110 blocks, N_p = 1 027 082, 39 GiB packed fp64 P);
   one Naive-EKF update with n = 8 / 16 / 32 per-sample gradients (fekf_kf_update_naive) against one FEKF
   update (fekf_kf_update, default p_defer), CUDA events on the launching stream.  The naive update is
   DMMA-bound: algorithmic flops = sum_b [2 n_b^2 n (U = P G over the symmetric block) + n_b (n_b + 1) n
   (the rank-n correction of the stored triangle)], reported against the measured fp64 DMMA peak
   (tools/fp64_peak.cu: 37.1 TFLOP/s on this pool's B200; MEASURED_PEAKS.json has no fp64 entry).
2. Step level (`--step`): one minibatch (1 energy + 4 force updates) of each optimizer on a config,
   images/s; Naive-EKF runs per-image Jacobians (eager) + rank-B updates.
"""
import argparse
import json
import os
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_ppopp_huzslmlwtj24_b200 as fk  # noqa: E402
from fixtures import get_config, make_dataset, init_weights, force_groups  # noqa: E402

FP64_DMMA_TFLOPS = 37.1   # tools/fp64_peak.cu on the B200


def kalman(args):
    wl = get_config("c2_water64")
    _, blocks = fk.plan_layout(wl.model, wl.opt.block_size)
    N = sum(blocks)
    kf = fk.KalmanFilter(blocks, dict(block_size=wl.opt.block_size))
    w = torch.zeros(N, dtype=torch.float64, device="cuda")
    gen = torch.Generator(device="cuda").manual_seed(1)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    # FEKF update (the funnel), same filter
    g = torch.randn(args.warmup + args.iters, N, dtype=torch.float64, device="cuda", generator=gen) * 1e-2
    abe1 = torch.full((1,), 0.05, dtype=torch.float64, device="cuda")
    for i in range(args.warmup):
        kf.update(g[i], abe1, 5.0, w)
    torch.cuda.synchronize()
    e0.record()
    for i in range(args.iters):
        kf.update(g[args.warmup + i], abe1, 5.0, w)
    e1.record()
    torch.cuda.synchronize()
    fekf_ms = e0.elapsed_time(e1) / args.iters
    del g
    print(json.dumps({"what": "fekf_update", "n_params": N, "blocks": len(blocks), "update_ms": fekf_ms}), flush=True)
    for n in args.n:
        G = torch.randn(n, N, dtype=torch.float64, device="cuda", generator=gen) * 1e-2
        abe = torch.rand(n, dtype=torch.float64, device="cuda", generator=gen) * 0.1
        for _ in range(args.warmup):
            kf.update_naive(G, abe, w)
        torch.cuda.synchronize()
        e0.record()
        for _ in range(args.iters):
            kf.update_naive(G, abe, w)
        e1.record()
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / args.iters
        flops = float(sum(2.0 * b * b * n + b * (b + 1.0) * n for b in blocks))
        tf = flops / (ms / 1e3) / 1e12
        print(json.dumps({"what": "naive_update", "n_samples": n, "n_params": N, "update_ms": ms,
                          "vs_fekf_update": ms / fekf_ms,
                          "roofline": {"bound": "tensor", "achieved": tf, "peak": FP64_DMMA_TFLOPS, "unit": "TFLOP/s",
                                       "frac": tf / FP64_DMMA_TFLOPS, "alg_flops_per_update": flops,
                                       "peak_source": "tools/fp64_peak.cu (measured DMMA, fp64)"},
                          "state": kf.state()}), flush=True)
        del G
    kf.close()
    torch.cuda.empty_cache()


def step(args):
    wl = get_config(args.config)
    m, opt = wl.model, wl.opt
    B = args.batch or wl.batch
    ds = make_dataset(args.config, B)
    na = len(ds["types"])
    w0 = init_weights(m, 3, float(ds["energy"].mean() / na))
    cu = lambda x, dt=torch.float64: torch.as_tensor(np.ascontiguousarray(x)).to(dt).cuda()
    inp = [cu(ds["coord"]), cu(ds["box"]), cu(ds["energy"]), cu(ds["force"])]
    res = {}
    for mode in ("fekf", "naive"):
        ctx = fk.Context(m, opt, types=ds["types"], local_batch=B, global_batch=B)
        ctx.set_params(cu(w0))
        fn = ctx.train_step if mode == "fekf" else ctx.naive_train_step
        groups = [cu(force_groups(na, s, 17, opt.force_groups, opt.atoms_per_group), torch.int32)
                  for s in range(args.warmup + args.steps)]
        for s in range(args.warmup):
            fn(*inp, groups[s])
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        t0 = time.perf_counter()
        e0.record()
        for s in range(args.steps):
            met = fn(*inp, groups[args.warmup + s])
        e1.record()
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / args.steps
        res[mode] = ms
        print(json.dumps({"what": f"{mode}_step", "config": args.config, "images_per_step": B, "ms_per_step": ms,
                          "images_per_s": B / (ms / 1e3), "launches_per_step": ctx.last_launch_count(),
                          "wall_ms_per_step": (time.perf_counter() - t0) * 1e3 / args.steps,
                          "metrics": met.cpu().tolist()}), flush=True)
        ctx.close()
        torch.cuda.empty_cache()
    print(json.dumps({"what": "naive_over_fekf_step_time", "config": args.config, "ratio": res["naive"] / res["fekf"]}))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--kalman", action="store_true")
    ap.add_argument("--step", action="store_true")
    ap.add_argument("--n", type=int, nargs="+", default=[8, 16, 32])
    ap.add_argument("--config", default="c2_water64")
    ap.add_argument("--batch", type=int, default=0)
    ap.add_argument("--iters", type=int, default=5)
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--warmup", type=int, default=2)
    args = ap.parse_args()
    if not (args.kalman or args.step):
        args.kalman = args.step = True
    if args.kalman:
        kalman(args)
    if args.step:
        step(args)


if __name__ == "__main__":
    main()
