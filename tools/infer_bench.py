#!/usr/bin/env python
"""Inference / evaluation path (the online-learning loop's model evaluation):
energy, per-atom energy, forces and virial of new configurations with given weights, through the C ABI
(`fekf_forward`: a1-a5 kernels only).  Times `--iters` batches of `--batch` images on one GPU with CUDA
events (inputs resident in HBM).  Parity of this path at the bench batch size against the fp64 CPU
oracle is tests/test_parity_gpu.py::test_forward_full_batch_sampled.

  python tools/infer_bench.py [--config c2_water64] [--batch 32] [--iters 20]
Prints one JSON line: images/s and atom-evaluations/s.
"""
import argparse
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_ppopp_huzslmlwtj24_b200 as fk  # noqa: E402
from fixtures import get_config, make_dataset, init_weights  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="c2_water64")
    ap.add_argument("--batch", type=int, default=0)
    ap.add_argument("--iters", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    a = ap.parse_args()
    wl = get_config(a.config)
    m = wl.model
    B = a.batch or wl.batch
    ds = make_dataset(a.config, B, split="test")
    na = len(ds["types"])
    w = init_weights(m, 3, float(ds["energy"].mean() / na))
    dev = lambda x: torch.as_tensor(np.ascontiguousarray(x)).cuda()
    ctx = fk.Context(m, wl.opt, types=ds["types"], local_batch=B, global_batch=B)
    ctx.set_params(dev(w))
    X, BX = dev(ds["coord"]), dev(ds["box"])
    for _ in range(a.warmup):
        ctx.forward(X, BX)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(a.iters):
        _, e, f, v = ctx.forward(X, BX)
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / a.iters
    out = {"metric": "inference images/s (E, F, virial)", "config": a.config, "batch": B, "ms_per_batch": ms,
           "images_per_s": B / (ms / 1e3), "atom_evals_per_s": B * na / (ms / 1e3), "dtype": "f64"}
    ctx.close()
    print(json.dumps(out), flush=True)


if __name__ == "__main__":
    main()
