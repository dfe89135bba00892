#!/usr/bin/env python
"""Kalman P-update microbench (BASELINE.json configs[4]): standalone blocked Kalman filter over
`--nblocks` blocks of `--block` (fp64, packed-symmetric), timed with CUDA events on the launching stream.

Reports the P-pass kernel (pending rank-1 apply + u = P g, one read + one write of every stored
element) in algorithmic GB/s = 8 * sum n_i (n_i + 1) / t, against MEASURED_PEAKS.json hbm_gbs.
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


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--block", type=int, default=10240)
    ap.add_argument("--nblocks", type=int, default=8)
    ap.add_argument("--params", type=int, default=0, help="total params (overrides nblocks; last block ragged)")
    ap.add_argument("--iters", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    args = ap.parse_args()
    if args.params:
        q, r = divmod(args.params, args.block)
        blocks = [args.block] * q + ([r] if r else [])
    else:
        blocks = [args.block] * args.nblocks
    N = sum(blocks)
    kf = fk.KalmanFilter(blocks, dict(block_size=args.block))
    g = torch.randn(N, dtype=torch.float64, device="cuda")
    w = torch.zeros(N, dtype=torch.float64, device="cuda")
    abe = torch.full((1,), 0.1, dtype=torch.float64, device="cuda")
    for _ in range(args.warmup):
        kf.update(g, abe, 5.0, w)
    torch.cuda.synchronize()
    kf.timing(True)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(args.iters):
        kf.update(g, abe, 5.0, w)
    e1.record()
    torch.cuda.synchronize()
    pass_ms, n = kf.timing(False)
    upd_ms = e0.elapsed_time(e1) / args.iters
    alg = 8.0 * sum(b * (b + 1) for b in blocks)
    with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
        peak = json.load(f)["hbm_gbs"]
    pms = pass_ms / n
    out = {"blocks": f"{len(blocks)} x {args.block}" + (f" (+{blocks[-1]})" if blocks[-1] != args.block else ""),
           "n_params": N, "p_bytes": kf.info()["p_bytes_local"], "alg_bytes_per_pass": alg,
           "pass_ms": pms, "pass_GBps": alg / pms / 1e6, "pass_frac_of_measured_hbm": alg / pms / 1e6 / peak,
           "update_ms": upd_ms, "update_GBps": alg / upd_ms / 1e6, "peak_hbm_gbs": peak, "state": kf.state()}
    print(json.dumps(out))


if __name__ == "__main__":
    main()
