#!/usr/bin/env python
"""Kalman P-update microbench (BASELINE.json configs[4]): standalone blocked Kalman filter over
`--nblocks` blocks of `--block` (fp64 or fp32 storage, packed-symmetric), timed with CUDA events on the
launching stream.  `--sweep` runs the configs[4] grid (N_b 1024..10240 x N_p 26 651..1 027 082 x fp64/fp32,
p_defer 1 = every pass read-write, and the default 15) and prints one JSON line per point.

Reports the P-pass kernel in algorithmic GB/s: one stream of the symmetric blocks is
esize * sum n_i (n_i + 1) / 2 bytes; a read-write pass (the one that rewrites P) moves it twice, a read-only
pass once.  Fresh random g every update.  Against MEASURED_PEAKS.json hbm_gbs.
"""
import argparse
import json
import os
import sys

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
    ap.add_argument("--defer", type=int, default=15)
    ap.add_argument("--precision", type=int, default=64, choices=[64, 32])
    ap.add_argument("--sweep", action="store_true")
    args = ap.parse_args()
    if args.sweep:
        for prec in (64, 32):
            for nb in (1024, 2048, 4096, 8192, 10240):
                for npar in (26651, 131072, 507091, 1027082):
                    for d in (1, 15):
                        a = argparse.Namespace(**{**vars(args), "block": nb, "params": npar, "precision": prec,
                                                  "defer": d, "iters": 16 if d == 15 else 10})
                        run(a)
        return
    run(args)


def run(args):
    if args.params:
        q, r = divmod(args.params, args.block)
        blocks = [args.block] * q + ([r] if r else [])
    else:
        blocks = [args.block] * args.nblocks
    N = sum(blocks)
    kf = fk.KalmanFilter(blocks, dict(block_size=args.block, p_defer=args.defer, precision=args.precision))
    gs = torch.randn(args.warmup + args.iters, N, dtype=torch.float64, device="cuda")
    w = torch.zeros(N, dtype=torch.float64, device="cuda")
    abe = torch.full((1,), 0.1, dtype=torch.float64, device="cuda")
    for i in range(args.warmup):
        kf.update(gs[i], abe, 5.0, w)
    torch.cuda.synchronize()
    kf.timing(True)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for i in range(args.iters):
        kf.update(gs[args.warmup + i], abe, 5.0, w)
    e1.record()
    torch.cuda.synchronize()
    pass_ms, n, n_rw = kf.timing(False)
    upd_ms = e0.elapsed_time(e1) / args.iters
    stream = (4.0 if args.precision == 64 else 2.0) * sum(b * (b + 1) for b in blocks)
    alg = stream * (2 * n_rw + (n - n_rw))
    with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
        peak = json.load(f)["hbm_gbs"]
    gbps = alg / (pass_ms / 1000.0) / 1e9
    out = {"blocks": f"{len(blocks)} x {args.block}" + (f" (+{blocks[-1]})" if blocks[-1] != args.block else ""),
           "n_params": N, "precision": args.precision, "p_bytes": kf.info()["p_bytes_local"], "defer": args.defer, "passes": n, "rw_passes": n_rw,
           "avg_pass_ms": pass_ms / n, "pass_GBps": gbps, "pass_frac_of_measured_hbm": gbps / peak,
           "update_ms": upd_ms, "updates_per_s": 1000.0 / upd_ms, "peak_hbm_gbs": peak, "state": kf.state()}
    print(json.dumps(out), flush=True)
    kf.close()
    del gs
    torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
