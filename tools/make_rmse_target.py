#!/usr/bin/env python
"""Writes tests/golden/rmse_<config>.json: the fp64 CPU oracle's FEKF training trajectory (test-set
RMSE) and the time-to-target goal of the BASELINE.json metric "minutes to target RMSE".

Calls only oracle/ (the plain CPU implementation) and fixtures/ (seeded inputs): no value in the file
comes from the CUDA path.  The GPU side (tools/time_to_rmse.py, tests/test_parity_gpu.py) trains from
the same initial weights on the same minibatch / force-atom schedule and is compared against it.

Protocol: S_o oracle minibatch steps (1 energy + 4 force updates each) from
init_weights(m, 3, mean train E/atom); minibatch k = batch_schedule(n_train, B, k, seed); force atoms
of step k = force_groups(N_a, k, seed); test RMSE = E_rmse (per atom) + F_rmse (per component) on the
test split every `--every` steps.  The target is the best (lowest) RMSE the oracle reaches within its
S_o steps (reading R1 of DESIGN.md: the EKF trajectory is not monotone, so "the oracle's RMSE after S_o
steps" is taken as the best one it attained), with the step it first reached it.

  python tools/make_rmse_target.py [--config c1_cu32] [--steps 200] [--every 8] [--threads N] [--out PATH]
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
import oracle as O  # noqa: E402
from fixtures import get_config, make_dataset, init_weights, batch_schedule, force_groups  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="c1_cu32")
    ap.add_argument("--steps", type=int, default=64)
    ap.add_argument("--every", type=int, default=8)
    ap.add_argument("--threads", type=int, default=0)
    ap.add_argument("--out", default="")
    args = ap.parse_args()
    torch.set_num_threads(args.threads or os.cpu_count() or 1)
    wl = get_config(args.config)
    m, opt = wl.model, wl.opt
    tr = make_dataset(args.config, split="train")
    te = make_dataset(args.config, split="test")
    na = len(tr["types"])
    w0 = init_weights(m, 3, float(tr["energy"].mean() / na))
    st = O.FEKF.create(w0, m, opt)
    traj = []
    t0 = time.perf_counter()

    def evaluate(step):
        e, f = O.rmse(st.w, te["coord"], te["box"], te["types"], te["energy"], te["force"], m)
        traj.append([step, e, f])
        print(f"step {step:4d}  E_rmse {e:.6e}  F_rmse {f:.6e}  ({time.perf_counter() - t0:.0f} s)", flush=True)

    evaluate(0)
    train_s = 0.0
    for k in range(args.steps):
        idx = batch_schedule(wl.n_train, wl.batch, k, wl.seed)
        groups = force_groups(na, k, wl.seed, opt.force_groups, opt.atoms_per_group)
        t1 = time.perf_counter()
        O.train_step(st, tr["coord"][idx], tr["box"][idx], tr["types"], tr["energy"][idx], tr["force"][idx],
                     groups, m, opt)
        train_s += time.perf_counter() - t1
        if (k + 1) % args.every == 0 or k + 1 == args.steps:
            evaluate(k + 1)
    out = {
        "_source": "tools/make_rmse_target.py (fp64 CPU oracle only; fixtures/ seeded inputs)",
        "_protocol": "SURVEY 8d(iii): S_o oracle steps from init_weights(m, 3, mean train E/atom); "
                     "batch_schedule / force_groups with the workload seed; RMSE = E_rmse + F_rmse (P:L299) "
                     "on the test split",
        "config": args.config, "S_o": args.steps, "every": args.every, "init_seed": 3,
        "trajectory": traj, "target": min(e + f for _, e, f in traj),
        "target_step": min(traj, key=lambda x: x[1] + x[2])[0], "final": traj[-1][1] + traj[-1][2],
        "oracle_train_seconds": train_s, "oracle_threads": torch.get_num_threads(),
    }
    path = args.out or os.path.join(ROOT, "tests", "golden", f"rmse_{args.config}.json")
    with open(path, "w") as f:
        json.dump(out, f, indent=1)
    print("wrote", path, "target", out["target"])


if __name__ == "__main__":
    main()
