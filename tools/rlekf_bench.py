#!/usr/bin/env python
"""the RLEKF instance-by-instance schedule (bs = 1; Table 5 column 1) on
the same kernels: one image per minibatch (1 energy + 4 force updates each), graph-replayed steps, timed
with CUDA events.  Prints one JSON line with images/s next to the FEKF minibatch figure of the same run.

  python tools/rlekf_bench.py [--config c2_water64] [--images 40] [--fekf-steps 10]
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
from fixtures import get_config, make_dataset, init_weights, force_groups  # noqa: E402


def timed(ctx, batches, warm=3):
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
    for k in range(warm):
        ctx.train_step(*batches[k % len(batches)])
    torch.cuda.synchronize()
    ev[0].record()
    for b in batches:
        ctx.train_step(*b)
    ev[1].record()
    torch.cuda.synchronize()
    return ev[0].elapsed_time(ev[1])


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="c2_water64")
    ap.add_argument("--images", type=int, default=40)
    ap.add_argument("--fekf-steps", type=int, default=10)
    a = ap.parse_args()
    wl = get_config(a.config)
    m, opt = wl.model, wl.opt
    B = wl.batch
    n = max(a.images, B)
    ds = make_dataset(a.config, n)
    na = len(ds["types"])
    w0 = init_weights(m, 3, float(ds["energy"].mean() / na))
    dev = lambda x, dt=torch.float64: torch.as_tensor(np.ascontiguousarray(x)).to(dt).cuda()
    out = {"config": a.config, "metric": "EKF train images/sec"}
    # RLEKF: one image per step
    ctx = fk.Context(m, opt, types=ds["types"], local_batch=1, global_batch=1)
    ctx.set_params(dev(w0))
    bat = [(dev(ds["coord"][i:i + 1]), dev(ds["box"][i:i + 1]), dev(ds["energy"][i:i + 1]), dev(ds["force"][i:i + 1]),
            dev(force_groups(na, i, wl.seed), torch.int32)) for i in range(a.images)]
    ms = timed(ctx, bat)
    out["rlekf_bs1"] = {"images_per_s": a.images / (ms / 1000.0), "ms_per_image": ms / a.images, "images": a.images}
    ctx.close()
    # FEKF minibatch of the workload's batch
    ctx = fk.Context(m, opt, types=ds["types"], local_batch=B, global_batch=B)
    ctx.set_params(dev(w0))
    bat = [(dev(ds["coord"][:B]), dev(ds["box"][:B]), dev(ds["energy"][:B]), dev(ds["force"][:B]),
            dev(force_groups(na, s, wl.seed), torch.int32)) for s in range(a.fekf_steps)]
    ms = timed(ctx, bat)
    out["fekf_minibatch"] = {"images_per_s": B * a.fekf_steps / (ms / 1000.0), "ms_per_step": ms / a.fekf_steps,
                             "batch": B}
    out["throughput_ratio_fekf_over_rlekf"] = out["fekf_minibatch"]["images_per_s"] / out["rlekf_bs1"]["images_per_s"]
    ctx.close()
    print(json.dumps(out), flush=True)


if __name__ == "__main__":
    main()
