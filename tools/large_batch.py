#!/usr/bin/env python
"""Large-batch FEKF on one B200 (proxy): one rank's share of a B_g = 16 x L job.

The paper's large-batch runs (Table 5) use B_g up to 4096 over 16 GPUs with the bs > 1024
preset lambda_0 = 0.90, nu = 0.996.  Only one GPU is available here, so this measures the per-GPU
step of such a job: local batch L images of water-64 on this GPU, global batch 16 L (sqrt(bs) of Eq. 2
and the preset follow B_g via fekf_opt_defaults), the full replicated P.  Not included: the two
all-reduces a 16-rank job adds per update (g: N_p + 1 doubles = 8.2 MB, and u when P is sharded), i.e.
this is the compute of one rank, not a multi-node measurement.  One JSON line per L.
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


def run(L, ranks, steps, warmup, config):
    wl = get_config(config)
    m = wl.model
    Bg = L * ranks
    od = fk.opt_defaults(Bg)
    opt = type(wl.opt)(**{**wl.opt.__dict__, "lambda0": od["lambda0"], "nu": od["nu"]})
    ds = make_dataset(config, L, seed=wl.seed + 7)
    na = len(ds["types"])
    w0 = init_weights(m, 3, float(ds["energy"].mean() / na))
    free0 = torch.cuda.mem_get_info()[0]
    ctx = fk.Context(m, opt, types=ds["types"], local_batch=L, global_batch=Bg)
    ctx.set_params(torch.as_tensor(w0).cuda())
    cu = lambda x, dt=torch.float64: torch.as_tensor(np.ascontiguousarray(x)).to(dt).cuda()
    inp = [cu(ds["coord"]), cu(ds["box"]), cu(ds["energy"]), cu(ds["force"])]
    groups = [cu(force_groups(na, s, wl.seed, opt.force_groups, opt.atoms_per_group), torch.int32)
              for s in range(warmup + steps)]
    for s in range(warmup):
        ctx.train_step(*inp, groups[s])
    torch.cuda.synchronize()
    used = free0 - torch.cuda.mem_get_info()[0]
    ctx.kf.timing(True)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for s in range(steps):
        met = ctx.train_step(*inp, groups[warmup + s])
    e1.record()
    torch.cuda.synchronize()
    pass_ms, pass_n, _ = ctx.kf.timing(False)
    ms = e0.elapsed_time(e1) / steps
    out = {"what": "large_batch_per_gpu", "config": config, "local_batch": L, "global_batch": Bg,
           "ranks_emulated": ranks, "lambda0": od["lambda0"], "nu": od["nu"], "ms_per_step": ms,
           "images_per_s_per_gpu": L / (ms / 1e3), "p_pass_ms_per_step": pass_ms / steps,
           "p_pass_share": pass_ms / steps / ms, "device_bytes_used": int(used),
           "metrics": met.cpu().tolist(),
           "note": "one rank's compute of a %d-rank job; the per-update all-reduces are not included" % ranks}
    print(json.dumps(out), flush=True)
    ctx.close()
    torch.cuda.empty_cache()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--batches", type=int, nargs="+", default=[32, 64, 128, 256])
    ap.add_argument("--ranks", type=int, default=16)
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--warmup", type=int, default=2)
    ap.add_argument("--config", default="c2_water64")
    a = ap.parse_args()
    for L in a.batches:
        run(L, a.ranks, a.steps, a.warmup, a.config)


if __name__ == "__main__":
    main()
