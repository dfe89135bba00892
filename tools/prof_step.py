#!/usr/bin/env python
"""Kernel timeline of the bench step without ncu (CUPTI activity records through torch.profiler: real
concurrency, no cache flushes, no serialisation).  Prints per-kernel totals for the profiled steps and the
timeline of one force update (start offset, duration, stream) to read the critical path.

  python tools/prof_step.py [--config c2_water64] [--steps 2] [--eager]
"""
import argparse
import collections
import json
import os
import re
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_ppopp_huzslmlwtj24_b200 as fk  # noqa: E402
from fixtures import get_config, make_dataset, init_weights, force_groups  # noqa: E402


def short(n):
    n = n.replace("fekf::n64::", "fekf::").replace("fekf::n32::", "fekf::")
    m = re.search(r"dgemm_kernel<(\d+), (\d+), \d+, \d+, (\w+), (\w+), fekf::(\w+)", n)
    if m:
        return "dgemm<%s,%s,%s>" % (m.group(1), m.group(2), m.group(5))
    n = re.sub(r"\(.*", "", n).replace("void ", "").replace("fekf::", "")
    return re.sub(r"<fekf::EmbW<[^>]*>>", "", n)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="c2_water64")
    ap.add_argument("--steps", type=int, default=2)
    ap.add_argument("--eager", action="store_true")
    ap.add_argument("--precision", type=int, default=64)
    ap.add_argument("--net-precision", type=int, default=0)
    a = ap.parse_args()
    wl = get_config(a.config)
    m, opt = wl.model, wl.opt
    opt = type(opt)(**{**opt.__dict__, "precision": a.precision, "net_precision": a.net_precision})
    B = wl.batch
    ds = make_dataset(a.config, B)
    na = len(ds["types"])
    w0 = init_weights(m, 3, float(ds["energy"].mean() / na))
    ctx = fk.Context(m, opt, types=ds["types"], local_batch=B, global_batch=B, graph=not a.eager)
    dev = lambda x, dt=torch.float64: torch.as_tensor(np.ascontiguousarray(x)).to(dt).cuda()
    ctx.set_params(dev(w0))
    X, BX, E, F = dev(ds["coord"]), dev(ds["box"]), dev(ds["energy"]), dev(ds["force"])
    gi = [dev(force_groups(na, s, wl.seed), torch.int32) for s in range(20)]
    for s in range(3):
        ctx.train_step(X, BX, E, F, gi[s])
    torch.cuda.synchronize()
    from torch.profiler import profile, ProfilerActivity
    with profile(activities=[ProfilerActivity.CUDA]) as prof:
        for s in range(a.steps):
            ctx.train_step(X, BX, E, F, gi[3 + s])
        torch.cuda.synchronize()
    evs = [e for e in prof.events() if e.device_type == torch.autograd.DeviceType.CUDA and "Memcpy" not in e.name
           and "Memset" not in e.name]
    evs.sort(key=lambda e: e.time_range.start)
    tot = collections.defaultdict(float)
    cnt = collections.Counter()
    for e in evs:
        k = short(e.name)
        tot[k] += e.time_range.elapsed_us()
        cnt[k] += 1
    t0, t1 = evs[0].time_range.start, max(e.time_range.end for e in evs)
    span = (t1 - t0) / a.steps
    print("wall per step (first kernel start -> last kernel end) %.1f us" % span)
    print("| kernel | launches/step | us/step (sum of durations) |")
    for k, v in sorted(tot.items(), key=lambda x: -x[1])[:25]:
        print("| %s | %.0f | %.1f |" % (k, cnt[k] / a.steps, v / a.steps))
    # timeline of the second update of the first profiled step
    ups, cur = [], []
    for e in evs:
        cur.append(e)
        if short(e.name) == "kf_vec_kernel":
            ups.append(cur)
            cur = []
    u = ups[int(os.environ.get("PROF_UPDATE", "1"))]
    b0 = u[0].time_range.start
    print("\ntimeline of update %d: start offset, duration (us), kernel" % (ups.index(u) + 1))
    for e in u:
        print("%9.1f %8.1f  %s" % (e.time_range.start - b0, e.time_range.elapsed_us(), short(e.name)))
    ctx.close()


if __name__ == "__main__":
    main()
