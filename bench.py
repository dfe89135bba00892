#!/usr/bin/env python
"""EKF training throughput of the B200-native FEKF DeePMD step (BASELINE.json metric).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config c2_water64] [--impl fekf|reference]

One step = one minibatch of the paper's schedule: 1 energy update + 4 force updates, each a
forward, a Jacobian, the early reduction (NCCL all-reduce over ranks) and the blocked Kalman update.
Workload at N=1: BASELINE.json configs[1] (water-64, 192 atoms, se_a 6.0/0.5, sel [46,92], embedding
(25,50,100), M^<=16, fitting (240,240,240), 32 images per GPU, N_b = 10240 -> 1 027 082 parameters,
110 P blocks, 39 GiB of packed fp64 P).  Weak scaling: 32 images per GPU, global batch 32*N, P sharded.
Prints ONE JSON line on rank 0.
"""
import argparse
import json
import math
import os
import statistics
import subprocess
import sys
import tempfile
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

from fixtures import get_config, make_dataset, init_weights, force_groups  # noqa: E402

METRIC = "EKF train images/sec"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=16)   # 16 steps = 80 updates = 5 cycles of the read-write pass (p_defer 15)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="c2_water64")
    ap.add_argument("--impl", default="fekf", choices=["fekf", "reference"])
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--precision", type=int, default=64, choices=[64, 32],
                    help="64, or 32 = the fp32 variant (P stored fp32 and fp32 nets, reading Z22)")
    ap.add_argument("--net-precision", type=int, default=0, choices=[0, 32, 64],
                    help="nets' arithmetic: 0 = follow --precision, 32 or 64")
    ap.add_argument("--p-defer", type=int, default=None, help="override the deferred-correction depth")
    ap.add_argument("--p-mode", type=int, default=0, choices=[0, 1],
                    help="N > 1: 0 = P sharded over ranks (partial u all-reduced), 1 = replicated (the paper, P:L229)")
    return ap.parse_args()


def dist_env():
    return int(os.environ.get("RANK", 0)), int(os.environ.get("WORLD_SIZE", 1)), int(os.environ.get("LOCAL_RANK", 0))


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured"
    return 6650.0, "fallback (B200_PROFILING.md)"


# ---------------------------------------------------------------------------------------------
# clocks sampled during the timed region (B200_PROFILING.md clocks line)
# ---------------------------------------------------------------------------------------------
class Clocks:
    """SM clock and clock-event reasons sampled every 20 ms by an NVML thread (nvidia_ml_py) between mark()
    and stop() — the timed region; initialised before the warm-up so NVML's start-up never overlaps it.
    Falls back to an `nvidia-smi -lms 100` subprocess when NVML is unavailable."""
    REASONS = (("hw_slowdown", 0x8), ("hw_thermal_slowdown", 0x40), ("sw_thermal_slowdown", 0x20),
               ("sw_power_cap", 0x4))

    def __init__(self, index):
        import threading
        self.index = index
        self.rows = []
        self.on = False
        self.stop_ev = threading.Event()
        self.nv = None
        self.p = None
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.max_mhz = float(pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM))
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        except Exception:
            self.nv = None
            self.f = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)
            q = ("timestamp,clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
                 "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
            try:
                self.p = subprocess.Popen(["nvidia-smi", "-i", str(index), f"--query-gpu={q}",
                                           "--format=csv,noheader,nounits", "-lms", "100"],
                                          stdout=self.f, stderr=subprocess.DEVNULL)
            except Exception:
                self.p = None

    def _run(self):
        while not self.stop_ev.is_set():
            if self.on:
                try:
                    sm = float(self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM))
                    rs = int(self.nv.nvmlDeviceGetCurrentClocksEventReasons(self.h))
                    self.rows.append((sm, rs))
                except Exception:
                    pass
            self.stop_ev.wait(0.02)

    def mark(self):
        import datetime
        self.t0 = datetime.datetime.now()
        self.on = True

    def stop(self):
        import datetime
        t1 = datetime.datetime.now()
        self.on = False
        if self.nv is not None:
            self.stop_ev.set()
            self.t.join(1.0)
            if not self.rows:
                return None
            sm = [r[0] for r in self.rows]
            reasons = sorted({n for _, m in self.rows for n, bit in self.REASONS if m & bit})
            return {"sm_mhz": statistics.median(sm), "sm_max_mhz": self.max_mhz, "reasons": reasons,
                    "samples": len(self.rows), "source": "nvml, 20 ms"}
        if self.p is None:
            return None
        self.p.terminate()
        try:
            self.p.wait(5)
        except Exception:
            self.p.kill()
        self.f.flush()
        rows = []
        with open(self.f.name) as f:
            for line in f:
                parts = [x.strip() for x in line.split(",")]
                if len(parts) >= 7:
                    try:
                        ts = datetime.datetime.strptime(parts[0], "%Y/%m/%d %H:%M:%S.%f")
                    except ValueError:
                        continue
                    if getattr(self, "t0", None) is None or self.t0 <= ts <= t1:
                        rows.append(parts[1:])
        os.unlink(self.f.name)
        if not rows:
            return None
        sm = [float(r[0]) for r in rows if r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in rows if r[1].replace(".", "").isdigit()]
        names = [n for n, _ in self.REASONS]
        reasons = sorted({names[k] for r in rows for k in range(4) if r[2 + k].lower().startswith("active")})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(rows), "source": "nvidia-smi, 100 ms"}


# ---------------------------------------------------------------------------------------------
# oracle timings (cpu_baseline leg and --impl reference): the oracle as it stands, host cores
# ---------------------------------------------------------------------------------------------
def oracle_sample(name, n_img=1, kf_blocks=1, seed=99):
    """Bounded sample of one minibatch step: the oracle's nets (1 energy + 4 force gradients) on
    `n_img` images and its Kalman update on `kf_blocks` blocks; extrapolated to a full step of the
    workload (nets scale with images, Kalman with sum n_i^2 over all blocks, 5 updates per step)."""
    import torch
    import oracle as O
    wl = get_config(name)
    m, opt = wl.model, wl.opt
    ds = make_dataset(name, n_img, seed=seed)
    na = len(ds["types"])
    w = init_weights(m, 3, float(ds["energy"].mean() / na))
    sizes = [int(np.prod(s)) for _, s in O.param_tensors(m)]
    blocks = O.block_split(sizes, opt.block_size)
    groups = force_groups(na, 0, 5)
    t0 = time.perf_counter()
    nl = O.build_nlist(ds["coord"], ds["box"], ds["types"], m.rcut, m.sel)
    O.energy_grad(w, ds["coord"], ds["box"], ds["types"], nl[0], nl[1], ds["energy"], m)
    for a in groups:
        O.force_grad(w, ds["coord"], ds["box"], ds["types"], nl[0], nl[1], ds["force"], a, m)
    t_nets = time.perf_counter() - t0
    big = sorted(blocks)[::-1][:kf_blocks]
    st = O.FEKF(np.zeros(sum(big)), big, lam=opt.lambda0, nu=opt.nu)
    st.P = [np.eye(n) for n in big]
    rng = np.random.default_rng(1)
    t0 = time.perf_counter()
    st.update(rng.standard_normal(sum(big)), 0.1, wl.batch)
    t_kf = time.perf_counter() - t0
    frac = sum(n * n for n in big) / sum(n * n for n in blocks)
    step_s = t_nets * wl.batch / n_img + 5 * t_kf / frac
    return {"step_s": step_s, "t_nets": t_nets, "t_kf": t_kf, "cores": torch.get_num_threads(),
            "sample": f"oracle nets (1 E + 4 F gradients) on {n_img} image(s) + oracle Kalman update on "
                      f"{kf_blocks} of {len(blocks)} P blocks ({big[0]}^2), extrapolated to {wl.batch} images and "
                      f"5 updates over all blocks"}


FP64_PEAK_TFLOPS = 37.1   # measured DMMA rate (tools/fp64_peak.cu on this pool's B200, round 1); guide-derived
                          # 148 SMs x 64 DFMA/clk x 2 x 1.965 GHz = 37.2
# fp32 nets: the rate of their contraction primitive, the fp32-accurate 8x8x4 product from two
# mma.sync.m16n8k4 tf32 (real.cuh), measured by tools/fp32_peak.cu on this pool's B200
# (mma.sync.m16n8k4 tf32 measured at 138.5 TFLOP/s; an fp32-accurate 8x8x4 product takes two of them = the
# four hi/lo products: 138.5 / 4 = 34.6; the microbench's loop, which re-splits its operands every product,
# reaches 24.5).  FP32 FFMA measured 71.5 TFLOP/s.
FP32_SPLIT_PEAK_TFLOPS = 34.6
FP32_PEAK_SOURCE = "measured mma.sync tf32 rate / 4 split products (tools/fp32_peak.cu)"


def nets_work(m, nl_j, types, groups):
    """Executed FLOPs of the nets in one minibatch step (1 energy + len(groups) force updates), counted
    from the step's own neighbour list: GEMM work as 2 flops per multiply-add over the VALID rows only
    (n_v per type pair), the force updates' tangent / restricted rows over the ACTIVE rows only (rows
    whose centre or neighbour is a selected atom).  Elementwise work (tanh, adjoint products) is counted
    separately as tanh evaluations.  nl_j [B][Na][N_m] (int), types [Na]."""
    nl_j = np.asarray(nl_j)
    types = np.asarray(types)
    B, na, _ = nl_j.shape
    sec = np.concatenate([[0], np.cumsum(m.sel)]).astype(int)
    d = list(m.emb)
    din = [1] + d[:-1]
    fwd_row = 2 * sum(a * b for a, b in zip(din, d))
    dg_row = 2 * sum(a * b for a, b in zip(din[1:], d[1:]))
    wg_row = 2 * sum((a + 1) * b for a, b in zip(din, d))
    M, M2 = m.emb[-1], m.m2
    desc_row = 2 * 4 * M                 # X += R~^T G (per row), reverse: Gbar and dR~ (x2)
    desc_atom = 2 * 4 * M * M2           # D = X^T X^<, reverse Eq. 4 (x2)
    h = [M * M2] + list(m.fit)
    fit_fwd = 2 * (sum(a * b for a, b in zip(h[:-1], h[1:])) + h[-1])
    fit_dg = fit_fwd
    fit_wg = 2 * (sum((a + 1) * b for a, b in zip(h[:-1], h[1:])) + h[-1] + 1)
    valid = nl_j >= 0
    N = int(valid.sum())                  # valid embedding rows (all pairs)
    F = B * na                            # fitting rows
    fl = 0.0
    # energy update: forward, full reverse with weight gradients
    fl += N * (fwd_row + desc_row) + F * (desc_atom + fit_fwd)
    fl += F * (fit_dg + fit_wg + 2 * desc_atom) + N * (dg_row + wg_row + 2 * desc_row)
    T_all = []
    for g in groups:
        sel = np.zeros(na, bool)
        sel[np.asarray(g)] = True
        j = np.where(valid, nl_j, 0)
        act = valid & (sel[None, :, None] | sel[j])
        T = int(act.sum())
        T_all.append(T)
        fl += N * (fwd_row + desc_row) + F * (desc_atom + fit_fwd)                  # primal forward
        fl += F * (fit_dg + 2 * desc_atom) + T * (dg_row + 2 * desc_row)          # forces on S_k (restricted)
        fl += T * (fwd_row + 2 * desc_row) + F * (2 * desc_atom + fit_fwd)        # tangent forward
        fl += 2 * F * (fit_dg + fit_wg) + F * 4 * desc_atom                       # dual reverse, fitting
        fl += (N + T) * (dg_row + wg_row) + (N + T) * 2 * desc_row                 # dual reverse, embedding
    ng = len(groups)
    tanh = (N * sum(d) + F * sum(m.fit)) * (1 + ng)      # primal forwards only (tangent rows reuse y)
    return {"flops_per_step": fl, "valid_rows": N, "padded_slots": int(nl_j.size), "fitting_rows": F,
            "active_rows_per_force_update": (sum(T_all) / max(ng, 1)), "tanh_per_step": int(tanh)}


def run_reference(args, rank, world):
    if rank != 0:
        return
    wl = get_config(args.config)
    vals = []
    info = None
    for k in range(args.warmup + args.steps):
        info = oracle_sample(args.config, n_img=1, kf_blocks=1, seed=1000 + k)
        if k >= args.warmup:
            vals.append(wl.batch / info["step_s"])
    v = statistics.median(vals)
    out = {"impl": "reference", "metric": METRIC, "value": v, "unit": "images/s", "n_gpus": args.gpus,
           "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1000.0 * wl.batch / v, "higher_is_better": True,
           "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic (seeded LJ-labelled lattices)",
           "config": {"workload": args.config, "images_per_step": wl.batch},
           "cpu_baseline": {"value": v, "unit": "images/s", "cores": info["cores"], "kind": "oracle",
                            "sample": info["sample"]},
           "e2e": {"value": v, "unit": "images/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(out), flush=True)


# ---------------------------------------------------------------------------------------------
# the CUDA path
# ---------------------------------------------------------------------------------------------
def run_fekf(args, rank, world, local):
    import torch
    import torch.distributed as dist
    import paper_conf_ppopp_huzslmlwtj24_b200 as fk

    torch.cuda.set_device(local)
    wl = get_config(args.config)
    m, opt = wl.model, wl.opt
    over = {"precision": args.precision, "p_mode": args.p_mode, "net_precision": args.net_precision}
    if args.p_defer is not None:
        over["p_defer"] = args.p_defer
    opt = type(opt)(**{**opt.__dict__, **over})
    B = wl.batch
    Bg = B * world
    net_prec = args.net_precision or args.precision
    ds = make_dataset(args.config, 2 * B, seed=wl.seed + 1000 * rank)
    na = len(ds["types"])
    w0 = init_weights(m, 3, float(make_dataset(args.config, 4, seed=wl.seed)["energy"].mean() / na))
    comm = fk.Comm.from_process_group() if world > 1 else None
    ctx = fk.Context(m, opt, types=ds["types"], local_batch=B, global_batch=Bg, comm=comm)
    ctx.set_params(torch.as_tensor(w0).cuda())
    nsteps = args.warmup + args.steps
    dev = lambda x, dt=torch.float64: torch.as_tensor(np.ascontiguousarray(x)).to(dt).cuda()
    coord = [dev(ds["coord"][h * B:(h + 1) * B]) for h in range(2)]
    box = [dev(ds["box"][h * B:(h + 1) * B]) for h in range(2)]
    elab = [dev(ds["energy"][h * B:(h + 1) * B]) for h in range(2)]
    flab = [dev(ds["force"][h * B:(h + 1) * B]) for h in range(2)]
    gidx = np.stack([force_groups(na, s, wl.seed, opt.force_groups, opt.atoms_per_group) for s in range(nsteps)])
    fidx = dev(gidx, torch.int32)
    metrics = torch.zeros(8, dtype=torch.float64, device="cuda")

    def barrier():
        if world > 1:
            dist.barrier()

    def step(s):
        h = s % 2
        ctx.train_step(coord[h], box[h], elab[h], flab[h], fidx[s], metrics)

    clocks = Clocks(local)
    for s in range(args.warmup):
        step(s)
    torch.cuda.synchronize()
    barrier()
    clocks.mark()
    ctx.kf.timing(True)
    stream = torch.cuda.current_stream()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    barrier()
    torch.cuda.synchronize()
    e0.record(stream)
    for s in range(args.warmup, nsteps):
        step(s)
    e1.record(stream)
    torch.cuda.synchronize()
    barrier()
    pass_ms, pass_n, pass_rw = ctx.kf.timing(False)
    parts = ctx.kf.timing_parts()
    span_ms = ctx.kf.timing_span()
    clk = clocks.stop()
    ms = e0.elapsed_time(e1)
    launches = ctx.last_launch_count() * args.steps
    met = metrics.cpu().numpy()
    if world > 1:
        t = torch.tensor([ms, pass_ms / max(pass_n, 1)], dtype=torch.float64, device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t[0])
    value = Bg * args.steps / (ms / 1000.0)

    # ---- end to end through the public API with host buffers (pinned), copies inside the timed region
    e2e = None
    if not args.no_e2e:
        pin = lambda x, dt=torch.float64: torch.as_tensor(np.ascontiguousarray(x)).to(dt).pin_memory()
        hc = [pin(ds["coord"][h * B:(h + 1) * B]) for h in range(2)]
        hb = [pin(ds["box"][h * B:(h + 1) * B]) for h in range(2)]
        he = [pin(ds["energy"][h * B:(h + 1) * B]) for h in range(2)]
        hf = [pin(ds["force"][h * B:(h + 1) * B]) for h in range(2)]
        hi = pin(gidx, torch.int32)
        dc, db, de, df = (torch.empty_like(coord[0]), torch.empty_like(box[0]), torch.empty_like(elab[0]),
                          torch.empty_like(flab[0]))
        di = torch.empty_like(fidx[0])
        hm = torch.empty(8, dtype=torch.float64).pin_memory()
        h2d = (hc[0].numel() + hb[0].numel() + he[0].numel() + hf[0].numel()) * 8 + hi[0].numel() * 4
        d2h = 8 * 8
        barrier()
        torch.cuda.synchronize()
        t0 = torch.cuda.Event(enable_timing=True)
        t1 = torch.cuda.Event(enable_timing=True)
        t0.record(stream)
        for s in range(args.warmup, nsteps):
            h = s % 2
            dc.copy_(hc[h], non_blocking=True)
            db.copy_(hb[h], non_blocking=True)
            de.copy_(he[h], non_blocking=True)
            df.copy_(hf[h], non_blocking=True)
            di.copy_(hi[s], non_blocking=True)
            ctx.train_step(dc, db, de, df, di, metrics)
            hm.copy_(metrics, non_blocking=True)
            stream.synchronize()
        t1.record(stream)
        torch.cuda.synchronize()
        barrier()
        ems = t0.elapsed_time(t1)
        if world > 1:
            t = torch.tensor([ems], dtype=torch.float64, device="cuda")
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            ems = float(t[0])
        e2e = {"value": Bg * args.steps / (ems / 1000.0), "unit": "images/s", "h2d_bytes_per_step": h2d,
               "d2h_bytes_per_step": d2h}

    # ---- roofline of the dominant kernel (the P pass), measured live in the timed region
    info = ctx.kf.info()
    blocks = ctx.kf.blocks
    nt = [(n + 63) // 64 for n in blocks]
    total_tiles = sum(x * (x + 1) // 2 for x in nt)
    # algorithmic bytes of one stream over this rank's share of the symmetric blocks: 8 * n(n+1)/2 each;
    # a read-write pass (the one that rewrites P) moves it twice, a read-only pass once
    esize = 8 if args.precision == 64 else 4
    stream = esize / 2 * sum(n * (n + 1) for n in blocks) * info["tiles_local"] / total_tiles
    alg_total = stream * (2 * pass_rw + (pass_n - pass_rw))
    alg_bytes = alg_total / max(pass_n, 1)
    # a split pass is two overlapping launches (early on the side stream, late on the producing one); the
    # pass's duration is its wall span (early start -> later end), the launch-duration sum double-counts
    # the overlap and is reported beside it
    avg_pass_s = (span_ms / max(pass_n, 1)) / 1000.0
    peak, peak_kind = load_peaks()
    achieved = alg_total / (span_ms / 1000.0) / 1e9 if span_ms > 0 else None
    achieved_sum = alg_total / (pass_ms / 1000.0) / 1e9 if pass_ms > 0 else None
    traffic = None
    prof = os.path.join(ROOT, "profiles", "kf_pass_traffic.json")
    if os.path.exists(prof) and pass_n > 0:
        try:
            with open(prof) as f:
                pj = json.load(f)
            pp = pj.get("by_precision", {}).get(str(args.precision))
            if pj.get("workload") == args.config and world == 1 and pp:
                # DRAM bytes per launch from ncu captures, scaled to this run's algorithmic bytes and blended
                # over its read-only / read-write launches
                ro = pp["ro_dram_bytes_per_launch"] / pp["ro_alg_bytes_per_launch"]
                rwr = pp["rw_dram_bytes_per_launch"] / pp["rw_alg_bytes_per_launch"]
                traffic = (stream * ro * (pass_n - pass_rw) + 2 * stream * rwr * pass_rw) / pass_n
        except Exception:
            pass
    # the same kernel alone (one read-only pass over the whole P on every SM, after the timed region): in
    # the step the fitting blocks' pass shares the GPU with the tail of the reverse pass (split pass), so
    # the live figure above includes that contention
    standalone = None
    if world == 1 and pass_n > 0:
        gs = torch.randn(ctx.n_params, dtype=torch.float64, device="cuda")
        ctx.kf.pass_only(gs)
        torch.cuda.synchronize()
        ctx.kf.timing(True)
        for _ in range(3):
            ctx.kf.pass_only(gs)
        torch.cuda.synchronize()
        sa_ms, sa_n, _ = ctx.kf.timing(False)
        sa = stream / (sa_ms / sa_n / 1000.0) / 1e9
        standalone = {"achieved": sa, "frac": sa / peak, "avg_launch_ms": sa_ms / sa_n, "launches": sa_n,
                      "pass": "read-only, all SMs"}
        del gs
    # ---- nets roofline: the step's nets work (E Jacobian + force_groups force Jacobians, the same kernels
    # the step runs, on all SMs, eager launches on this stream) against the fp64 DMMA peak
    nets = None
    try:
        nj, _, _ = ctx.build_nlist(coord[0], box[0])
        s0 = nsteps - 1
        work = nets_work(m, nj.cpu().numpy(), ds["types"], gidx[s0])
        torch.cuda.synchronize()
        reps = 3
        n0, n1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        cs = torch.cuda.current_stream()
        for r in range(reps + 1):
            if r == 1:
                n0.record(cs)
            ctx.energy_jacobian(coord[0], box[0], elab[0])
            for k in range(opt.force_groups):
                ctx.force_jacobian(coord[0], box[0], flab[0], fidx[s0][k])
        n1.record(cs)
        torch.cuda.synchronize()
        nets_ms = n0.elapsed_time(n1) / reps
        tf = work["flops_per_step"] / (nets_ms / 1000.0) / 1e12
        if net_prec == 32:
            npk, nsrc, nbound = FP32_SPLIT_PEAK_TFLOPS, FP32_PEAK_SOURCE, "fp32 (split-tf32 tensor products)"
        else:
            npk, nsrc, nbound = FP64_PEAK_TFLOPS, "measured DMMA (tools/fp64_peak.cu)", "fp64"
        nets = {"kernels": "emb_fwd/emb_bwd/dgemm/desc_* (E + %d F Jacobians)" % opt.force_groups, "bound": nbound,
                "achieved": tf, "peak": npk, "unit": "TFLOP/s", "frac": tf / npk,
                "peak_source": nsrc, "ms_per_step_alone": nets_ms,
                "share_of_step_if_serial": nets_ms / (ms / args.steps), **work}
    except Exception as e:   # instrumentation only: never lose the bench line over it
        nets = {"error": str(e)[:200]}
    split_sms = int(os.environ.get("FEKF_SPLIT_SMS", "96" if args.precision == 64 else "80"))
    f_local = info["tiles_local"] / total_tiles
    if "FEKF_SPLIT_SMS" not in os.environ and f_local < 0.999 and split_sms > 0:
        # the library's rule for a rank streaming a fraction f of a sharded P (api.cu, Ctx::init)
        nsm = torch.cuda.get_device_properties(local).multi_processor_count
        s1 = min(split_sms, nsm - 1)
        split_sms = max(8, round(nsm * f_local / (f_local + (nsm - s1) / s1)))
    roof = {"kernel": "kf_pass_kernel", "bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
            "frac": (achieved / peak) if achieved else None, "traffic": traffic,
            "peak_source": peak_kind, "alg_bytes_per_launch": alg_bytes, "avg_launch_ms": avg_pass_s * 1000.0,
            "duration": "wall span per pass (split pass: early launch start -> later launch end), CUDA events",
            "achieved_launch_sum": achieved_sum, "frac_launch_sum": (achieved_sum / peak) if achieved_sum else None,
            "launches_timed": pass_n, "rw_launches": pass_rw, "share_of_step": (span_ms / max(ms, 1e-9)),
            "split_pass_early_sms": split_sms, "split_updates": "energy and force updates" if os.environ.get("FEKF_SPLIT_E", "1") != "0" else "force updates",
            "standalone": standalone,
            "split_ms_per_pass": dict(zip(["early", "late", "early_start_to_reverse_done"],
                                          [x / max(pass_n, 1) for x in parts]))}

    out = {"metric": METRIC, "value": value, "unit": "images/s", "n_gpus": world, "steps": args.steps,
           "warmup": args.warmup, "ms_per_step": ms / args.steps, "higher_is_better": True, "scaling": "weak",
           "vs_baseline": None, "dtype": {(64, 64): "f64", (32, 32): "f32", (32, 64): "f64 nets / f32 P",
                                           (64, 32): "f32 nets / f64 P"}[(args.precision, net_prec)],
           "data": "synthetic (seeded perturbed %s snapshots, LJ labels)" % wl.system.name,
           "config": {"workload": args.config, "images_per_gpu": B, "global_batch": Bg, "n_atoms": na,
                      "n_params": ctx.n_params, "p_blocks": len(blocks), "p_bytes_per_gpu": info["p_bytes_local"],
                      "parallelism": f"dp{world}" + ((" + P replicated" if args.p_mode else " + P sharded") if world > 1 else ""),
                      "p_precision": args.precision, "net_precision": net_prec, "p_defer": opt.p_defer,
                      "l2": "inputs larger than L2: P (%.1f GiB packed) is streamed 5x per step"
                            % (info["p_bytes_local"] / 2**30)},
           "roofline": roof, "roofline_nets": nets, "e2e": e2e, "gpu_launches": int(launches), "clocks": clk,
           "last_metrics": {"abe_e": met[0], "abe_f": list(met[1:5]), "A_last": met[5], "lambda": met[6],
                            "flags": met[7]}}
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cb = oracle_sample(args.config, n_img=2, kf_blocks=2)
        out["cpu_baseline"] = {"value": wl.batch / cb["step_s"], "unit": "images/s", "cores": cb["cores"],
                               "kind": "oracle", "sample": cb["sample"]}
    if rank == 0:
        print(json.dumps(out), flush=True)
    ctx.close()
    if comm:
        comm.close()


def main():
    args = parse()
    rank, world, local = dist_env()
    if args.impl == "reference":
        run_reference(args, rank, world)
        return
    if world > 1:
        import torch
        import torch.distributed as dist
        torch.cuda.set_device(local)
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    run_fekf(args, rank, world, local)
    if world > 1:
        import torch.distributed as dist
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
