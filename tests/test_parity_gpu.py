"""GPU parity: the CUDA path (through the C ABI) against the fp64 CPU oracle on the same seeded inputs.

Tolerances (north_star): neighbour lists / indices bit-exact; descriptor, energy, force rel 1e-12;
weights and P after 10 EKF steps rel 1e-9.  "rel" is normwise: max|gpu - ref| / max|ref| per tensor
(reading Z19).  Jacobians: rel 1e-11.
"""
import os

import numpy as np
import pytest
import torch

import oracle as O
from fixtures import get_config, make_dataset, init_weights, force_groups

pytestmark = pytest.mark.gpu

fk = pytest.importorskip("paper_conf_ppopp_huzslmlwtj24_b200")


def rel(a, b):
    a = np.asarray(a, dtype=np.float64)
    b = np.asarray(b, dtype=np.float64)
    den = np.abs(b).max()
    return float(np.abs(a - b).max() / (den if den > 0 else 1.0))


def elem_rel(a, b, floor=1e-6):
    """Element-wise relative error down to `floor` of the tensor's scale: max_i |a_i - b_i| / max(|b_i|,
    floor max|b|) (the normwise rel above lets small entries such as P's off-diagonal drift)."""
    a = np.asarray(a, dtype=np.float64)
    b = np.asarray(b, dtype=np.float64)
    scale = np.abs(b).max()
    if scale == 0:
        return float(np.abs(a).max())
    return float((np.abs(a - b) / np.maximum(np.abs(b), floor * scale)).max())


def cu(x, dtype=torch.float64):
    return torch.as_tensor(np.ascontiguousarray(x)).to(dtype).cuda()


@pytest.fixture(scope="module", autouse=True)
def _gpu():
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    fk.lib()


def _setup(name, nb, sel=None, seed=3):
    wl = get_config(name)
    m = wl.model
    if sel is not None:
        m = type(m)(**{**m.__dict__, "sel": sel})
    ds = make_dataset(name, nb)
    w = init_weights(m, seed, float(ds["energy"].mean() / len(ds["types"])))
    ctx = fk.Context(m, wl.opt, types=ds["types"], local_batch=nb, global_batch=nb)
    ctx.set_params(cu(w))
    return wl, m, ds, w, ctx


CASES = [("t2_tiny", 3), ("c1_cu32", 4), ("paper_cu108", 2), ("c2_water64", 2)]


@pytest.mark.parametrize("name,nb", CASES)
def test_nlist_bit_exact(name, nb):
    wl, m, ds, w, ctx = _setup(name, nb)
    nj, ns, ov = ctx.build_nlist(cu(ds["coord"]), cu(ds["box"]))
    rj, rs, rov = O.build_nlist(ds["coord"], ds["box"], ds["types"], m.rcut, m.sel)
    assert np.array_equal(nj.cpu().numpy(), rj)
    assert np.array_equal(ns.cpu().numpy(), rs)
    assert np.array_equal(ov.cpu().numpy(), rov)


def test_nlist_overflow_bit_exact():
    wl, m, ds, w, ctx = _setup("t2_tiny", 3, sel=[5, 9])
    nj, ns, ov = ctx.build_nlist(cu(ds["coord"]), cu(ds["box"]))
    rj, rs, rov = O.build_nlist(ds["coord"], ds["box"], ds["types"], m.rcut, [5, 9])
    assert rov.sum() > 0
    assert np.array_equal(nj.cpu().numpy(), rj) and np.array_equal(ns.cpu().numpy(), rs)
    assert np.array_equal(ov.cpu().numpy(), rov)


@pytest.mark.parametrize("name,nb", CASES)
def test_env_mat(name, nb):
    wl, m, ds, w, ctx = _setup(name, nb)
    rj, rs, _ = O.build_nlist(ds["coord"], ds["box"], ds["types"], m.rcut, m.sel)
    em, jac, rij = ctx.env_mat(cu(ds["coord"]), cu(ds["box"]), cu(rj, torch.int32), cu(rs, torch.int32))
    d, R, mask = O.env_mat(torch.as_tensor(ds["coord"]), ds["box"], rj, rs, m.rcut, m.rcut_smth)
    assert rel(rij.cpu(), d) < 1e-14
    assert rel(em.cpu(), R) < 1e-12
    # J = dR~/dd by autograd on the oracle's R~(d)
    dl = d.detach().clone().requires_grad_(True)
    rows = O.env_rows(dl, mask, m.rcut, m.rcut_smth)
    J = torch.stack([torch.autograd.grad(rows[..., k].sum(), dl, retain_graph=True)[0] for k in range(4)], dim=-2)
    assert rel(jac.cpu(), J) < 1e-12


@pytest.mark.parametrize("name,nb", CASES)
def test_forward_energy_force_virial(name, nb):
    wl, m, ds, w, ctx = _setup(name, nb)
    ea, e, f, v = ctx.forward(cu(ds["coord"]), cu(ds["box"]))
    rj, rs, _ = O.build_nlist(ds["coord"], ds["box"], ds["types"], m.rcut, m.sel)
    Ea, E, F, V = O.energy_force_virial(w, ds["coord"], ds["box"], ds["types"], rj, rs, m)
    assert rel(ea.cpu(), Ea) < 1e-12
    assert rel(e.cpu(), E) < 1e-12
    assert rel(f.cpu(), F) < 1e-12
    assert rel(v.cpu().reshape(-1, 3, 3), V) < 1e-12


@pytest.mark.parametrize("name,nb", CASES)
def test_energy_jacobian(name, nb):
    wl, m, ds, w, ctx = _setup(name, nb)
    g, s = ctx.energy_jacobian(cu(ds["coord"]), cu(ds["box"]), cu(ds["energy"]))
    rj, rs, _ = O.build_nlist(ds["coord"], ds["box"], ds["types"], m.rcut, m.sel)
    gr, sr, _ = O.energy_grad(w, ds["coord"], ds["box"], ds["types"], rj, rs, ds["energy"], m)
    assert rel(g.cpu(), gr) < 1e-11
    assert elem_rel(g.cpu(), gr, 1e-3) < 1e-9
    assert abs(float(s.cpu()[0]) - sr) <= 1e-13 * max(1.0, abs(sr))


@pytest.mark.parametrize("name,nb", CASES)
def test_force_jacobian(name, nb):
    wl, m, ds, w, ctx = _setup(name, nb)
    atoms = force_groups(len(ds["types"]), 0, 5)[0]
    g, s = ctx.force_jacobian(cu(ds["coord"]), cu(ds["box"]), cu(ds["force"]), cu(atoms, torch.int32))
    rj, rs, _ = O.build_nlist(ds["coord"], ds["box"], ds["types"], m.rcut, m.sel)
    gr, sr, _ = O.force_grad(w, ds["coord"], ds["box"], ds["types"], rj, rs, ds["force"], atoms, m)
    assert rel(g.cpu(), gr) < 1e-11 and elem_rel(g.cpu(), gr, 1e-3) < 1e-9
    assert abs(float(s.cpu()[0]) - sr) <= 1e-12 * max(1.0, abs(sr))


def _rand_spd(rng, n):
    a = rng.standard_normal((n, n))
    return a @ a.T / n + np.eye(n)


@pytest.mark.parametrize("blocks", [[5, 70, 130], [64], [1, 200, 127, 65]])
@pytest.mark.parametrize("noise_mode,p_defer", [(0, 5), (1, 1), (0, 3), (1, 8), (0, 16)])
def test_kalman_updates(blocks, noise_mode, p_defer):
    rng = np.random.default_rng(7)
    opt = dict(lambda0=0.98, nu=0.9987, block_size=1024, noise_mode=noise_mode, p_defer=p_defer)
    kf = fk.KalmanFilter(blocks, opt)
    N = sum(blocks)
    st = O.FEKF(np.zeros(N), blocks, lam=0.98, nu=0.9987, noise_mode=noise_mode)
    st.P = [_rand_spd(rng, n) for n in blocks]
    for b, P in enumerate(st.P):
        kf.set_block(b, cu(P))
    w = torch.zeros(N, dtype=torch.float64, device="cuda")
    for it in range(max(10, p_defer + 4)):   # at least one read-write pass
        g = rng.standard_normal(N)
        abe = float(rng.uniform(0.01, 1.0))
        kf.update(cu(g), cu([abe]), 3.0, w)
        st.update(g, abe, 9)
    torch.cuda.synchronize()
    assert rel(w.cpu(), st.w) < 1e-12 and elem_rel(w.cpu(), st.w) < 1e-9
    for b in range(len(blocks)):
        Pb = kf.get_block(b).cpu()
        assert rel(Pb, st.P[b]) < 1e-12 and elem_rel(Pb, st.P[b]) < 1e-9
    assert abs(kf.state()["lambda"] - st.lam) < 1e-15
    kf.flush()
    for b in range(len(blocks)):
        assert rel(kf.get_block(b).cpu(), st.P[b]) < 1e-12


@pytest.mark.parametrize("blocks", [[5, 70, 130], [1, 200, 127, 65]])
@pytest.mark.parametrize("p_defer", [1, 5, 16])
def test_kalman_updates_fp32(blocks, p_defer):
    """fp32 variant (P stored fp32, reading Z22) against the fp64 oracle: rel 1e-4 (north_star)."""
    rng = np.random.default_rng(11)
    opt = dict(lambda0=0.98, nu=0.9987, block_size=1024, noise_mode=0, p_defer=p_defer, precision=32)
    kf = fk.KalmanFilter(blocks, opt)
    assert kf.info()["p_bytes_local"] == 4 * 64 * 64 * sum((x + 1) * x // 2 for x in [(n + 63) // 64 for n in blocks])
    N = sum(blocks)
    st = O.FEKF(np.zeros(N), blocks, lam=0.98, nu=0.9987, noise_mode=0)
    st.P = [_rand_spd(rng, n) for n in blocks]
    for b, P in enumerate(st.P):
        kf.set_block(b, cu(P))
    w = torch.zeros(N, dtype=torch.float64, device="cuda")
    for it in range(max(10, p_defer + 4)):
        g = rng.standard_normal(N)
        abe = float(rng.uniform(0.01, 1.0))
        kf.update(cu(g), cu([abe]), 3.0, w)
        st.update(g, abe, 9)
    torch.cuda.synchronize()
    assert rel(w.cpu(), st.w) < 1e-4
    for b in range(len(blocks)):
        assert rel(kf.get_block(b).cpu(), st.P[b]) < 1e-4
    kf.flush()
    for b in range(len(blocks)):
        Pb = kf.get_block(b).cpu().numpy()
        assert rel(Pb, st.P[b]) < 1e-4
        assert np.array_equal(Pb, Pb.T)


@pytest.mark.parametrize("precision", [64, 32])
def test_kalman_full_size_sampled_blocks(precision):
    """Bench-size Kalman filter (water-64: 110 blocks, 39 GiB packed P, default p_defer): one update
    checked on sampled blocks against the update recomputed in numpy from the GPU's previous P
    (P_new = (P - A u u^T)/lambda with u = P g per block; w increment sqrt(bs) ABE A u)."""
    wl = get_config("c2_water64")
    _, blocks = fk.plan_layout(wl.model, wl.opt.block_size)
    assert len(blocks) == 110
    kf = fk.KalmanFilter(blocks, dict(block_size=wl.opt.block_size, precision=precision))
    tol = 1e-11 if precision == 64 else 1e-6   # fp32: the stored P_new is rounded to fp32 (rel 2^-24)
    N = sum(blocks)
    off = np.concatenate([[0], np.cumsum(blocks)])
    gen = torch.Generator(device="cuda").manual_seed(3)
    w = torch.zeros(N, dtype=torch.float64, device="cuda")
    abe = torch.full((1,), 0.05, dtype=torch.float64, device="cuda")
    for _ in range(wl.opt.p_defer + 2):   # crosses one read-write pass
        kf.update(torch.randn(N, dtype=torch.float64, device="cuda", generator=gen), abe, 4.0, w)
    sample = [0, 37, 109]
    before = {b: kf.get_block(b).cpu().numpy() for b in sample}
    lam = kf.state()["lambda"]
    w0 = w.cpu().numpy()
    g = torch.randn(N, dtype=torch.float64, device="cuda", generator=gen)
    kf.update(g, abe, 4.0, w)
    A = kf.state()["A"]
    assert np.isfinite(A) and A > 0
    gn, w1 = g.cpu().numpy(), w.cpu().numpy()
    for b in sample:
        sl = slice(off[b], off[b + 1])
        u = before[b] @ gn[sl]
        ref = (before[b] - A * np.outer(u, u)) / lam
        assert rel(kf.get_block(b).cpu(), ref) < tol
        assert rel(w1[sl] - w0[sl], 4.0 * 0.05 * A * u) < tol


@pytest.mark.parametrize("name,steps,precision", [("c1_cu32", 10, 64), ("t2_tiny", 4, 64), ("c1_cu32", 10, 32)])
def test_train_steps(name, steps, precision):
    """10 minibatch steps (50 KF updates, reading Z20): w and P within rel 1e-9 of the fp64 oracle; P stored
    fp32 over the fp64 nets within rel 1e-4 (north_star; the fp32 nets: test_parity_gpu_fp32.py)."""
    wl = get_config(name)
    m, opt = wl.model, wl.opt
    opt = type(opt)(**{**opt.__dict__, "precision": precision, "net_precision": 64})
    tol = 1e-9 if precision == 64 else 1e-4
    ds = make_dataset(name, wl.batch * 2)
    na = len(ds["types"])
    w0 = init_weights(m, 3, float(ds["energy"].mean() / na))
    B = wl.batch
    ctx = fk.Context(m, opt, types=ds["types"], local_batch=B, global_batch=B)
    ctx.set_params(cu(w0))
    st = O.FEKF.create(w0, m, opt)
    for step in range(steps):
        sl = slice((step % 2) * B, (step % 2) * B + B)
        groups = force_groups(na, step, 17, opt.force_groups, opt.atoms_per_group)
        met = ctx.train_step(cu(ds["coord"][sl]), cu(ds["box"][sl]), cu(ds["energy"][sl]), cu(ds["force"][sl]),
                             cu(groups, torch.int32))
        ref = O.train_step(st, ds["coord"][sl], ds["box"][sl], ds["types"], ds["energy"][sl], ds["force"][sl],
                           groups, m, opt)
        mt = met.cpu().numpy()
        assert abs(mt[0] - ref["abe_e"]) <= tol * abs(ref["abe_e"])
        np.testing.assert_allclose(mt[1:5], ref["abe_f"], rtol=tol)
        assert abs(mt[6] - ref["lambda"]) < 1e-14
        assert mt[7] == 0
    wg = ctx.get_params().cpu()
    assert rel(wg, st.w) < tol and elem_rel(wg, st.w) < 100 * tol
    for b, n in enumerate(st.blocks):
        Pb = ctx.kf.get_block(b).cpu()
        assert rel(Pb, st.P[b]) < tol and elem_rel(Pb, st.P[b]) < 100 * tol


@pytest.mark.parametrize("precision", [64, 32])
def test_train_steps_split_pass(precision):
    """The split P pass (one GPU: the force updates' fitting-block pass overlaps the reverse pass on a side
    stream; the late launch takes the embedding blocks, then steals the early launch's unclaimed items):
    c1_cu32 with N_b = 1024 has the embedding parameters in block 0 and fitting-only blocks after it, so
    the split is active.  8 minibatch steps in graph mode (crossing read-write passes, p_defer 3) match
    the oracle at rel 1e-9 (w, every block of P)."""
    wl = get_config("c1_cu32")
    m = wl.model
    opt = type(wl.opt)(**{**wl.opt.__dict__, "block_size": 1024, "p_defer": 3, "precision": precision})
    tol = 1e-9 if precision == 64 else 1e-4
    ds = make_dataset("c1_cu32", wl.batch * 2)
    na = len(ds["types"])
    w0 = init_weights(m, 3, float(ds["energy"].mean() / na))
    B = wl.batch
    _, blocks = fk.plan_layout(m, 1024)
    assert len(blocks) > 2
    ctx = fk.Context(m, opt, types=ds["types"], local_batch=B, global_batch=B)
    ctx.set_params(cu(w0))
    st = O.FEKF.create(w0, m, opt)
    ctx.kf.timing(True)
    for step in range(8):
        sl = slice((step % 2) * B, (step % 2) * B + B)
        groups = force_groups(na, step, 17, opt.force_groups, opt.atoms_per_group)
        ctx.train_step(cu(ds["coord"][sl]), cu(ds["box"][sl]), cu(ds["energy"][sl]), cu(ds["force"][sl]),
                       cu(groups, torch.int32))
        O.train_step(st, ds["coord"][sl], ds["box"][sl], ds["types"], ds["energy"][sl], ds["force"][sl],
                     groups, m, opt)
    torch.cuda.synchronize()
    ctx.kf.timing(False)
    parts = ctx.kf.timing_parts()
    assert parts[1] > 0.0            # late launches ran: the split was active
    assert rel(ctx.get_params().cpu(), st.w) < tol
    for b in range(len(st.blocks)):
        assert rel(ctx.kf.get_block(b).cpu(), st.P[b]) < tol


def test_step_graph_matches_eager():
    """a10: the captured step graph (default) and eager launches give bit-identical weights, P and metrics
    across graph variants (p_defer 2: read-write passes at different updates of a step) — every reduction in
    the step has a fixed order, the force scatter included (reverse neighbour map, no fp64 atomics) — and
    the live P-pass timing sees every pass inside replayed graphs."""
    wl = get_config("t2_tiny")
    m = wl.model
    opt = type(wl.opt)(**{**wl.opt.__dict__, "p_defer": 2})
    B = wl.batch
    ds = make_dataset("t2_tiny", B)
    na = len(ds["types"])
    w0 = init_weights(m, 3, float(ds["energy"].mean() / na))
    out = []
    for graph in (True, False):
        ctx = fk.Context(m, opt, types=ds["types"], local_batch=B, global_batch=B, graph=graph)
        ctx.set_params(cu(w0))
        ctx.kf.timing(True)
        mets = []
        for step in range(5):
            groups = force_groups(na, step, 17, opt.force_groups, opt.atoms_per_group)
            mets.append(ctx.train_step(cu(ds["coord"]), cu(ds["box"]), cu(ds["energy"]), cu(ds["force"]),
                                       cu(groups, torch.int32)).clone())
        ms, n, n_rw = ctx.kf.timing(False)
        npend, rw_expect = 0, 0
        for _ in range(25):                              # host mirror of the deferral rule
            rw = npend >= opt.p_defer
            rw_expect += rw
            npend = 1 if rw else npend + 1
        assert n == 25 and n_rw == rw_expect == 12 and ms > 0
        assert ctx.last_launch_count() > 50
        out.append((ctx.get_params().cpu(), [ctx.kf.get_block(b).cpu() for b in range(len(ctx.kf.blocks))],
                    torch.stack(mets).cpu()))
        ctx.close()
    assert torch.equal(out[0][0], out[1][0])
    assert all(torch.equal(a, b) for a, b in zip(out[0][1], out[1][1]))
    assert torch.equal(out[0][2], out[1][2])


@pytest.mark.parametrize("name,precision", [("c1_cu32", 64), ("t2_tiny", 64), ("t2_tiny", 32)])
def test_step_bit_reproducible(name, precision):
    """Two runs of the bench's model class (with the split pass: N_b 1024) give bit-identical weights, P,
    forces and metrics: no floating-point atomics anywhere in the step.  The second run launches the type
    pairs' embedding kernels one after another instead of side by side (FEKF_PAIR_STREAMS=0; the 2-type
    model has 4 pairs): concurrency changes no result either.  Both precisions."""
    wl = get_config(name)
    m = wl.model
    opt = type(wl.opt)(**{**wl.opt.__dict__, "block_size": 1024, "p_defer": 3, "precision": precision})
    B = wl.batch
    ds = make_dataset(name, B)
    na = len(ds["types"])
    w0 = init_weights(m, 3, float(ds["energy"].mean() / na))
    out = []
    for run in range(2):
        if run == 1:
            os.environ["FEKF_PAIR_STREAMS"] = "0"
        try:
            ctx = fk.Context(m, opt, types=ds["types"], local_batch=B, global_batch=B)
        finally:
            os.environ.pop("FEKF_PAIR_STREAMS", None)
        ctx.set_params(cu(w0))
        mets = [ctx.train_step(cu(ds["coord"]), cu(ds["box"]), cu(ds["energy"]), cu(ds["force"]),
                               cu(force_groups(na, s, 17), torch.int32)).clone() for s in range(4)]
        ea, e, f, v = ctx.forward(cu(ds["coord"]), cu(ds["box"]))
        out.append((ctx.get_params().cpu(), [ctx.kf.get_block(b).cpu() for b in range(len(ctx.kf.blocks))],
                    torch.stack(mets).cpu(), f.cpu(), v.cpu()))
        ctx.close()
    assert torch.equal(out[0][0], out[1][0]) and torch.equal(out[0][2], out[1][2])
    assert all(torch.equal(a, b) for a, b in zip(out[0][1], out[1][1]))
    assert torch.equal(out[0][3], out[1][3]) and torch.equal(out[0][4], out[1][4])


def test_rmse_trajectory_and_time_to_target():
    """Metric (iii), minutes to target RMSE (tests/golden/rmse_c1_cu32.json, written by
    tools/make_rmse_target.py from the oracle alone: S_o = 200 steps, target = the oracle's best test
    RMSE).  The GPU's trajectory follows the oracle's at rel 1e-9 up to the learning onset
    (step 56); from there on rounding differences grow by ~1e4 per 8 steps (2e-8 at step 64, 6e-3 at 72:
    the sign flips of Alg. 1 lines 3-4 amplify them), so the two runs are different samples of the same
    training; the GPU must reach the oracle's target within 1.5 S_o steps."""
    import json
    import os
    import sys
    sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(__file__)), "tools"))
    import time_to_rmse
    gold = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "rmse_c1_cu32.json")))
    out = time_to_rmse.run("c1_cu32", int(1.5 * gold["S_o"]), gold["every"], stop_at_target=True)
    assert out["flags"] == 0
    early = [d for s, d in out["dev_vs_oracle"] if s <= 56]
    assert len(early) == 8 and max(early) < 1e-9
    assert out["reached"] is not None and out["reached"]["step"] <= int(1.5 * gold["S_o"])


_C4_GOLD = sorted(f[5:-5] for f in os.listdir(os.path.join(os.path.dirname(__file__), "golden"))
                  if f.startswith("rmse_c4s_") and f.endswith(".json"))


@pytest.mark.parametrize("config", _C4_GOLD)
def test_c4_time_to_target(config):
    """Metric (iii) on the Table-3 systems (C4 small-batch variants, tests/golden/rmse_c4s_*.json: the
    oracle alone, S_o = 300 steps, every 20).  The GPU trajectory equals the oracle's at rel 1e-9 on the
    plateau before the learning onset (the oracle's RMSE still above 0.9 x its step-20 value) and through
    step 100 at most: rounding differences grow chaotically from there (NaCl-64, onset at step 240: 2e-11
    at step 100, 5e-9 at 180, 3e-7 at 220), as in the c1 test.  The GPU must reach the oracle's S_o-step
    RMSE within 1.5 S_o steps."""
    import json
    import sys
    sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(__file__)), "tools"))
    import time_to_rmse
    gold = json.load(open(os.path.join(os.path.dirname(__file__), "golden", f"rmse_{config}.json")))
    out = time_to_rmse.run(config, int(1.5 * gold["S_o"]), gold["every"], stop_at_target=True)
    assert out["flags"] == 0
    tr = gold["trajectory"]
    plateau = 0.9 * (tr[1][1] + tr[1][2])
    onset = next(s for s, e, f in tr[1:] if e + f < plateau)
    early = [d for s, d in out["dev_vs_oracle"] if s < min(onset, 120)]
    assert len(early) >= 4 and max(early) < 1e-9
    assert out["reached"] is not None and out["reached"]["step"] <= int(1.5 * gold["S_o"])


@pytest.mark.parametrize("world", [2, 3])
@pytest.mark.parametrize("precision", [64, 32])
def test_kalman_sharded_ranks(world, precision):
    """P sharded over `world` ranks (north_star; fekf_plan_shard tile-row segments) run in one process:
    each rank's filter streams only its own tiles, the partial u's are summed (the all-reduce the NCCL
    path does), and the weights and every block of P match the fp64 oracle after updates that cross
    read-write passes (rel 1e-12; fp32 P storage rel 1e-4)."""
    rng = np.random.default_rng(5)
    blocks = [5, 70, 130, 200, 64]
    opt = dict(lambda0=0.98, nu=0.9987, block_size=1024, noise_mode=0, p_defer=3, precision=precision)
    kfs = [fk.KalmanFilter(blocks, opt, shard=(world, r)) for r in range(world)]
    tiles = [kf.info()["tiles_local"] for kf in kfs]
    assert sum(tiles) == sum((x + 1) * x // 2 for x in [(n + 63) // 64 for n in blocks]) and min(tiles) > 0
    N = sum(blocks)
    st = O.FEKF(np.zeros(N), blocks, lam=0.98, nu=0.9987, noise_mode=0)
    st.P = [_rand_spd(rng, n) for n in blocks]
    for kf in kfs:
        for b, P in enumerate(st.P):
            kf.set_block(b, cu(P))
    ws = [torch.zeros(N, dtype=torch.float64, device="cuda") for _ in range(world)]
    for it in range(9):
        g = rng.standard_normal(N)
        abe = float(rng.uniform(0.01, 1.0))
        gd, ad = cu(g), cu([abe])
        for kf in kfs:
            kf.update_begin(gd)
        us = [kf.partial_u() for kf in kfs]
        tot = torch.stack(us).sum(0)
        for u in us:
            u.copy_(tot)
        for kf, w in zip(kfs, ws):
            kf.update_end(ad, 3.0, w)
        st.update(g, abe, 9)
    torch.cuda.synchronize()
    tol = 1e-12 if precision == 64 else 1e-4
    for w in ws:
        assert rel(w.cpu(), st.w) < tol
    for b, n in enumerate(blocks):
        full = torch.zeros(n, n, dtype=torch.float64, device="cuda")
        for kf in kfs:
            kf.get_block(b, out=full)           # each rank fills its own tiles (both triangles)
        assert rel(full.cpu(), st.P[b]) < tol


@pytest.mark.parametrize("p_mode", [0, 1])
def test_nccl_single_rank_step(p_mode):
    """a8 through NCCL on one GPU: a context built on a single-rank NCCL communicator (both all-reduces,
    [g || error sum] and the partial u, captured in the step graph; p_mode 1 = replicated P, no u
    exchange) trains exactly like one without."""
    wl = get_config("t2_tiny")
    m, opt = wl.model, wl.opt
    opt = type(opt)(**{**opt.__dict__, "p_mode": p_mode})
    B = wl.batch
    ds = make_dataset("t2_tiny", B)
    na = len(ds["types"])
    w0 = init_weights(m, 3, float(ds["energy"].mean() / na))
    comm = fk.Comm(0, 1, fk.Comm.unique_id())
    buf = torch.arange(5, dtype=torch.float64, device="cuda")
    comm.allreduce_sum(buf)
    torch.cuda.synchronize()
    assert torch.equal(buf.cpu(), torch.arange(5, dtype=torch.float64))
    outs = []
    for c in (comm, None):
        ctx = fk.Context(m, opt, types=ds["types"], local_batch=B, global_batch=B, comm=c)
        ctx.set_params(cu(w0))
        for step in range(3):
            groups = force_groups(na, step, 17, opt.force_groups, opt.atoms_per_group)
            met = ctx.train_step(cu(ds["coord"]), cu(ds["box"]), cu(ds["energy"]), cu(ds["force"]),
                                 cu(groups, torch.int32))
        assert met.cpu()[7] == 0
        outs.append(ctx.get_params().cpu())
        ctx.close()
    comm.close()
    assert rel(outs[0], outs[1]) < 1e-13


def test_rlekf_instance_by_instance():
    """batch size 1 (the RLEKF instance-by-instance schedule) on the same kernels:
    10 single-image minibatches (50 KF updates) against the oracle, rel 1e-9."""
    wl = get_config("c1_cu32")
    m, opt = wl.model, wl.opt
    ds = make_dataset("c1_cu32", 10)
    na = len(ds["types"])
    w0 = init_weights(m, 3, float(ds["energy"].mean() / na))
    ctx = fk.Context(m, opt, types=ds["types"], local_batch=1, global_batch=1)
    ctx.set_params(cu(w0))
    st = O.FEKF.create(w0, m, opt)
    for step in range(10):
        sl = slice(step, step + 1)
        groups = force_groups(na, step, 17, opt.force_groups, opt.atoms_per_group)
        met = ctx.train_step(cu(ds["coord"][sl]), cu(ds["box"][sl]), cu(ds["energy"][sl]), cu(ds["force"][sl]),
                             cu(groups, torch.int32))
        ref = O.train_step(st, ds["coord"][sl], ds["box"][sl], ds["types"], ds["energy"][sl], ds["force"][sl],
                           groups, m, opt)
        assert abs(met.cpu().numpy()[0] - ref["abe_e"]) <= 1e-9 * abs(ref["abe_e"])
    assert rel(ctx.get_params().cpu(), st.w) < 1e-9
    assert rel(ctx.kf.get_block(0).cpu(), st.P[0]) < 1e-9
    ctx.close()


def test_full_batch_water64_bench_config():
    """The bench's launch configuration (water-64, local_batch 32, 1 027 082 parameters, 41 GB of P)
    against the oracle: the energy and force Jacobians over all 32 images (rel 1e-11), the forward on
    sampled images (rel 1e-12), and the forces of the selected atoms a force update uses."""
    wl = get_config("c2_water64")
    m = wl.model
    B = wl.batch
    ds = make_dataset("c2_water64", B)
    na = len(ds["types"])
    w = init_weights(m, 3, float(ds["energy"].mean() / na))
    ctx = fk.Context(m, wl.opt, types=ds["types"], local_batch=B, global_batch=B)
    ctx.set_params(cu(w))
    X, BX = cu(ds["coord"]), cu(ds["box"])
    rj, rs, _ = O.build_nlist(ds["coord"], ds["box"], ds["types"], m.rcut, m.sel)
    g, s = ctx.energy_jacobian(X, BX, cu(ds["energy"]))
    gr, sr, _ = O.energy_grad(w, ds["coord"], ds["box"], ds["types"], rj, rs, ds["energy"], m)
    assert rel(g.cpu(), gr) < 1e-11
    assert abs(float(s.cpu()[0]) - sr) <= 1e-13 * max(1.0, abs(sr))
    atoms = force_groups(na, 3, wl.seed)[1]
    g, s = ctx.force_jacobian(X, BX, cu(ds["force"]), cu(atoms, torch.int32))
    gr, sr, _ = O.force_grad(w, ds["coord"], ds["box"], ds["types"], rj, rs, ds["force"], atoms, m)
    assert rel(g.cpu(), gr) < 1e-11
    assert abs(float(s.cpu()[0]) - sr) <= 1e-12 * max(1.0, abs(sr))
    ea, e, f, v = ctx.forward(X, BX)
    for b in (0, 17, 31):
        sl = slice(b, b + 1)
        Ea, E, F, V = O.energy_force_virial(w, ds["coord"][sl], ds["box"][sl], ds["types"], rj[sl], rs[sl], m)
        assert rel(e[sl].cpu(), E) < 1e-12
        assert rel(f[sl].cpu(), F) < 1e-12
        assert rel(v[sl].cpu().reshape(-1, 3, 3), V) < 1e-12
    ctx.close()


# ------------------------------------------------------------------------------------------
# Naive-EKF (Fig. 5; readings N1-N4): fekf_kf_update_naive and
# fekf_naive_train_step against oracle.NaiveEKF
# ------------------------------------------------------------------------------------------
@pytest.mark.parametrize("blocks", [[5, 70, 130], [64], [1, 200, 127, 65]])
@pytest.mark.parametrize("n", [1, 3, 8, 13, 32])
def test_naive_kalman_updates(blocks, n):
    """Rank-n updates over ragged blocks (tile tails, 1-element block, several tile rows), with FEKF
    updates in between so pending deferred corrections are flushed first: w, P, A_i rel 1e-12."""
    rng = np.random.default_rng(100 + n)
    opt = dict(lambda0=0.98, nu=0.9987, block_size=1024, noise_mode=0, p_defer=5)
    kf = fk.KalmanFilter(blocks, opt)
    N = sum(blocks)
    st = O.NaiveEKF(np.zeros(N), blocks, lam=0.98, nu=0.9987)
    st.P = [_rand_spd(rng, k) for k in blocks]
    for b, P in enumerate(st.P):
        kf.set_block(b, cu(P))
    w = torch.zeros(N, dtype=torch.float64, device="cuda")
    A_gpu = torch.zeros(n, dtype=torch.float64, device="cuda")
    for it in range(4):
        if it == 2:   # two FEKF updates: deferred corrections pending at the next naive update
            for _ in range(2):
                g = rng.standard_normal(N)
                kf.update(cu(g), cu([0.2]), 2.0, w)
                st.update(g, 0.2, 4)
        G = rng.standard_normal((n, N))
        abe = rng.uniform(0.01, 1.0, n)
        kf.update_naive(cu(G), cu(abe), w, A_gpu)
        A_ref = st.update_naive(list(G), list(abe))
        torch.cuda.synchronize()
        assert rel(A_gpu.cpu(), A_ref) < 1e-12
    assert rel(w.cpu(), st.w) < 1e-12
    for b in range(len(blocks)):
        assert rel(kf.get_block(b).cpu(), st.P[b]) < 1e-12
    assert abs(kf.state()["lambda"] - st.lam) < 1e-15


def test_naive_full_size_sampled_blocks():
    """Bench-size filter (water-64: 110 blocks, 39 GiB packed P), n = 32 samples: one naive update
    checked on sampled blocks against numpy from the GPU's previous P: u_i = P g_i per block,
    P_new = (P - sum_i (A_i/n) u_i u_i^T)/lambda, w += sum_i (ABE_i A_i / n) u_i."""
    wl = get_config("c2_water64")
    _, blocks = fk.plan_layout(wl.model, wl.opt.block_size)
    kf = fk.KalmanFilter(blocks, dict(block_size=wl.opt.block_size))
    N = sum(blocks)
    n = 32
    off = np.concatenate([[0], np.cumsum(blocks)])
    gen = torch.Generator(device="cuda").manual_seed(5)
    w = torch.zeros(N, dtype=torch.float64, device="cuda")
    abe = torch.rand(n, dtype=torch.float64, device="cuda", generator=gen) * 0.1
    A = torch.zeros(n, dtype=torch.float64, device="cuda")
    kf.update_naive(torch.randn(n, N, dtype=torch.float64, device="cuda", generator=gen) * 1e-2, abe, w, A)
    sample = [0, 55, 109]
    before = {b: kf.get_block(b).cpu().numpy() for b in sample}
    lam = kf.state()["lambda"]
    w0 = w.cpu().numpy()
    G = torch.randn(n, N, dtype=torch.float64, device="cuda", generator=gen) * 1e-2
    kf.update_naive(G, abe, w, A)
    Gn, An, ab, w1 = G.cpu().numpy(), A.cpu().numpy(), abe.cpu().numpy(), w.cpu().numpy()
    assert np.all(np.isfinite(An)) and np.all(An > 0)
    for b in sample:
        sl = slice(off[b], off[b + 1])
        U = before[b] @ Gn[:, sl].T                  # [n_b, n]
        ref = (before[b] - (U * (An / n)) @ U.T) / lam
        assert rel(kf.get_block(b).cpu(), ref) < 1e-11
        assert rel(w1[sl] - w0[sl], U @ (ab * An / n)) < 1e-11


@pytest.mark.parametrize("name,nb,steps", [("t2_tiny", 3, 2), ("c1_cu32", 4, 3)])
def test_naive_train_steps(name, nb, steps):
    """Naive-EKF minibatches through the C ABI (per-image Jacobians, rank-B updates) against
    oracle.naive_train_step: per-update ABE means, lambda, w and P."""
    wl = get_config(name)
    m, opt = wl.model, wl.opt
    ds = make_dataset(name, nb * 2)
    na = len(ds["types"])
    w0 = init_weights(m, 3, float(ds["energy"].mean() / na))
    ctx = fk.Context(m, opt, types=ds["types"], local_batch=nb, global_batch=nb)
    ctx.set_params(cu(w0))
    st = O.NaiveEKF.create(w0, m, opt)
    for step in range(steps):
        sl = slice((step % 2) * nb, (step % 2) * nb + nb)
        groups = force_groups(na, step, 17, opt.force_groups, opt.atoms_per_group)
        met = ctx.naive_train_step(cu(ds["coord"][sl]), cu(ds["box"][sl]), cu(ds["energy"][sl]),
                                   cu(ds["force"][sl]), cu(groups, torch.int32))
        ref = O.naive_train_step(st, ds["coord"][sl], ds["box"][sl], ds["types"], ds["energy"][sl],
                                 ds["force"][sl], groups, m)
        mt = met.cpu().numpy()
        assert abs(mt[0] - ref["abe_e"]) <= 1e-10 * abs(ref["abe_e"])
        np.testing.assert_allclose(mt[1:5], ref["abe_f"], rtol=1e-10)
        assert abs(mt[5] - ref["A_last"][-1]) <= 1e-10 * abs(ref["A_last"][-1])
        assert abs(mt[6] - ref["lambda"]) < 1e-14
        assert mt[7] == 0
    assert rel(ctx.get_params().cpu(), st.w) < 1e-9
    for b in range(len(st.blocks)):
        assert rel(ctx.kf.get_block(b).cpu(), st.P[b]) < 1e-9


@pytest.mark.parametrize("world", [2, 3])
def test_naive_sharded_ranks(world):
    """Naive-EKF with P sharded over `world` ranks in one process (the multi-GPU layout): every rank gets
    all samples' G, streams only its tiles, the partial U's are summed (the all-reduce of U that replaces
    the paper's P all-reduce, Fig. 5c), and w and every block of P match oracle.NaiveEKF (rel 1e-12)."""
    rng = np.random.default_rng(8)
    blocks = [5, 70, 130, 200, 64]
    opt = dict(lambda0=0.98, nu=0.9987, block_size=1024, noise_mode=0, p_defer=3)
    kfs = [fk.KalmanFilter(blocks, opt, shard=(world, r)) for r in range(world)]
    N = sum(blocks)
    st = O.NaiveEKF(np.zeros(N), blocks, lam=0.98, nu=0.9987)
    st.P = [_rand_spd(rng, n) for n in blocks]
    for kf in kfs:
        for b, P in enumerate(st.P):
            kf.set_block(b, cu(P))
    ws = [torch.zeros(N, dtype=torch.float64, device="cuda") for _ in range(world)]
    for it, n in enumerate([5, 12, 32]):
        G = rng.standard_normal((n, N))
        abe = rng.uniform(0.01, 1.0, n)
        Gd, ad = cu(G), cu(abe)
        for kf in kfs:
            kf.update_naive_begin(Gd)
        us = [kf.naive_partial_u() for kf in kfs]
        tot = torch.stack(us).sum(0)
        for u in us:
            u.copy_(tot)
        for kf, w in zip(kfs, ws):
            kf.update_naive_end(ad, w)
        st.update_naive(list(G), list(abe))
    torch.cuda.synchronize()
    for w in ws:
        assert rel(w.cpu(), st.w) < 1e-12
    for b, n in enumerate(blocks):
        full = torch.zeros(n, n, dtype=torch.float64, device="cuda")
        for kf in kfs:
            kf.get_block(b, out=full)
        assert rel(full.cpu(), st.P[b]) < 1e-12
    with pytest.raises(fk.FekfError):
        kfs[0].update_naive_end(ad, ws[0])        # end without begin


@pytest.mark.parametrize("rcut", [0.5, 1.2])
def test_degenerate_neighbourhoods(rcut):
    """Edge cases of the method's input: r_c = 0.5 A leaves every atom without neighbours (no embedding
    rows at all: D = 0, E_i = F(0), F = 0, the embedding-net gradients are 0); r_c = 1.2 A keeps only the
    O-H bonds (H atoms: one neighbour, no same-type neighbour, ragged per-type sections).  Forward, both
    Jacobians and one training step match the oracle."""
    wl = get_config("t2_tiny")
    m = type(wl.model)(**{**wl.model.__dict__, "rcut": rcut, "rcut_smth": rcut / 2})
    ds = make_dataset("t2_tiny", 2)
    w = init_weights(m, 3, float(ds["energy"].mean() / len(ds["types"])))
    ctx = fk.Context(m, wl.opt, types=ds["types"], local_batch=2, global_batch=2)
    ctx.set_params(cu(w))
    rj, rs, _ = O.build_nlist(ds["coord"], ds["box"], ds["types"], m.rcut, m.sel)
    nv = int((rj >= 0).sum())
    assert (nv == 0) if rcut < 0.9 else (0 < nv < rj.size // 4)
    ea, e, f, v = ctx.forward(cu(ds["coord"]), cu(ds["box"]))
    Ea, E, F, V = O.energy_force_virial(w, ds["coord"], ds["box"], ds["types"], rj, rs, m)
    assert rel(e.cpu(), E) < 1e-12 and rel(ea.cpu(), Ea) < 1e-12
    if nv == 0:
        assert float(f.abs().max()) == 0.0 and float(v.abs().max()) == 0.0
    else:
        assert rel(f.cpu(), F) < 1e-12 and rel(v.cpu().reshape(-1, 3, 3), V) < 1e-12
    g, s = ctx.energy_jacobian(cu(ds["coord"]), cu(ds["box"]), cu(ds["energy"]))
    gr, sr, _ = O.energy_grad(w, ds["coord"], ds["box"], ds["types"], rj, rs, ds["energy"], m)
    assert rel(g.cpu(), gr) < 1e-11
    atoms = force_groups(len(ds["types"]), 0, 5)[0]
    g, s = ctx.force_jacobian(cu(ds["coord"]), cu(ds["box"]), cu(ds["force"]), cu(atoms, torch.int32))
    gr, sr, _ = O.force_grad(w, ds["coord"], ds["box"], ds["types"], rj, rs, ds["force"], atoms, m)
    if nv == 0:
        assert float(g.abs().max()) == 0.0 and float(np.abs(gr).max()) == 0.0
    else:
        assert rel(g.cpu(), gr) < 1e-11
    st = O.FEKF.create(w, m, wl.opt)
    groups = force_groups(len(ds["types"]), 0, 17, wl.opt.force_groups, wl.opt.atoms_per_group)
    met = ctx.train_step(cu(ds["coord"]), cu(ds["box"]), cu(ds["energy"]), cu(ds["force"]), cu(groups, torch.int32))
    O.train_step(st, ds["coord"], ds["box"], ds["types"], ds["energy"], ds["force"], groups, m, wl.opt)
    assert np.all(np.isfinite(met.cpu().numpy()))
    assert rel(ctx.get_params().cpu(), st.w) < 1e-9
