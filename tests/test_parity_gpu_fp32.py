"""GPU parity of the fp32 nets (the north_star's fp32 variant as SURVEY §8b states it: "precision 32 switches
nets and P to fp32"; reading Z22) against the fp64 oracle.

Tolerances, from the arithmetic ("fp32 tolerances"): every fp32 operation rounds at
u = 2^-24 = 6e-8 and the products are fp32-exact (split tf32 operands, real.cuh); the longest sums are the
first fitting layer's K = M M^< = 1600 terms and the descriptor's N_m = 138 neighbours, so a statistical
bound on a value's relative error is about sqrt(K) u ~ 2.4e-6 and the depth (3 embedding + 4 fitting
layers, forward and reverse) multiplies it by a small factor: E, F, virial normwise 1e-5; the Jacobians,
which sum ~1e5 products per weight over rows of both signs (cancellation), normwise 1e-4; and w, P after
10 EKF steps 1e-4 (north_star).  The fp64-net path keeps its own bars (test_parity_gpu.py).
"""
import threading

import numpy as np
import pytest
import torch

import oracle as O
from fixtures import get_config, make_dataset, init_weights, force_groups, ModelConfig, OptConfig

pytestmark = pytest.mark.gpu

fk = pytest.importorskip("paper_conf_ppopp_huzslmlwtj24_b200")


def rel(a, b):
    a = np.asarray(a, dtype=np.float64)
    b = np.asarray(b, dtype=np.float64)
    den = np.abs(b).max()
    return float(np.abs(a - b).max() / (den if den > 0 else 1.0))


def cu(x, dtype=torch.float64):
    return torch.as_tensor(np.ascontiguousarray(x)).to(dtype).cuda()


@pytest.fixture(scope="module", autouse=True)
def _gpu():
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    fk.lib()


def _setup(name, nb, seed=3, **opt_over):
    wl = get_config(name)
    m = wl.model
    ds = make_dataset(name, nb)
    w = init_weights(m, seed, float(ds["energy"].mean() / len(ds["types"])))
    opt = type(wl.opt)(**{**wl.opt.__dict__, "net_precision": 32, **opt_over})
    ctx = fk.Context(m, opt, types=ds["types"], local_batch=nb, global_batch=nb)
    ctx.set_params(cu(w))
    return wl, m, ds, w, ctx


CASES = [("t2_tiny", 3), ("c1_cu32", 4), ("paper_cu108", 2), ("c2_water64", 2), ("c4_alloy108", 1)]


@pytest.mark.parametrize("name,nb", CASES)
def test_fp32_forward_energy_force_virial(name, nb):
    wl, m, ds, w, ctx = _setup(name, nb)
    ea, e, f, v = ctx.forward(cu(ds["coord"]), cu(ds["box"]))
    rj, rs, _ = O.build_nlist(ds["coord"], ds["box"], ds["types"], m.rcut, m.sel)
    Ea, E, F, V = O.energy_force_virial(w, ds["coord"], ds["box"], ds["types"], rj, rs, m)
    r = [rel(ea.cpu(), Ea), rel(e.cpu(), E), rel(f.cpu(), F), rel(v.cpu().reshape(-1, 3, 3), V)]
    assert max(r) < 1e-5, r
    # fp32, not fp64 (the nets really run in fp32): the force error is far above fp64 rounding
    assert rel(f.cpu(), F) > 1e-12


@pytest.mark.parametrize("name,nb", CASES)
def test_fp32_energy_jacobian(name, nb):
    wl, m, ds, w, ctx = _setup(name, nb)
    g, s = ctx.energy_jacobian(cu(ds["coord"]), cu(ds["box"]), cu(ds["energy"]))
    rj, rs, _ = O.build_nlist(ds["coord"], ds["box"], ds["types"], m.rcut, m.sel)
    gr, sr, _ = O.energy_grad(w, ds["coord"], ds["box"], ds["types"], rj, rs, ds["energy"], m)
    assert rel(g.cpu(), gr) < 1e-4, rel(g.cpu(), gr)
    assert abs(float(s.cpu()[0]) - sr) <= 1e-5 * max(1.0, abs(sr))


@pytest.mark.parametrize("name,nb", CASES)
def test_fp32_force_jacobian(name, nb):
    wl, m, ds, w, ctx = _setup(name, nb)
    atoms = force_groups(len(ds["types"]), 0, 5)[0]
    g, s = ctx.force_jacobian(cu(ds["coord"]), cu(ds["box"]), cu(ds["force"]), cu(atoms, torch.int32))
    rj, rs, _ = O.build_nlist(ds["coord"], ds["box"], ds["types"], m.rcut, m.sel)
    gr, sr, _ = O.force_grad(w, ds["coord"], ds["box"], ds["types"], rj, rs, ds["force"], atoms, m)
    assert rel(g.cpu(), gr) < 1e-4, rel(g.cpu(), gr)
    assert abs(float(s.cpu()[0]) - sr) <= 1e-5 * max(1.0, abs(sr))


@pytest.mark.parametrize("name,steps,precision,net_precision", [
    ("c1_cu32", 10, 32, 0),    # the fp32 variant: P and nets fp32
    ("c1_cu32", 10, 64, 32),   # fp32 nets over an fp64 P
    ("c1_cu32", 10, 32, 64),   # fp32 P over fp64 nets (round 2's variant)
])
def test_fp32_train_steps(name, steps, precision, net_precision):
    """10 minibatch steps (50 KF updates, reading Z20) against the fp64 oracle: w and P within rel 1e-4."""
    wl = get_config(name)
    m, opt = wl.model, wl.opt
    opt = type(opt)(**{**opt.__dict__, "precision": precision, "net_precision": net_precision})
    tol = 1e-4
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
    assert rel(wg, st.w) < tol
    for b, n in enumerate(st.blocks):
        assert rel(ctx.kf.get_block(b).cpu(), st.P[b]) < tol


def test_fp32_water64_bench_config_step():
    """The bench configuration (water-64, B = 32, 110 blocks, split pass) with the fp32 nets and P: one
    training step runs and its first energy update's ABE matches the oracle's fp64 forward."""
    wl = get_config("c2_water64")
    m = wl.model
    B = wl.batch
    ds = make_dataset("c2_water64", B)
    na = len(ds["types"])
    w0 = init_weights(m, 3, float(ds["energy"].mean() / na))
    opt = type(wl.opt)(**{**wl.opt.__dict__, "precision": 32})
    ctx = fk.Context(m, opt, types=ds["types"], local_batch=B, global_batch=B)
    ctx.set_params(cu(w0))
    groups = force_groups(na, 0, 17, opt.force_groups, opt.atoms_per_group)
    met = ctx.train_step(cu(ds["coord"]), cu(ds["box"]), cu(ds["energy"]), cu(ds["force"]), cu(groups, torch.int32))
    mt = met.cpu().numpy()
    rj, rs, _ = O.build_nlist(ds["coord"], ds["box"], ds["types"], m.rcut, m.sel)
    _, E, _, _ = O.energy_force_virial(w0, ds["coord"], ds["box"], ds["types"], rj, rs, m)
    abe_e = float(np.mean(np.abs(ds["energy"] - E)) / na)
    assert abs(mt[0] - abe_e) <= 1e-5 * abe_e
    assert mt[7] == 0 and np.all(np.isfinite(mt))
    assert np.all(np.isfinite(ctx.get_params().cpu().numpy()))


# ------------------------------------------------------------------------------------------
# the fp32 per-layer embedding path (widths outside the fused set), the reading flags and the
# multi-rank step, each against the fp64 oracle at the fp32 bars
# ------------------------------------------------------------------------------------------
def _model(m, **kw):
    return ModelConfig(**{**m.__dict__, **kw})


def _check_fp32_pieces(m, ds, w, nb):
    opt = OptConfig(net_precision=32)
    ctx = fk.Context(m, opt, types=ds["types"], local_batch=nb, global_batch=nb)
    ctx.set_params(cu(w))
    X, BX = cu(ds["coord"][:nb]), cu(ds["box"][:nb])
    types = ds["types"]
    rj, rs, _ = O.build_nlist(ds["coord"][:nb], ds["box"][:nb], types, m.rcut, m.sel)
    ea, e, f, v = ctx.forward(X, BX)
    Ea, E, F, V = O.energy_force_virial(w, ds["coord"][:nb], ds["box"][:nb], types, rj, rs, m)
    r = [rel(ea.cpu(), Ea), rel(e.cpu(), E), rel(f.cpu(), F), rel(v.cpu().reshape(-1, 3, 3), V)]
    assert max(r) < 1e-5, r
    g, s = ctx.energy_jacobian(X, BX, cu(ds["energy"][:nb]))
    gr, sr, _ = O.energy_grad(w, ds["coord"][:nb], ds["box"][:nb], types, rj, rs, ds["energy"][:nb], m)
    assert rel(g.cpu(), gr) < 1e-4
    atoms = force_groups(len(types), 0, 5)[0]
    g, s = ctx.force_jacobian(X, BX, cu(ds["force"][:nb]), cu(atoms, torch.int32))
    gr, sr, _ = O.force_grad(w, ds["coord"][:nb], ds["box"][:nb], types, rj, rs, ds["force"][:nb], atoms, m)
    assert rel(g.cpu(), gr) < 1e-4
    ctx.close()


def _train_fp32(m, opt, ds, w0, B, steps):
    na = len(ds["types"])
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
        np.testing.assert_allclose(mt[:5], [ref["abe_e"], *ref["abe_f"]], rtol=1e-4)
        assert mt[7] == 0
    assert rel(ctx.get_params().cpu(), st.w) < 1e-4
    for b, n in enumerate(st.blocks):
        assert rel(ctx.kf.get_block(b).cpu(), st.P[b]) < 1e-4
    ctx.close()


@pytest.mark.parametrize("emb", [[6, 12], [5, 10, 20], [8, 8, 8, 8], [4, 12, 36]])
def test_fp32_unfused_embedding_widths(emb):
    """fp32 per-layer embedding path (FFMA GEMMs with the activation-adjoint epilogues, the layer-0 and seed
    kernels, prod_force) and the MODE_FORCE fallback: forward, both Jacobians, 3 steps (fp32 P too)."""
    wl = get_config("c1_cu32")
    m = _model(wl.model, emb=emb, m2=min(4, emb[-1]))
    ds = make_dataset("c1_cu32", 4)
    w = init_weights(m, 3, float(ds["energy"].mean() / len(ds["types"])))
    _check_fp32_pieces(m, ds, w, 2)
    _train_fp32(m, OptConfig(p_defer=2, precision=32), ds, w, B=2, steps=3)


FLAGS = {
    "one_side": dict(type_one_side=1),
    "all": dict(switch_kind=1, type_one_side=1, env_avg=[[0.1, 0.0, 0.0, 0.0], [0.2, 0.0, 0.0, 0.0]],
                env_std=[[0.7, 0.6, 0.6, 0.6], [1.2, 0.8, 0.8, 0.8]]),
}


@pytest.mark.parametrize("emb", [[4, 8, 16], [5, 10, 20]])
@pytest.mark.parametrize("flag", sorted(FLAGS))
def test_fp32_reading_flags(flag, emb):
    """type_one_side (shared nets: the fp32 weight-gradient partials accumulate into the fp64 g), the cosine
    switch and the env statistics on the fused and per-layer fp32 paths."""
    wl = get_config("t2_tiny")
    m = _model(wl.model, emb=emb, **FLAGS[flag])
    ds = make_dataset("t2_tiny", 4)
    w = init_weights(m, 3, float(ds["energy"].mean() / len(ds["types"])))
    _check_fp32_pieces(m, ds, w, 2)
    _train_fp32(m, OptConfig(p_defer=2, precision=32), ds, w, B=2, steps=3)


def test_fp32_loopback_two_ranks():
    """The fp32 variant over 2 contexts on one GPU (loopback communicator, P sharded): B_g = 8 images, 3 steps
    equal oracle.train_step on the global batch at 1e-4."""
    wl = get_config("c1_cu32")
    m = wl.model
    opt = OptConfig(block_size=1024, p_defer=2, precision=32)
    Bg, world = 8, 2
    ds = make_dataset("c1_cu32", Bg)
    na = len(ds["types"])
    w0 = init_weights(m, 3, float(ds["energy"].mean() / na))
    B = Bg // world
    comms = fk.Comm.loopback(world)
    ctxs = [fk.Context(m, opt, types=ds["types"], local_batch=B, global_batch=Bg, comm=comms[r]) for r in range(world)]
    for c in ctxs:
        c.set_params(cu(w0))
    torch.cuda.synchronize()
    steps = 3
    groups = [force_groups(na, s, 17, opt.force_groups, opt.atoms_per_group) for s in range(steps)]
    out, errs = [None] * world, [None] * world

    def body(r):
        try:
            with torch.cuda.stream(torch.cuda.Stream()):
                sl = slice(r * B, (r + 1) * B)
                mets = [ctxs[r].train_step(cu(ds["coord"][sl]), cu(ds["box"][sl]), cu(ds["energy"][sl]),
                                           cu(ds["force"][sl]), cu(groups[s], torch.int32)).cpu().numpy()
                        for s in range(steps)]
                out[r] = (mets, ctxs[r].get_params().cpu().numpy())
                torch.cuda.current_stream().synchronize()
        except BaseException as e:   # noqa: BLE001 - surfaced below
            errs[r] = e

    ts = [threading.Thread(target=body, args=(r,)) for r in range(world)]
    for t in ts:
        t.start()
    for t in ts:
        t.join()
    for e in errs:
        if e is not None:
            raise e
    st = O.FEKF.create(w0, m, opt)
    refs = [O.train_step(st, ds["coord"], ds["box"], ds["types"], ds["energy"], ds["force"], groups[s], m, opt)
            for s in range(steps)]
    for r in range(world):
        mets, w = out[r]
        assert np.array_equal(w, out[0][1])
        for s in range(steps):
            np.testing.assert_allclose(mets[s][:5], [refs[s]["abe_e"], *refs[s]["abe_f"]], rtol=1e-4)
    assert rel(out[0][1], st.w) < 1e-4
    for c in ctxs:
        c.close()
    for c in comms:
        c.close()
