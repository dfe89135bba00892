"""GPU parity, round 2: the configurations round 1 left untested, the §8(b) boundary additions and the
multi-rank step on one GPU.  CUDA path through the C ABI against the fp64 CPU oracle on the same seeded
inputs.

  * C4 sweep systems (BASELINE configs[3]): triclinic hcp (Mg36), two-image-shell diamond
    (Si72), rocksalt (NaCl64), H2O-48, a 4-type random alloy, Al32 — nlist bit-exact, forward, both
    Jacobians;
  * perfect lattices (exact r^2 ties, overflow cutting a shell of equal r^2) bit-exact;
  * embedding widths without a fused kernel (the per-layer GEMM path and its MODE_FORCE fallback);
  * duplicate atoms in a force group;
  * the reading flags switch_kind (Z8), env statistics (Z11, fekf_set_env_stats), type_one_side (Z15);
  * fekf_comm_init_loopback: r = 2, 4, 8 contexts on one GPU, B_g / r images each, P sharded or
    replicated, against oracle.train_step on the global batch;
  * the bench's launch configuration (water-64, B = 32, graph + split pass, 110 blocks, p_defer 15)
    end to end over one step, against the closed form of the first two Kalman updates from P = I.

Besides the normwise rel (reading Z19) the weights, gradients and P are also checked element-wise:
|a - b| <= tol * max(|b|, floor * max|b|).
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


def elem_rel(a, b, floor=1e-6):
    """max_i |a_i - b_i| / max(|b_i|, floor * max|b|): relative error of every element down to `floor`
    of the tensor's scale (small entries such as P's off-diagonal are held to their own size)."""
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


def _model(m, **kw):
    return ModelConfig(**{**m.__dict__, **kw})


def _check_model_pieces(m, ds, w, nb, atoms=None, tol=1e-12, jtol=1e-11):
    """nlist bit-exact, E/F/virial, energy and force Jacobians of the CUDA path against the oracle."""
    ctx = fk.Context(m, OptConfig(), types=ds["types"], local_batch=nb, global_batch=nb)
    ctx.set_params(cu(w))
    X, BX = cu(ds["coord"][:nb]), cu(ds["box"][:nb])
    types = ds["types"]
    nj, ns, ov = ctx.build_nlist(X, BX)
    rj, rs, rov = O.build_nlist(ds["coord"][:nb], ds["box"][:nb], types, m.rcut, m.sel)
    assert np.array_equal(nj.cpu().numpy(), rj) and np.array_equal(ns.cpu().numpy(), rs)
    assert np.array_equal(ov.cpu().numpy(), rov)
    ea, e, f, v = ctx.forward(X, BX)
    Ea, E, F, V = O.energy_force_virial(w, ds["coord"][:nb], ds["box"][:nb], types, rj, rs, m)
    assert rel(ea.cpu(), Ea) < tol and rel(e.cpu(), E) < tol
    assert rel(f.cpu(), F) < tol and rel(v.cpu().reshape(-1, 3, 3), V) < tol
    g, s = ctx.energy_jacobian(X, BX, cu(ds["energy"][:nb]))
    gr, sr, _ = O.energy_grad(w, ds["coord"][:nb], ds["box"][:nb], types, rj, rs, ds["energy"][:nb], m)
    assert rel(g.cpu(), gr) < jtol and elem_rel(g.cpu(), gr, 1e-3) < 1e-9
    assert abs(float(s.cpu()[0]) - sr) <= 1e-13 * max(1.0, abs(sr))
    if atoms is None:
        atoms = force_groups(len(types), 0, 5)[0]
    g, s = ctx.force_jacobian(X, BX, cu(ds["force"][:nb]), cu(atoms, torch.int32))
    gr, sr, _ = O.force_grad(w, ds["coord"][:nb], ds["box"][:nb], types, rj, rs, ds["force"][:nb], atoms, m)
    assert rel(g.cpu(), gr) < jtol and elem_rel(g.cpu(), gr, 1e-3) < 1e-9
    assert abs(float(s.cpu()[0]) - sr) <= 1e-12 * max(1.0, abs(sr))
    ctx.close()


# ------------------------------------------------------------------------------------------
# C4 systems: lattice types the round-1 cases did not have
# ------------------------------------------------------------------------------------------
C4 = ["c4_mg36", "c4_si72", "c4_nacl64", "c4_h2o48", "c4_alloy108", "c4_al32"]


@pytest.mark.parametrize("name", C4)
def test_c4_system_model_parity(name):
    wl = get_config(name)
    m = wl.model
    ds = make_dataset(name, 2)
    w = init_weights(m, 3, float(ds["energy"].mean() / len(ds["types"])))
    _check_model_pieces(m, ds, w, 2)


def test_alloy4_wide_fitting_tiles_ragged():
    """The first fitting layer's 128 x 80 / 16-warp GEMM (taken from 2048 fitting rows, K = 1600) with per-type
    row counts that are not multiples of the tile (B = 24 images of the random 4-type alloy: 888 / 648 / 552 /
    504 rows): forward, both Jacobians (primal and tangent rows) against the oracle."""
    name = "c4_alloy108"
    wl = get_config(name)
    ds = make_dataset(name, 24)
    w = init_weights(wl.model, 3, float(ds["energy"].mean() / len(ds["types"])))
    rows = [24 * int((ds["types"] == t).sum()) for t in range(4)]
    assert sum(rows) >= 2048 and any(r % 128 for r in rows)
    _check_model_pieces(wl.model, ds, w, 24)


def test_alloy4_train_steps():
    """A 4-type system (FEKF_MAX_TYPES; 16 embedding nets) through whole minibatch steps, small nets."""
    wl = get_config("c4_alloy108")
    m = _model(wl.model, emb=[4, 8, 16], m2=4, fit=[16, 16])
    opt = OptConfig(block_size=2048, p_defer=3)
    ds = make_dataset("c4_alloy108", 4)
    na = len(ds["types"])
    w0 = init_weights(m, 3, float(ds["energy"].mean() / na))
    _train_compare(m, opt, ds, w0, B=2, steps=4, tol=1e-9)


def _train_compare(m, opt, ds, w0, B, steps, tol, graph=True, check_p=True):
    na = len(ds["types"])
    ctx = fk.Context(m, opt, types=ds["types"], local_batch=B, global_batch=B, graph=graph)
    ctx.set_params(cu(w0))
    st = O.FEKF.create(w0, m, opt)
    nsl = len(ds["coord"]) // B
    for step in range(steps):
        sl = slice((step % nsl) * B, (step % nsl) * B + B)
        groups = force_groups(na, step, 17, opt.force_groups, opt.atoms_per_group)
        met = ctx.train_step(cu(ds["coord"][sl]), cu(ds["box"][sl]), cu(ds["energy"][sl]), cu(ds["force"][sl]),
                             cu(groups, torch.int32))
        ref = O.train_step(st, ds["coord"][sl], ds["box"][sl], ds["types"], ds["energy"][sl], ds["force"][sl],
                           groups, m, opt)
        mt = met.cpu().numpy()
        assert abs(mt[0] - ref["abe_e"]) <= tol * abs(ref["abe_e"])
        np.testing.assert_allclose(mt[1:1 + len(ref["abe_f"])], ref["abe_f"], rtol=tol)
        assert mt[7] == 0
    wg = ctx.get_params().cpu()
    assert rel(wg, st.w) < tol and elem_rel(wg, st.w) < 100 * tol
    if check_p:
        for b in range(len(st.blocks)):
            Pb = ctx.kf.get_block(b).cpu()
            assert rel(Pb, st.P[b]) < tol and elem_rel(Pb, st.P[b]) < 100 * tol
    ctx.close()
    return st


# ------------------------------------------------------------------------------------------
# exact ties: perfect lattice, overflow inside a shell of equal r^2
# ------------------------------------------------------------------------------------------
@pytest.mark.parametrize("sel", [[48], [16], [12], [7]])
def test_perfect_lattice_ties_bit_exact(sel):
    """sigma = 0 fcc (every shell an exact r^2 tie on both sides): the (type, r^2, j, shift) order decides
    which neighbours fill the section; sel 16 cuts the second shell (6 at r = a), 12 keeps exactly the
    first shell, 7 cuts the first shell.  Lists, shifts and overflow counts bit-exact, energies rel 1e-12."""
    wl = get_config("t_cu32_perfect")
    m = _model(wl.model, sel=sel)
    ds = make_dataset("t_cu32_perfect", 2)
    assert np.array_equal(ds["coord"][0], ds["coord"][1])
    w = init_weights(m, 3, 0.0)
    ctx = fk.Context(m, OptConfig(), types=ds["types"], local_batch=2, global_batch=2)
    ctx.set_params(cu(w))
    X, BX = cu(ds["coord"]), cu(ds["box"])
    nj, ns, ov = ctx.build_nlist(X, BX)
    rj, rs, rov = O.build_nlist(ds["coord"], ds["box"], ds["types"], m.rcut, m.sel)
    assert np.array_equal(nj.cpu().numpy(), rj) and np.array_equal(ns.cpu().numpy(), rs)
    assert np.array_equal(ov.cpu().numpy(), rov)
    assert (rov.sum() > 0) == (sel[0] < 18)
    ea, e, f, v = ctx.forward(X, BX)
    Ea, E, F, V = O.energy_force_virial(w, ds["coord"], ds["box"], ds["types"], rj, rs, m)
    assert rel(ea.cpu(), Ea) < 1e-12
    assert np.abs(f.cpu().numpy() - F).max() < 1e-12 * max(1.0, np.abs(Ea).max())
    ctx.close()


# ------------------------------------------------------------------------------------------
# embedding widths without a fused kernel, duplicate force atoms
# ------------------------------------------------------------------------------------------
@pytest.mark.parametrize("emb", [[6, 12], [5, 10, 20], [8, 8, 8, 8]])
def test_unfused_embedding_widths(emb):
    """Widths outside the compiled fused set take the per-layer GEMM path (nets.cu) and the restricted
    force reverse falls back to MODE_FORCE; forward, both Jacobians and 3 steps against the oracle."""
    wl = get_config("c1_cu32")
    m = _model(wl.model, emb=emb, m2=min(4, emb[-1]))
    ds = make_dataset("c1_cu32", 4)
    na = len(ds["types"])
    w = init_weights(m, 3, float(ds["energy"].mean() / na))
    _check_model_pieces(m, ds, w, 2)
    _train_compare(m, OptConfig(p_defer=2), ds, w, B=2, steps=3, tol=1e-9)


@pytest.mark.parametrize("name", ["c1_cu32", "t2_tiny"])
def test_duplicate_force_atoms(name):
    """A force group with repeated atoms (the kernels accept any list, reading Z5): every occurrence is a
    term of sum s F_sel (oracle: fancy indexing repeats the component)."""
    wl = get_config(name)
    m = wl.model
    ds = make_dataset(name, 2)
    w = init_weights(m, 3, float(ds["energy"].mean() / len(ds["types"])))
    atoms = np.array([3, 3, 5, 7, 7, 7], dtype=np.int32)
    _check_model_pieces(m, ds, w, 2, atoms=atoms)


# ------------------------------------------------------------------------------------------
# reading flags: switch_kind (Z8), env statistics (Z11), type_one_side (Z15)
# ------------------------------------------------------------------------------------------
FLAGS = {
    "cosine": dict(switch_kind=1),
    "one_side": dict(type_one_side=1),
    "stats": dict(env_avg=[[0.15, 0.01, -0.02, 0.0], [-0.3, 0.0, 0.02, 0.01]],
                  env_std=[[0.6, 0.8, 0.7, 0.9], [1.3, 0.9, 1.1, 1.0]]),
    "all": dict(switch_kind=1, type_one_side=1, env_avg=[[0.1, 0.0, 0.0, 0.0], [0.2, 0.0, 0.0, 0.0]],
                env_std=[[0.7, 0.6, 0.6, 0.6], [1.2, 0.8, 0.8, 0.8]]),
}


@pytest.mark.parametrize("emb", [[4, 8, 16], [5, 10, 20]])
@pytest.mark.parametrize("flag", sorted(FLAGS))
def test_reading_flags(flag, emb):
    """Each flag on the fused (4,8,16) and the per-layer (5,10,20) embedding path: R~ / J against the
    oracle's model_env (+ autograd J), forward, both Jacobians, and 3 training steps."""
    wl = get_config("t2_tiny")
    m = _model(wl.model, emb=emb, **FLAGS[flag])
    ds = make_dataset("t2_tiny", 4)
    na = len(ds["types"])
    w = init_weights(m, 3, float(ds["energy"].mean() / na))
    ctx = fk.Context(m, OptConfig(), types=ds["types"], local_batch=2, global_batch=2)
    rj, rs, _ = O.build_nlist(ds["coord"][:2], ds["box"][:2], ds["types"], m.rcut, m.sel)
    em, jac, rij = ctx.env_mat(cu(ds["coord"][:2]), cu(ds["box"][:2]), cu(rj, torch.int32), cu(rs, torch.int32))
    x = torch.tensor(ds["coord"][:2], requires_grad=False)
    d, R, mask = O.model_env(m, x, ds["box"][:2], ds["types"], rj, rs)
    assert rel(em.cpu(), R) < 1e-12
    dl = d.detach().clone().requires_grad_(True)
    Rr = O.env_rows(dl, mask, m.rcut, m.rcut_smth, m.switch_kind)
    if m.env_avg is not None:
        Rr = O.normalize_env(Rr, mask, ds["types"], m.env_avg, m.env_std)
    J = torch.stack([torch.autograd.grad(Rr[..., k].sum(), dl, retain_graph=True)[0] for k in range(4)], dim=-2)
    assert rel(jac.cpu(), J) < 1e-12
    ctx.close()
    _check_model_pieces(m, ds, w, 2)
    _train_compare(m, OptConfig(p_defer=2), ds, w, B=2, steps=3, tol=1e-9)


def test_env_stats_rejects_bad_std():
    wl = get_config("t2_tiny")
    m = wl.model
    ctx = fk.Context(m, OptConfig(), types=make_dataset("t2_tiny", 1)["types"], local_batch=1)
    with pytest.raises(fk.FekfError):
        ctx.set_env_stats(None, [[1.0, 1.0, 0.0, 1.0], [1.0, 1.0, 1.0, 1.0]])
    ctx.close()


# ------------------------------------------------------------------------------------------
# loopback communicator: the data-parallel step with sharded / replicated P on one GPU
# ------------------------------------------------------------------------------------------
def _run_ranks(world, fn):
    errs = [None] * world
    out = [None] * world

    def body(r):
        try:
            with torch.cuda.stream(torch.cuda.Stream()):
                out[r] = fn(r)
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
    return out


def test_loopback_allreduce_sum():
    world = 4
    comms = fk.Comm.loopback(world)

    def fn(r):
        buf = torch.full((1000,), float(r + 1), dtype=torch.float64, device="cuda")
        buf[0] = 0.1 * r
        for _ in range(3):
            comms[r].allreduce_sum(buf)
        return buf.cpu()

    outs = _run_ranks(world, fn)
    for o in outs:
        assert torch.equal(o, outs[0])
    assert float(outs[0][5]) == 10.0 * 16
    for c in comms:
        c.close()


@pytest.mark.parametrize("p_mode", [0, 1])
@pytest.mark.parametrize("world", [2, 4, 8])
def test_loopback_ranks_train_step(world, p_mode):
    """B_g = 8 images over `world` contexts on one GPU (local batch 8/world), P sharded by tile-row
    segments (p_mode 0: partial u all-reduced) or replicated (p_mode 1), [g || sum|e|] all-reduced
    (the early reduction), sqrt(B_g) and ABE / B_g (readings Z2-Z4): 3 minibatch steps with
    N_b = 1024 (several blocks, read-write passes at p_defer 2) equal oracle.train_step on the global batch.
    The force updates keep the split P pass at N > 1 (gradient all-reduced in two segments)."""
    wl = get_config("c1_cu32")
    m = wl.model
    opt = OptConfig(block_size=1024, p_defer=2, p_mode=p_mode)
    Bg = 8
    ds = make_dataset("c1_cu32", Bg)
    na = len(ds["types"])
    w0 = init_weights(m, 3, float(ds["energy"].mean() / na))
    B = Bg // world
    comms = fk.Comm.loopback(world)
    ctxs = [fk.Context(m, opt, types=ds["types"], local_batch=B, global_batch=Bg, comm=comms[r]) for r in range(world)]
    for c in ctxs:
        c.set_params(cu(w0))
    torch.cuda.synchronize()
    ctxs[0].kf.timing(True)
    steps = 3
    groups = [force_groups(na, s, 17, opt.force_groups, opt.atoms_per_group) for s in range(steps)]

    def fn(r):
        sl = slice(r * B, (r + 1) * B)
        mets = []
        for s in range(steps):
            met = ctxs[r].train_step(cu(ds["coord"][sl]), cu(ds["box"][sl]), cu(ds["energy"][sl]),
                                     cu(ds["force"][sl]), cu(groups[s], torch.int32))
            mets.append(met.cpu().numpy())
        return mets, ctxs[r].get_params().cpu().numpy()

    outs = _run_ranks(world, fn)
    ctxs[0].kf.timing(False)
    # the split pass stays on with a communicator: the all-reduce of g runs in two segments (the fitting
    # blocks' on the side stream ahead of the early pass), the late launch ran
    assert ctxs[0].kf.timing_parts()[1] > 0.0
    st = O.FEKF.create(w0, m, opt)
    refs = [O.train_step(st, ds["coord"], ds["box"], ds["types"], ds["energy"], ds["force"], groups[s], m, opt)
            for s in range(steps)]
    for r in range(world):
        mets, w = outs[r]
        assert np.array_equal(w, outs[0][1])           # every rank applies the identical update
        for s in range(steps):
            assert abs(mets[s][0] - refs[s]["abe_e"]) <= 1e-9 * abs(refs[s]["abe_e"])
            np.testing.assert_allclose(mets[s][1:5], refs[s]["abe_f"], rtol=1e-9)
            assert mets[s][7] == 0
    assert rel(outs[0][1], st.w) < 1e-9 and elem_rel(outs[0][1], st.w) < 1e-7
    for b, n in enumerate(st.blocks):
        if p_mode == 1:
            full = ctxs[0].kf.get_block(b).cpu()
        else:
            full = torch.zeros(n, n, dtype=torch.float64, device="cuda")
            for c in ctxs:
                c.kf.get_block(b, out=full)            # each rank fills the tiles it owns
            full = full.cpu()
        assert rel(full, st.P[b]) < 1e-9 and elem_rel(full, st.P[b]) < 1e-7
    for c in ctxs:
        c.close()
    for c in comms:
        c.close()


# ------------------------------------------------------------------------------------------
# the bench's launch configuration, end to end over one step
# ------------------------------------------------------------------------------------------
def test_bench_config_step_closed_form():
    """water-64 at the bench's configuration (B = 32, 1 027 082 parameters in 110 blocks of N_b = 10240,
    p_defer 15, step graph, split P pass with stealing), one minibatch with one force update.  From P = I
    the two updates have a closed form in the oracle's gradients (Alg. 1 lines 8-13, per block i):
      u1 = g_E,  A1 = 1/(L lam0 + g_E.g_E),  w1 = w0 + sqrt(B) ABE_E A1 g_E,  P1_i = (I - A1 g_E,i g_E,i^T)/lam0
      u2_i = (g_F,i - A1 g_E,i (g_E,i . g_F,i)) / lam0,  A2 = 1/(L lam1 + sum_i g_F,i . u2_i),
      w2 = w1 + sqrt(B) ABE_F A2 u2,  P2_i = (P1_i - A2 u2_i u2_i^T) / lam1
    with g_F the oracle's force gradient at w1.  w2 (every element) and sampled blocks of P2 are compared."""
    wl = get_config("c2_water64")
    m = wl.model
    opt = OptConfig(force_groups=1)
    B = wl.batch
    ds = make_dataset("c2_water64", B)
    na = len(ds["types"])
    w0 = init_weights(m, 3, float(ds["energy"].mean() / na))
    groups = force_groups(na, 0, wl.seed, 1, opt.atoms_per_group)
    ctx = fk.Context(m, opt, types=ds["types"], local_batch=B, global_batch=B)
    ctx.set_params(cu(w0))
    ctx.kf.timing(True)
    met = ctx.train_step(cu(ds["coord"]), cu(ds["box"]), cu(ds["energy"]), cu(ds["force"]), cu(groups, torch.int32))
    torch.cuda.synchronize()
    ctx.kf.timing(False)
    assert ctx.kf.timing_parts()[1] > 0.0      # the split pass ran
    mt = met.cpu().numpy()
    assert mt[7] == 0
    rj, rs, _ = O.build_nlist(ds["coord"], ds["box"], ds["types"], m.rcut, m.sel)
    gE, sE, _ = O.energy_grad(w0, ds["coord"], ds["box"], ds["types"], rj, rs, ds["energy"], m)
    sizes = [int(np.prod(s)) for _, s in O.param_tensors(m)]
    blocks = O.block_split(sizes, opt.block_size)
    assert len(blocks) == 110
    L = len(blocks)
    off = np.concatenate([[0], np.cumsum(blocks)])
    lam0, nu = opt.lambda0, opt.nu
    lam1 = lam0 * nu + 1 - nu
    abe_e = sE / B
    A1 = 1.0 / (L * lam0 + gE @ gE)
    w1 = w0 + np.sqrt(B) * abe_e * A1 * gE
    gF, sF, _ = O.force_grad(w1, ds["coord"], ds["box"], ds["types"], rj, rs, ds["force"], groups[0], m)
    abe_f = sF / (B * len(groups[0]) * 3) / na
    u2 = np.empty_like(gF)
    for i in range(L):
        sl = slice(off[i], off[i + 1])
        u2[sl] = (gF[sl] - A1 * gE[sl] * (gE[sl] @ gF[sl])) / lam0
    A2 = 1.0 / (L * lam1 + gF @ u2)
    w2 = w1 + np.sqrt(B) * abe_f * A2 * u2
    assert abs(mt[0] - abe_e) <= 1e-12 * abe_e and abs(mt[1] - abe_f) <= 1e-11 * abe_f
    assert abs(mt[5] - A2) <= 1e-10 * abs(A2)
    wg = ctx.get_params().cpu().numpy()
    assert rel(wg - w0, w2 - w0) < 1e-10 and elem_rel(wg - w0, w2 - w0, 1e-4) < 1e-7
    assert rel(wg, w2) < 1e-12
    for b in (0, 1, 2, 57, 109):
        sl = slice(off[b], off[b + 1])
        n = blocks[b]
        P1 = (np.eye(n) - A1 * np.outer(gE[sl], gE[sl])) / lam0
        P2 = (P1 - A2 * np.outer(u2[sl], u2[sl])) / lam1
        Pg = ctx.kf.get_block(b).cpu().numpy()
        assert rel(Pg, P2) < 1e-12
        dP = P2 - np.eye(n) / lam1     # the rank-2 part, held element-wise
        assert elem_rel(Pg - np.eye(n) / lam1, dP, 1e-4) < 1e-6
    ctx.close()


# ------------------------------------------------------------------------------------------
# the large-batch preset (B_g > 1024: lambda0 0.90, nu 0.996)
# ------------------------------------------------------------------------------------------
def test_large_batch_preset_train_steps():
    """A global minibatch of 1100 images (> 1024, so fekf_opt_defaults gives the paper's large-batch
    setting lambda0 = 0.90, nu = 0.996) in one context (local batch 1100: the energy seeds of
    more than 1024 images per launch) against the oracle, 2 minibatch steps, rel 1e-9."""
    wl = get_config("t2_tiny")
    m = wl.model
    d = fk.opt_defaults(1100)
    assert d["lambda0"] == 0.90 and d["nu"] == 0.996
    opt = OptConfig(**{k: d[k] for k in ("lambda0", "nu", "block_size", "noise_mode", "grad_reduce", "force_groups",
                                         "atoms_per_group", "p_defer")})
    B = 1100
    ds = make_dataset("t2_tiny", B)
    na = len(ds["types"])
    w0 = init_weights(m, 3, float(ds["energy"].mean() / na))
    _train_compare(m, opt, ds, w0, B=B, steps=2, tol=1e-9)


# ------------------------------------------------------------------------------------------
# fault handling: a non-finite update is dropped (flag latched, optimizer state kept)
# ------------------------------------------------------------------------------------------
def test_nonfinite_update_is_skipped():
    """A NaN energy label makes the energy update's ABE non-finite: that update is a no-op (w, P and lambda
    keep their values) with bit 1 of the fault flags set, and the step's 4 force updates proceed, so the
    weights equal those of a step whose energy update was skipped (lambda advanced 4 times, not 5)."""
    wl = get_config("t2_tiny")
    m, opt = wl.model, OptConfig(p_defer=2)
    B = wl.batch
    ds = make_dataset("t2_tiny", B)
    na = len(ds["types"])
    w0 = init_weights(m, 3, float(ds["energy"].mean() / na))
    groups = force_groups(na, 0, 17, opt.force_groups, opt.atoms_per_group)
    e_bad = ds["energy"].copy()
    e_bad[1] = np.nan
    ctx = fk.Context(m, opt, types=ds["types"], local_batch=B, global_batch=B)
    ctx.set_params(cu(w0))
    met = ctx.train_step(cu(ds["coord"]), cu(ds["box"]), cu(e_bad), cu(ds["force"]), cu(groups, torch.int32))
    mt = met.cpu().numpy()
    assert int(mt[7]) & 2
    lam = 1.0 - (1.0 - opt.lambda0) * opt.nu ** 4
    assert abs(mt[6] - lam) < 1e-14
    # reference: the oracle's step without its energy update (the 4 force updates from the same w, P = I)
    st = O.FEKF.create(w0, m, opt)
    nl = O.build_nlist(ds["coord"], ds["box"], ds["types"], m.rcut, m.sel)
    for atoms in groups:
        g, s, _ = O.force_grad(st.w, ds["coord"], ds["box"], ds["types"], nl[0], nl[1], ds["force"], atoms, m)
        st.update(g, s / (B * len(atoms) * 3) / na, B)
    wg = ctx.get_params().cpu().numpy()
    assert np.all(np.isfinite(wg))
    assert rel(wg, st.w) < 1e-9
    for b in range(len(st.blocks)):
        Pb = ctx.kf.get_block(b).cpu().numpy()
        assert np.all(np.isfinite(Pb)) and rel(Pb, st.P[b]) < 1e-9
    ctx.close()
