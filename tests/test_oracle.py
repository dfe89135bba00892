"""Pins of the CPU oracle to things other than itself (paper values, closed forms, invariances,
finite differences, brute force).  CPU only (`-m "not gpu"`)."""
import itertools
import json
import math
import os

import numpy as np
import pytest
import torch

import oracle as O
from fixtures import (get_config, make_dataset, init_weights, force_groups, random_rotation,
                      ModelConfig, OptConfig, tensor_shapes)

GOLD = os.path.join(os.path.dirname(__file__), "golden", "paper_model.json")


@pytest.fixture(scope="module")
def gold():
    with open(GOLD) as f:
        return json.load(f)


# ------------------------------------------------------------------------------------------
# 1. layout + block split: values printed by the paper
# ------------------------------------------------------------------------------------------
def _paper_model(gold, dt=1):
    g = gold["model"]
    return ModelConfig(1, 6.0, 0.5, [96], g["emb"], g["m2"], g["fit"], fit_resnet_dt=dt)


def test_paper_param_count(gold):
    m = _paper_model(gold)
    assert O.param_count(m) == gold["model"]["n_params"] == 26651
    # the timestep vectors (reading Z14) are what makes the printed count come out
    assert O.param_count(_paper_model(gold, dt=0)) == 26651 - 100
    # fitting input is M * M^< = 400 ("[400, 50, 50, 50, 1]")
    assert dict(O.param_tensors(m))["fit0.W0"] == (400, 50)


def test_paper_block_split(gold):
    m = _paper_model(gold)
    sizes = [int(np.prod(s)) for _, s in O.param_tensors(m)]
    blocks = O.block_split(sizes, gold["block_size"]["value"])
    assert blocks == gold["blocks"]["sizes"]
    mib = [n * n * 8 / 2**20 for n in blocks]
    np.testing.assert_allclose(mib, gold["block_mb"]["values"], atol=0.006)
    assert round(sum(mib)) == gold["block_mb"]["total"]
    gmb = [n * 8 / 2**20 for n in blocks]
    np.testing.assert_allclose(gmb, gold["grad_mb"]["values"], atol=0.006)
    assert round(sum(gmb), 1) == gold["grad_mb"]["total"]


def test_block_split_rules():
    assert O.block_split([5, 5, 5], 100) == [15]
    assert O.block_split([60, 60], 100) == [60, 60]
    assert O.block_split([10, 250, 3], 100) == [10, 100, 100, 50, 3]
    assert O.block_split([100], 100) == [100]
    assert O.block_split([40, 60, 1], 100) == [100, 1]
    for sizes in ([3, 7, 11, 200, 5], [1] * 50, [99, 2, 99]):
        bl = O.block_split(sizes, 37)
        assert sum(bl) == sum(sizes) and max(bl) <= 37


def test_layout_matches_fixture_shapes():
    for name in ("c1_cu32", "c2_water64", "t2_tiny", "paper_cu108"):
        m = get_config(name).model
        assert [s for _, s in O.param_tensors(m)] == [s for _, s in tensor_shapes(m)]


# ------------------------------------------------------------------------------------------
# 2. neighbour list: brute force over a wide image range, scipy for short cutoffs
# ------------------------------------------------------------------------------------------
def _brute_pairs(coord, box, rcut, i, span=3):
    out = []
    for n in itertools.product(range(-span, span + 1), repeat=3):
        S = n[0] * box[0] + n[1] * box[1] + n[2] * box[2]
        for j in range(len(coord)):
            if j == i and n == (0, 0, 0):
                continue
            d = coord[j] + S - coord[i]
            if float(d @ d) < rcut * rcut:
                out.append((j, O.shift_id(*n), float(np.sqrt(d @ d))))
    return out


@pytest.mark.parametrize("name", ["c1_cu32", "t2_tiny"])
def test_nlist_brute_force(name):
    wl = get_config(name)
    m = wl.model
    ds = make_dataset(name, 2)
    nl_j, nl_s, ov = O.build_nlist(ds["coord"], ds["box"], ds["types"], m.rcut, m.sel)
    sec = np.concatenate([[0], np.cumsum(m.sel)])
    for b in range(2):
        for i in range(len(ds["types"])):
            ref = _brute_pairs(ds["coord"][b], ds["box"][b], m.rcut, i)
            for t in range(m.ntypes):
                rt = sorted([(r, j, s) for (j, s, r) in ref if ds["types"][j] == t])
                got_j = nl_j[b, i, sec[t]:sec[t + 1]]
                got_s = nl_s[b, i, sec[t]:sec[t + 1]]
                k = min(len(rt), m.sel[t])
                assert [(j, s) for (_, j, s) in rt[:k]] == list(zip(got_j[:k], got_s[:k]))
                assert np.all(got_j[k:] == -1) and np.all(got_s[k:] == -1)
    assert ov.sum() == 0


def test_nlist_overflow_keeps_nearest():
    wl = get_config("t2_tiny")
    m = wl.model
    ds = make_dataset("t2_tiny", 1)
    small = [5, 9]
    nl_j, nl_s, ov = O.build_nlist(ds["coord"], ds["box"], ds["types"], m.rcut, small)
    full_j, full_s, _ = O.build_nlist(ds["coord"], ds["box"], ds["types"], m.rcut, [200, 200])
    tot = 0
    for i in range(len(ds["types"])):
        for t, (a, b) in enumerate([(0, 5), (5, 14)]):
            fa = full_j[0, i, 200 * t:200 * (t + 1)]
            n = int((fa >= 0).sum())
            tot += max(0, n - small[t])
            assert list(nl_j[0, i, a:b][:min(n, small[t])]) == list(fa[:min(n, small[t])])
    assert ov[0] == tot > 0


def test_nlist_matches_kdtree_short_cutoff():
    from scipy.spatial import cKDTree
    name = "c2_water64"
    m = get_config(name).model
    ds = make_dataset(name, 1)
    L = ds["box"][0, 0, 0]
    assert m.rcut < L / 2
    x = ds["coord"][0]
    tree = cKDTree(np.mod(x, L), boxsize=L)
    pairs = tree.query_pairs(m.rcut)
    cnt = np.zeros(len(x), dtype=int)
    for a, b in pairs:
        cnt[a] += 1
        cnt[b] += 1
    nl_j, _, ov = O.build_nlist(ds["coord"], ds["box"], ds["types"], m.rcut, m.sel)
    assert ov[0] == 0
    np.testing.assert_array_equal((nl_j[0] >= 0).sum(1), cnt)


# ------------------------------------------------------------------------------------------
# 3. s(r) and R~: closed forms of P:L83
# ------------------------------------------------------------------------------------------
def test_switch_closed_form_and_smoothness():
    rcs, rc = 1.0, 4.0
    r = np.linspace(0.2, 0.999, 50)
    np.testing.assert_allclose(O.switch(r, rcs, rc), 1.0 / r, rtol=0, atol=0)   # "1/x for x < r_cs"
    assert O.switch(np.array([rc]), rcs, rc)[0] == 0.0
    assert np.all(O.switch(np.array([rc + 0.1, 7.0]), rcs, rc) == 0.0)
    sw = lambda x: O.switch(x, rcs, rc) * x
    h = 1e-6
    for x0, side in ((rcs, +1), (rc, -1)):
        # sw is continuous with zero first and second derivative at both ends (C2 quintic, Z8)
        v0 = sw(np.array([x0 + side * 1e-12]))[0]
        v1, v2 = sw(np.array([x0 + side * h]))[0], sw(np.array([x0 + 2 * side * h]))[0]
        assert abs(v0 - (1.0 if x0 == rcs else 0.0)) < 1e-9
        assert abs((v1 - v0) / h) < 1e-4 and abs((v2 - 2 * v1 + v0) / (h * h)) < 1e-2
    x = np.linspace(rcs, rc, 1001)
    assert np.all(np.diff(sw(x)) <= 1e-15)                   # monotone decay on [r_cs, r_c]


def test_env_mat_properties():
    name = "t2_tiny"
    m = get_config(name).model
    ds = make_dataset(name, 2)
    nl_j, nl_s, _ = O.build_nlist(ds["coord"], ds["box"], ds["types"], m.rcut, m.sel)
    d, R, mask = O.env_mat(torch.as_tensor(ds["coord"]), ds["box"], nl_j, nl_s, m.rcut, m.rcut_smth)
    R = R.numpy(); d = d.numpy(); mask = mask.numpy()
    assert np.all(R[~mask] == 0)
    r = np.linalg.norm(d[mask], axis=-1)
    assert np.all(r < m.rcut) and np.all(r > 0)
    np.testing.assert_allclose(np.linalg.norm(R[mask][:, 1:], axis=-1), np.abs(R[mask][:, 0]), rtol=1e-14)
    below = r < m.rcut_smth
    np.testing.assert_allclose(R[mask][below, 0], 1.0 / r[below], rtol=1e-15)


# ------------------------------------------------------------------------------------------
# 4-7. invariances and F = -grad E
# ------------------------------------------------------------------------------------------
def _setup(name, n=2, seed=3):
    wl = get_config(name)
    m = wl.model
    ds = make_dataset(name, n)
    w = init_weights(m, seed, float(ds["energy"].mean() / len(ds["types"])))
    return wl, m, ds, w


def _efv(w, coord, box, types, m):
    nl_j, nl_s, _ = O.build_nlist(coord, box, types, m.rcut, m.sel)
    return O.energy_force_virial(w, coord, box, types, nl_j, nl_s, m)


@pytest.mark.parametrize("name", ["t2_tiny", "c1_cu32"])
def test_invariances(name):
    wl, m, ds, w = _setup(name)
    Ea, E, F, V = _efv(w, ds["coord"], ds["box"], ds["types"], m)
    rng = np.random.default_rng(5)
    # rotation of coordinates and box
    Q = random_rotation(rng)
    Er, Fr = _efv(w, ds["coord"] @ Q.T, ds["box"] @ Q.T, ds["types"], m)[1:3]
    np.testing.assert_allclose(Er, E, rtol=1e-12)
    np.testing.assert_allclose(Fr, F @ Q.T, rtol=0, atol=1e-11 * np.abs(F).max())
    # translation (wrapped back into the cell: periodic images make it exact)
    sh = np.array([0.37, -1.1, 2.3])
    c2 = ds["coord"] + sh
    fr = np.einsum("bna,bak->bnk", c2, np.linalg.inv(ds["box"]))
    c2 = np.einsum("bnk,bka->bna", fr - np.floor(fr), ds["box"])
    Et, Ft = _efv(w, c2, ds["box"], ds["types"], m)[1:3]
    np.testing.assert_allclose(Et, E, rtol=1e-12)
    np.testing.assert_allclose(Ft, F, atol=1e-11 * np.abs(F).max())
    # permutation of same-type atoms
    perm = np.arange(len(ds["types"]))
    for t in range(m.ntypes):
        idx = np.nonzero(ds["types"] == t)[0]
        perm[idx] = rng.permutation(idx)
    Ep, Fp = _efv(w, ds["coord"][:, perm], ds["box"], ds["types"], m)[1:3]
    np.testing.assert_allclose(Ep, E, rtol=1e-12)
    np.testing.assert_allclose(Fp, F[:, perm], atol=1e-11 * np.abs(F).max())
    # translation invariance => forces sum to zero
    assert np.abs(F.sum(1)).max() < 1e-11 * np.abs(F).max()


@pytest.mark.parametrize("name", ["t2_tiny", "c1_cu32"])
def test_force_is_minus_grad_energy_fd(name):
    wl, m, ds, w = _setup(name, n=1)
    nl_j, nl_s, _ = O.build_nlist(ds["coord"], ds["box"], ds["types"], m.rcut, m.sel)
    _, E, F, _ = O.energy_force_virial(w, ds["coord"], ds["box"], ds["types"], nl_j, nl_s, m)
    h = 1e-5
    rng = np.random.default_rng(1)
    for _ in range(8):
        a, c = int(rng.integers(len(ds["types"]))), int(rng.integers(3))
        xp = ds["coord"].copy(); xp[0, a, c] += h
        xm = ds["coord"].copy(); xm[0, a, c] -= h
        Ep = O.energy_force_virial(w, xp, ds["box"], ds["types"], nl_j, nl_s, m, need_force=False)[1]
        Em = O.energy_force_virial(w, xm, ds["box"], ds["types"], nl_j, nl_s, m, need_force=False)[1]
        fd = -(Ep[0] - Em[0]) / (2 * h)
        assert abs(fd - F[0, a, c]) <= 1e-6 * max(1.0, np.abs(F).max())


def test_virial_is_strain_derivative():
    wl, m, ds, w = _setup("c1_cu32", n=1)
    nl_j, nl_s, _ = O.build_nlist(ds["coord"], ds["box"], ds["types"], m.rcut, m.sel)
    _, E, F, V = O.energy_force_virial(w, ds["coord"], ds["box"], ds["types"], nl_j, nl_s, m)
    h = 1e-6
    fd = np.zeros((3, 3))
    for a in range(3):
        for c in range(3):
            eps = np.zeros((3, 3)); eps[a, c] = h
            Ep = O.energy_force_virial(w, ds["coord"] @ (np.eye(3) + eps), ds["box"] @ (np.eye(3) + eps),
                                       ds["types"], nl_j, nl_s, m, need_force=False)[1][0]
            Em = O.energy_force_virial(w, ds["coord"] @ (np.eye(3) - eps), ds["box"] @ (np.eye(3) - eps),
                                       ds["types"], nl_j, nl_s, m, need_force=False)[1][0]
            fd[a, c] = -(Ep - Em) / (2 * h)
    np.testing.assert_allclose(V[0], fd, atol=1e-6 * np.abs(V).max())
    np.testing.assert_allclose(V[0], V[0].T, atol=1e-12 * np.abs(V).max())


# ------------------------------------------------------------------------------------------
# 8-9. gradients w.r.t. the weights by finite differences
# ------------------------------------------------------------------------------------------
def test_energy_grad_fd():
    wl, m, ds, w = _setup("t2_tiny", n=2)
    nl_j, nl_s, _ = O.build_nlist(ds["coord"], ds["box"], ds["types"], m.rcut, m.sel)
    g, abs_sum, E = O.energy_grad(w, ds["coord"], ds["box"], ds["types"], nl_j, nl_s, ds["energy"], m)
    na = len(ds["types"])
    sgn = np.where(E >= ds["energy"], -1.0, 1.0)
    assert abs(abs_sum - np.abs((ds["energy"] - E) / na).sum()) < 1e-14
    f = lambda ww: (sgn * O.energy_force_virial(ww, ds["coord"], ds["box"], ds["types"], nl_j, nl_s, m,
                                                need_force=False)[1]).sum() / na
    rng = np.random.default_rng(2)
    h = 1e-6
    for k in list(rng.choice(len(w), 12, replace=False)) + [0, len(w) - 1]:
        e = np.zeros_like(w); e[k] = h
        fd = (f(w + e) - f(w - e)) / (2 * h)
        assert abs(fd - g[k]) <= 1e-6 * max(1e-3, np.abs(g).max())


def test_force_grad_fd():
    wl, m, ds, w = _setup("t2_tiny", n=2)
    nl_j, nl_s, _ = O.build_nlist(ds["coord"], ds["box"], ds["types"], m.rcut, m.sel)
    atoms = [1, 4, 9, 17]
    g, abs_sum, Fsel = O.force_grad(w, ds["coord"], ds["box"], ds["types"], nl_j, nl_s, ds["force"], atoms, m)
    na = len(ds["types"])
    Fl = ds["force"][:, atoms]
    sgn = np.where(Fsel >= Fl, -1.0, 1.0)
    assert abs(abs_sum - np.abs(Fl - Fsel).sum()) < 1e-12
    def f(ww):
        F = O.energy_force_virial(ww, ds["coord"], ds["box"], ds["types"], nl_j, nl_s, m)[2]
        return (sgn * F[:, atoms]).sum() / (na * len(atoms) * 3)
    rng = np.random.default_rng(3)
    h = 1e-6
    for k in list(rng.choice(len(w), 12, replace=False)) + [len(w) - 2]:
        e = np.zeros_like(w); e[k] = h
        fd = (f(w + e) - f(w - e)) / (2 * h)
        assert abs(fd - g[k]) <= 1e-6 * max(1e-4, np.abs(g).max())
    # b_out cannot change a force
    assert g[len(w) - 1] == 0.0


# ------------------------------------------------------------------------------------------
# 10. Kalman algebra: Sherman-Morrison closed form, RLEKF special case, lambda schedule
# ------------------------------------------------------------------------------------------
def _rand_spd(rng, n):
    a = rng.standard_normal((n, n))
    return a @ a.T / n + np.eye(n)


@pytest.mark.parametrize("noise_mode", [0, 1])
def test_kalman_matches_explicit_inverse(noise_mode):
    rng = np.random.default_rng(11)
    blocks = [3, 5, 2]
    st = O.FEKF(np.zeros(10), blocks, lam=0.97, nu=0.99, noise_mode=noise_mode)
    st.P = [_rand_spd(rng, n) for n in blocks]
    for it in range(6):
        g = rng.standard_normal(10)
        abe = float(rng.uniform(0.1, 1.0))
        Pbd = np.zeros((10, 10))
        off = np.concatenate([[0], np.cumsum(blocks)])
        for i, P in enumerate(st.P):
            Pbd[off[i]:off[i + 1], off[i]:off[i + 1]] = P
        lam = st.lam
        c = len(blocks) * lam if noise_mode == 0 else lam
        K_ref = Pbd @ g / (c + g @ Pbd @ g)
        P_ref = np.linalg.inv(np.linalg.inv(Pbd) + np.outer(g, g) / c) / lam
        w0 = st.w.copy()
        st.update(g, abe, bs=4)
        np.testing.assert_allclose(st.w - w0, 2.0 * abe * K_ref, rtol=1e-12, atol=1e-15)
        for i in range(len(blocks)):
            sl = slice(off[i], off[i + 1])
            np.testing.assert_allclose(st.P[i], P_ref[sl, sl], rtol=1e-11, atol=1e-13)
            assert np.array_equal(st.P[i], st.P[i].T)
            np.linalg.cholesky(st.P[i])                      # stays SPD
        assert abs(st.lam - (lam * 0.99 + 0.01)) < 4e-16


def test_fekf_bs1_is_rlekf():
    """Alg. 1 at bs = 1 with the sign trick equals RLEKF with epsilon = y - h."""
    rng = np.random.default_rng(4)
    blocks = [4, 6]
    P0 = [_rand_spd(rng, n) for n in blocks]
    st = O.FEKF(np.zeros(10), blocks, lam=0.98, nu=0.9987)
    st.P = [p.copy() for p in P0]
    H = rng.standard_normal(10)
    eps = -0.37                      # y - h < 0  =>  h >= y  =>  flip: g = -H, ABE = |eps|
    st.update(-H, abs(eps), bs=1)
    # RLEKF, layer-wise: a = lam^-1 sum H_i^T P_i H_i + L ; K_i = lam^-1 P_i H_i / a ;
    # P_i = (I - K_i H_i^T) lam^-1 P_i ; w += K eps
    lam, L = 0.98, len(blocks)
    Hs = [H[:4], H[4:]]
    a = sum(h @ p @ h for h, p in zip(Hs, P0)) / lam + L
    K = [p @ h / lam / a for h, p in zip(Hs, P0)]
    Pn = [(np.eye(len(h)) - np.outer(k, h)) @ p / lam for h, p, k in zip(Hs, P0, K)]
    np.testing.assert_allclose(st.w, np.concatenate(K) * eps, rtol=1e-13)
    for i in range(2):
        np.testing.assert_allclose(st.P[i], Pn[i], rtol=1e-12, atol=1e-14)


# Naive-EKF (fusiform; readings N1-N4)
def test_naive_one_sample_is_rlekf():
    """bs = 1: E(K . ABE) = K . ABE, the single-sample EKF (RLEKF) written out independently."""
    rng = np.random.default_rng(21)
    blocks = [4, 6]
    P0 = [_rand_spd(rng, n) for n in blocks]
    st = O.NaiveEKF(np.zeros(10), blocks, lam=0.98, nu=0.9987)
    st.P = [p.copy() for p in P0]
    H = rng.standard_normal(10)
    eps = 0.41
    st.update_naive([H], [eps])
    lam, L = 0.98, len(blocks)
    Hs = [H[:4], H[4:]]
    a = sum(h @ p @ h for h, p in zip(Hs, P0)) / lam + L
    K = [p @ h / lam / a for h, p in zip(Hs, P0)]
    Pn = [(np.eye(len(h)) - np.outer(k, h)) @ p / lam for h, p, k in zip(Hs, P0, K)]
    np.testing.assert_allclose(st.w, np.concatenate(K) * eps, rtol=1e-13)
    for i in range(2):
        np.testing.assert_allclose(st.P[i], Pn[i], rtol=1e-12, atol=1e-14)


def test_naive_scalar_closed_form():
    """1 x 1 P: A_i = 1/(lam + g_i^2 p), P' = (p / lam) mean_i(lam / (lam + g_i^2 p)),
    w' = w + mean_i(ABE_i A_i p g_i) — the averaged scalar Kalman filter by hand."""
    p, lam = 1.7, 0.95
    g = np.array([0.3, -1.1, 2.0, 0.05])
    abe = np.array([0.2, 0.7, 0.01, 1.3])
    st = O.NaiveEKF(np.array([0.5]), [1], lam=lam, nu=0.99)
    st.P = [np.array([[p]])]
    st.update_naive([np.array([x]) for x in g], abe)
    A = 1.0 / (lam + g * g * p)
    assert st.P[0][0, 0] == pytest.approx(p / lam * np.mean(lam * A), rel=1e-14)
    assert st.w[0] == pytest.approx(0.5 + np.mean(abe * A * p * g), rel=1e-14)
    assert st.lam == pytest.approx(lam * 0.99 + 0.01, abs=4e-16)


def test_naive_identical_samples_and_permutation():
    """n copies of one sample = that sample alone; the update is invariant under sample order;
    P stays symmetric positive definite; the per-sample P_i obey Sherman-Morrison (1 block: c = lam)."""
    rng = np.random.default_rng(5)
    blocks = [7]
    P0 = _rand_spd(rng, 7)
    g = rng.standard_normal(7)
    one = O.NaiveEKF(np.zeros(7), blocks, lam=0.97, nu=0.99)
    one.P = [P0.copy()]
    one.update_naive([g], [0.3])
    many = O.NaiveEKF(np.zeros(7), blocks, lam=0.97, nu=0.99)
    many.P = [P0.copy()]
    many.update_naive([g] * 5, [0.3] * 5)
    np.testing.assert_allclose(many.P[0], one.P[0], rtol=1e-13, atol=1e-15)
    np.testing.assert_allclose(many.w, one.w, rtol=1e-13, atol=1e-16)
    # Sherman-Morrison: P_1 = (P0^-1 + g g^T / lam)^-1 / lam
    np.testing.assert_allclose(one.P[0], np.linalg.inv(np.linalg.inv(P0) + np.outer(g, g) / 0.97) / 0.97,
                               rtol=1e-11, atol=1e-13)
    G = [rng.standard_normal(7) for _ in range(6)]
    ab = list(rng.uniform(0.1, 1.0, 6))
    a = O.NaiveEKF(np.zeros(7), blocks, lam=0.97, nu=0.99)
    a.P = [P0.copy()]
    a.update_naive(G, ab)
    perm = [3, 0, 5, 1, 4, 2]
    b = O.NaiveEKF(np.zeros(7), blocks, lam=0.97, nu=0.99)
    b.P = [P0.copy()]
    b.update_naive([G[i] for i in perm], [ab[i] for i in perm])
    np.testing.assert_allclose(a.P[0], b.P[0], rtol=1e-13, atol=1e-15)
    np.testing.assert_allclose(a.w, b.w, rtol=1e-13, atol=1e-16)
    assert np.array_equal(a.P[0], a.P[0].T)
    np.linalg.cholesky(a.P[0])
    # the mean of per-sample SPD matrices, each (P0^-1 + g_i g_i^T / lam)^-1 / lam
    ref = sum(np.linalg.inv(np.linalg.inv(P0) + np.outer(x, x) / 0.97) / 0.97 for x in G) / 6
    np.testing.assert_allclose(a.P[0], ref, rtol=1e-10, atol=1e-12)


def test_naive_train_step_runs():
    wl, m, ds, w = _setup("t2_tiny", n=2)
    st = O.NaiveEKF.create(w, m, wl.opt)
    out = O.naive_train_step(st, ds["coord"], ds["box"], ds["types"], ds["energy"], ds["force"],
                             force_groups(len(ds["types"]), 0, 9), m)
    assert len(out["abe_f"]) == 4 and len(out["A_e"]) == 2
    assert np.all(np.isfinite(st.w)) and st.t == 5
    for P in st.P:
        np.linalg.cholesky(P)


def test_lambda_closed_form(gold):
    lam0, nu = gold["lambda"]["lambda0"], gold["lambda"]["nu"]
    st = O.FEKF(np.zeros(2), [2], lam=lam0, nu=nu)
    st.P = [np.eye(2)]
    for t in range(1, 400):
        st.update(np.array([0.1, -0.2]), 0.0, 1)
        assert abs(st.lam - (1 - (1 - lam0) * nu ** t)) < 1e-13   # Eq. 3 iterated


def test_train_step_runs_and_is_deterministic():
    wl, m, ds, w = _setup("t2_tiny", n=3)
    res = []
    for _ in range(2):
        st = O.FEKF.create(w, m, wl.opt)
        out = O.train_step(st, ds["coord"], ds["box"], ds["types"], ds["energy"], ds["force"],
                           force_groups(len(ds["types"]), 0, 9), m, wl.opt)
        res.append((st.w.copy(), [p.copy() for p in st.P], out))
    assert np.array_equal(res[0][0], res[1][0])
    assert res[0][2]["lambda"] == pytest.approx(1 - 0.02 * 0.9987 ** 5, abs=1e-15)
    assert len(res[0][2]["abe_f"]) == 4
