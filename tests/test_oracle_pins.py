"""Value pins of the CPU oracle's model arithmetic and of the flags added for SURVEY §8(b)/(c)
(switch_kind Z8, env statistics Z11, type_one_side Z15), plus the RMSE criterion and the
minibatch scaling of train_step (Alg. 1 line 7 sum, Eq. 2 sqrt(bs)).  CPU only (`-m "not gpu"`).

Every expected value here comes from something other than the oracle itself: a scalar evaluation with
the `math` module (tests/golden/tiny_model.json, written by tools/make_tiny_golden.py), a closed form,
an equivalence between two model parametrisations, or a statistic computed in the test with numpy.
"""
import json
import math
import os

import numpy as np
import pytest
import torch

import oracle as O
from fixtures import ModelConfig, OptConfig, get_config, make_dataset, init_weights

GOLD = os.path.join(os.path.dirname(__file__), "golden", "tiny_model.json")


def _tiny_case(case, g):
    m = ModelConfig(len(case["sel"]), g["rcut"], g["rcut_smth"], case["sel"], g["emb"], g["m2"], g["fit"], 1,
                    case["switch_kind"], case["type_one_side"], case["env_avg"], case["env_std"])
    coord = np.array([g["coord"]], dtype=np.float64)
    box = np.array([g["box"]], dtype=np.float64)
    types = np.array(case["types"], dtype=np.int32)
    return m, coord, box, types


@pytest.mark.parametrize("k", range(4))
def test_tiny_model_hand_values(k):
    """E_i of hand-sized models (switch, [h,h] skip, 1/N_m, D = X^T X^<, fitting dt, per-type
    nets, Z11 statistics) equal a scalar-by-scalar math-module evaluation."""
    g = json.load(open(GOLD))
    case = g["cases"][k]
    m, coord, box, types = _tiny_case(case, g)
    assert O.param_count(m) == len(case["weights"])
    nl_j, nl_s, ov = O.build_nlist(coord, box, types, m.rcut, m.sel)
    assert ov.sum() == 0
    Ea, E, F, V = O.energy_force_virial(np.array(case["weights"]), coord, box, types, nl_j, nl_s, m)
    np.testing.assert_allclose(Ea[0], case["e_atom"], rtol=0, atol=2e-15)
    assert abs(E[0] - sum(case["e_atom"])) < 1e-14


def test_tiny_model_cases_are_distinguishing():
    """The golden cases differ where the readings differ (a pin that cannot fail pins nothing)."""
    g = json.load(open(GOLD))
    ea = {c["name"]: np.array(c["e_atom"]) for c in g["cases"]}
    assert np.abs(ea["one_type"] - ea["one_type_cosine"]).min() > 1e-6   # every atom has a switched neighbour
    assert np.abs(ea["two_type_pair_nets"] - ea["two_type_one_side_stats"]).min() > 1e-3


def test_rmse_hand_case():
    """P:L299 RMSE = E_rmse (per atom, RMS over images) + F_rmse (RMS over all force components).
    With every weight zero but b_out = c the model predicts E_i = c and F = 0 exactly."""
    wl = get_config("t2_tiny")
    m = wl.model
    ds = make_dataset("t2_tiny", 2)
    na = len(ds["types"])
    c = 0.5
    w = np.zeros(O.param_count(m))
    names = [n for n, _ in O.param_tensors(m)]
    offs = np.cumsum([0] + [int(np.prod(s)) for _, s in O.param_tensors(m)])
    for t in range(m.ntypes):
        w[offs[names.index(f"fit{t}.bout")]] = c
    e_label = np.array([na * c + 0.3 * na, na * c - 0.6 * na])      # per-atom errors -0.3, +0.6
    f_label = np.zeros_like(ds["force"])
    f_label[0, 0, 0] = 3.0
    f_label[1, 2, 1] = -4.0
    e, f = O.rmse(w, ds["coord"], ds["box"], ds["types"], e_label, f_label, m)
    assert e == pytest.approx(math.sqrt((0.09 + 0.36) / 2), rel=1e-14)
    assert f == pytest.approx(math.sqrt((9.0 + 16.0) / (2 * na * 3)), rel=1e-14)


def test_cosine_switch_closed_form():
    """Z8 flag: sw(u) = 0.5 cos(pi u) + 0.5: 3/4 at u = 1/3, 1/4 at u = 2/3, continuous with a zero
    first derivative at both ends (C1), 1/r below r_cs and 0 from r_c on."""
    rcs, rc = 1.0, 4.0
    sw = lambda x: O.switch(np.array([x]), rcs, rc, 1)[0] * x
    assert sw(2.0) == pytest.approx(0.75, abs=1e-15)
    assert sw(3.0) == pytest.approx(0.25, abs=1e-15)
    assert sw(0.5) == 1.0 and sw(rc) == 0.0
    h = 1e-6
    for x0, side, v in ((rcs, +1, 1.0), (rc, -1, 0.0)):
        v1 = sw(x0 + side * h)
        assert abs(v1 - v) < 1e-9 and abs((v1 - v) / h) < 1e-4


def _stats_model(m, avg, std):
    return ModelConfig(**{**m.__dict__, "env_avg": avg, "env_std": std})


def test_env_stats_standardize_valid_rows():
    """Z11: with avg/std computed per centre type from the valid rows (the usual descriptor statistics,
    computed here with numpy), the normalised valid rows have mean 0 and unit std per type and component;
    padded rows stay exactly 0."""
    wl = get_config("t2_tiny")
    m = wl.model
    ds = make_dataset("t2_tiny", 3)
    nl_j, nl_s, _ = O.build_nlist(ds["coord"], ds["box"], ds["types"], m.rcut, m.sel)
    _, R, mask = O.env_mat(torch.as_tensor(ds["coord"]), ds["box"], nl_j, nl_s, m.rcut, m.rcut_smth)
    R, mask = R.numpy(), mask.numpy()
    types = ds["types"]
    avg = np.zeros((m.ntypes, 4))
    std = np.ones((m.ntypes, 4))
    for t in range(m.ntypes):
        rows = R[:, types == t][mask[:, types == t]]
        avg[t] = rows.mean(0)
        std[t] = rows.std(0)
    m2 = _stats_model(m, avg.tolist(), std.tolist())
    _, Rn, mk = O.model_env(m2, torch.as_tensor(ds["coord"]), ds["box"], types, nl_j, nl_s)
    Rn = Rn.numpy()
    assert np.all(Rn[~mk.numpy()] == 0.0)
    for t in range(m.ntypes):
        rows = Rn[:, types == t][mask[:, types == t]]
        np.testing.assert_allclose(rows.mean(0), 0.0, atol=1e-13)
        np.testing.assert_allclose(rows.std(0), 1.0, rtol=1e-12)


def test_env_stats_scale_is_a_weight_transform():
    """Z11 with avg = 0 and one std sigma for all components: every R~ row is divided by sigma, so the
    embedding input s -> s/sigma (W0 -> W0/sigma) and D = X^T X^< -> D/sigma^2 (fitting W0 -> W0/sigma^2):
    E_stats(w) == E_plain(w')."""
    wl = get_config("t2_tiny")
    m = wl.model
    ds = make_dataset("t2_tiny", 2)
    w = init_weights(m, 3, 0.1)
    sig = 1.7
    m2 = _stats_model(m, np.zeros((m.ntypes, 4)).tolist(), np.full((m.ntypes, 4), sig).tolist())
    w2 = w.copy()
    off = 0
    for name, shp in O.param_tensors(m):
        n = int(np.prod(shp))
        if name.startswith("emb") and name.endswith(".W0"):
            w2[off:off + n] /= sig
        if name.startswith("fit") and name.endswith(".W0"):
            w2[off:off + n] /= sig * sig
        off += n
    nl_j, nl_s, _ = O.build_nlist(ds["coord"], ds["box"], ds["types"], m.rcut, m.sel)
    Ea, E, F, V = O.energy_force_virial(w, ds["coord"], ds["box"], ds["types"], nl_j, nl_s, m2)
    Eb, E2, F2, V2 = O.energy_force_virial(w2, ds["coord"], ds["box"], ds["types"], nl_j, nl_s, m)
    np.testing.assert_allclose(Ea, Eb, rtol=1e-13, atol=1e-14)
    np.testing.assert_allclose(F, F2, rtol=1e-12, atol=1e-13)


def test_type_one_side_equals_duplicated_pair_nets():
    """Z15 flag: one embedding net per neighbour type t_j gives the model in which the per-pair net
    (t_i, t_j) is a copy of net t_j for every t_i."""
    wl = get_config("t2_tiny")
    m = wl.model
    m1 = ModelConfig(**{**m.__dict__, "type_one_side": 1})
    ds = make_dataset("t2_tiny", 2)
    w1 = init_weights(m1, 5, 0.1)
    p1 = dict(zip([n for n, _ in O.param_tensors(m1)],
                  np.split(w1, np.cumsum([int(np.prod(s)) for _, s in O.param_tensors(m1)])[:-1])))
    assert O.param_count(m) - O.param_count(m1) == (m.ntypes - 1) * m.ntypes * sum(
        (a + 1) * b for a, b in zip([1] + m.emb[:-1], m.emb))
    parts = []
    for name, shp in O.param_tensors(m):
        if name.startswith("emb"):
            tj = name[4]
            parts.append(p1["emb" + tj + name[5:]])
        else:
            parts.append(p1[name])
    w2 = np.concatenate(parts)
    nl_j, nl_s, _ = O.build_nlist(ds["coord"], ds["box"], ds["types"], m.rcut, m.sel)
    Ea, _, Fa, _ = O.energy_force_virial(w1, ds["coord"], ds["box"], ds["types"], nl_j, nl_s, m1)
    Eb, _, Fb, _ = O.energy_force_virial(w2, ds["coord"], ds["box"], ds["types"], nl_j, nl_s, m)
    assert np.array_equal(Ea, Eb) and np.array_equal(Fa, Fb)


@pytest.mark.parametrize("flags", [dict(switch_kind=1), dict(type_one_side=1),
                                   dict(env_avg=[[0.1, 0.0, 0.0, 0.0], [-0.2, 0.0, 0.0, 0.0]],
                                        env_std=[[0.6, 0.8, 0.8, 0.8], [1.3, 0.9, 0.9, 0.9]])])
def test_flag_models_forces_are_minus_grad_energy(flags):
    """F = -dE/dx by central differences for every flag variant (h = 1e-5, rel 1e-6)."""
    wl = get_config("t2_tiny")
    m = ModelConfig(**{**wl.model.__dict__, **flags})
    ds = make_dataset("t2_tiny", 1)
    w = init_weights(m, 3, 0.1)
    coord, box, types = ds["coord"], ds["box"], ds["types"]
    nl_j, nl_s, _ = O.build_nlist(coord, box, types, m.rcut, m.sel)
    _, E, F, _ = O.energy_force_virial(w, coord, box, types, nl_j, nl_s, m)
    h = 1e-5
    rng = np.random.default_rng(1)
    for a in rng.choice(len(types), 4, replace=False):
        for al in range(3):
            cp, cm = coord.copy(), coord.copy()
            cp[0, a, al] += h
            cm[0, a, al] -= h
            ep = O.energy_force_virial(w, cp, box, types, nl_j, nl_s, m, need_force=False)[1][0]
            em = O.energy_force_virial(w, cm, box, types, nl_j, nl_s, m, need_force=False)[1][0]
            fd = -(ep - em) / (2 * h)
            assert abs(fd - F[0, a, al]) <= 1e-6 * max(1.0, np.abs(F).max())


def test_train_step_energy_update_batch_scaling():
    """Alg. 1 line 7 (g summed over the minibatch, Z2), Eq. 2 (sqrt(bs), Z3) and the batch-mean ABE:
    B identical images give g_B = B g_1 and the same ABE, so from P = I the energy update is
    dw_B = sqrt(B) ABE B g_1 / (c + B^2 |g_1|^2) = r dw_1 with r = sqrt(B) B (c + |g_1|^2) / (c + B^2 |g_1|^2)."""
    wl = get_config("t2_tiny")
    m = wl.model
    ds = make_dataset("t2_tiny", 1)
    w = init_weights(m, 3, float(ds["energy"].mean() / len(ds["types"])))
    opt = OptConfig(block_size=1 << 30)            # one block: c = lambda
    B = 4
    rep = lambda x: np.repeat(x, B, axis=0)
    st1 = O.FEKF.create(w, m, opt)
    O.train_step(st1, ds["coord"], ds["box"], ds["types"], ds["energy"], ds["force"], [], m, opt)
    stB = O.FEKF.create(w, m, opt)
    O.train_step(stB, rep(ds["coord"]), rep(ds["box"]), ds["types"], rep(ds["energy"]), rep(ds["force"]), [], m, opt)
    nl_j, nl_s, _ = O.build_nlist(ds["coord"], ds["box"], ds["types"], m.rcut, m.sel)
    g1, _, _ = O.energy_grad(w, ds["coord"], ds["box"], ds["types"], nl_j, nl_s, ds["energy"], m)
    c = opt.lambda0
    gg = float(g1 @ g1)
    r = math.sqrt(B) * B * (c + gg) / (c + B * B * gg)
    dw1 = st1.w - w
    np.testing.assert_allclose(stB.w - w, r * dw1, rtol=1e-11, atol=1e-13 * np.abs(dw1).max())
