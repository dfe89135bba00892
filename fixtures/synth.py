"""Seeded synthetic workloads (inputs only; see package docstring).

Every generator takes an explicit seed and uses numpy's PCG64, so the same call produces
byte-identical arrays on every machine.  The recipe for each configuration is written out in
DESIGN.md section "Input recipe"; the shapes follow BASELINE.json `configs` and SURVEY.md §8(d).

Layout conventions shared by both sides (interfaces, not arithmetic):
  coord  float64 [n_img, n_atoms, 3]   Cartesian, Angstrom
  box    float64 [n_img, 3, 3]         rows are the lattice vectors a, b, c
  types  int32   [n_atoms]             same for every image; atoms sorted by type
  energy float64 [n_img]               eV
  force  float64 [n_img, n_atoms, 3]   eV/Angstrom
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field, asdict

import numpy as np

__all__ = [
    "ModelConfig", "OptConfig", "SystemSpec", "CONFIGS", "get_config",
    "make_dataset", "init_weights", "tensor_shapes", "batch_schedule", "force_groups",
    "lj_energy_forces", "random_rotation",
]

SEED_BASE = 20240302


# ----------------------------------------------------------------------------------------------
# configuration records (plain data)
# ----------------------------------------------------------------------------------------------
@dataclass
class ModelConfig:
    """DeePMD se_a hyper-parameters."""
    ntypes: int
    rcut: float
    rcut_smth: float
    sel: list
    emb: list            # embedding widths d_1..d_E  (M = d_E)
    m2: int              # M^< (16)
    fit: list            # fitting hidden widths h_1..h_F
    fit_resnet_dt: int = 1   # SURVEY §8c Z14, pinned by the 26 651 count
    switch_kind: int = 0     # Z8: 0 = C2 quintic sw(u), 1 = cosine 0.5 cos(pi u) + 0.5
    type_one_side: int = 0   # Z15: 0 = embedding net per (t_i, t_j), 1 = per neighbour type t_j only
    env_avg: list = None     # Z11: per centre type [ntypes][4] shift of the R~ rows (None = 0)
    env_std: list = None     # Z11: per centre type [ntypes][4] scale of the R~ rows (None = 1)

    @property
    def nm(self):
        return int(sum(self.sel))

    @property
    def M(self):
        return int(self.emb[-1])


@dataclass
class OptConfig:
    """FEKF hyper-parameters (Alg. 1)."""
    lambda0: float = 0.98
    nu: float = 0.9987
    block_size: int = 10240
    noise_mode: int = 0      # 0: c = L*lambda (RLEKF); 1: c = lambda (Alg. 1 line 8)
    grad_reduce: int = 0     # 0: sum over the global batch (Alg. 1 line 7); 1: mean (Eq. 1)
    force_groups: int = 4
    atoms_per_group: int = 6
    p_defer: int = 15        # CUDA path only: deferred rank-1 corrections of P (same P up to rounding)
    precision: int = 64      # CUDA path only: 32 = the fp32 variant (P stored fp32 and fp32 nets, reading Z22)
    net_precision: int = 0   # CUDA path only: nets' arithmetic, 0 = follow precision, 32 / 64
    p_mode: int = 0          # CUDA path only, world > 1: 0 = P sharded over ranks, 1 = replicated


@dataclass
class SystemSpec:
    name: str
    kind: str                      # lattice builder name
    params: dict = field(default_factory=dict)
    sigma: float = 0.05            # Gaussian position noise, Angstrom
    strain: float = 0.0            # isotropic strain amplitude U(-strain, +strain)
    lj: dict = field(default_factory=dict)   # (ti,tj) -> (eps, sigma); cut
    lj_cut: float = 6.0


@dataclass
class Workload:
    name: str
    system: SystemSpec
    model: ModelConfig
    batch: int
    n_train: int
    n_test: int
    opt: OptConfig = field(default_factory=OptConfig)
    seed: int = SEED_BASE

    def to_dict(self):
        return asdict(self)


# ----------------------------------------------------------------------------------------------
# lattices
# ----------------------------------------------------------------------------------------------
def _fcc(a, cells):
    base = np.array([[0, 0, 0], [0, .5, .5], [.5, 0, .5], [.5, .5, 0]], dtype=np.float64)
    pts = []
    for i in range(cells[0]):
        for j in range(cells[1]):
            for k in range(cells[2]):
                for b in base:
                    pts.append((np.array([i, j, k], dtype=np.float64) + b) * a)
    box = np.diag(np.array(cells, dtype=np.float64) * a)
    return np.array(pts), box, np.zeros(len(pts), dtype=np.int32)


def _diamond(a, cells):
    fcc, box, _ = _fcc(a, cells)
    pts = np.concatenate([fcc, fcc + a * 0.25], axis=0)
    return pts, box, np.zeros(len(pts), dtype=np.int32)


def _rocksalt(a, cells):
    na, box, _ = _fcc(a, cells)
    cl = na + np.array([a / 2, 0, 0])
    pts = np.concatenate([na, cl], axis=0)
    types = np.concatenate([np.zeros(len(na)), np.ones(len(cl))]).astype(np.int32)
    return pts, box, types


def _hcp(a, c, cells):
    a1 = np.array([a, 0, 0]); a2 = np.array([-a / 2, a * math.sqrt(3) / 2, 0]); a3 = np.array([0, 0, c])
    basis = [np.array([0, 0, 0]), np.array([1 / 3, 2 / 3, 0.5])]
    pts = []
    for i in range(cells[0]):
        for j in range(cells[1]):
            for k in range(cells[2]):
                for f in basis:
                    fr = np.array([i, j, k], dtype=np.float64) + f
                    pts.append(fr[0] * a1 + fr[1] * a2 + fr[2] * a3)
    box = np.stack([a1 * cells[0], a2 * cells[1], a3 * cells[2]])
    return np.array(pts), box, np.zeros(len(pts), dtype=np.int32)


def random_rotation(rng):
    """Uniform random rotation matrix (QR of a Gaussian matrix, sign-fixed, det +1)."""
    q, r = np.linalg.qr(rng.standard_normal((3, 3)))
    q = q * np.sign(np.diag(r))
    if np.linalg.det(q) < 0:
        q[:, 0] = -q[:, 0]
    return q


def _molecules(kind, n_side, L, rng):
    """Molecules on an n_side^3 grid (or an (nx, ny, nz) grid of spacing L / n_side[0]) with random
    orientations. Heavy atoms first (type 0)."""
    grid = tuple(n_side) if isinstance(n_side, (tuple, list)) else (n_side, n_side, n_side)
    sp = L / grid[0]
    heavy, light = [], []
    if kind == "water":
        roh, ang = 0.9572, math.radians(104.52)
        local = np.array([[roh, 0, 0], [roh * math.cos(ang), roh * math.sin(ang), 0]])
    elif kind == "ch4":
        rch = 1.09
        t = np.array([[1, 1, 1], [1, -1, -1], [-1, 1, -1], [-1, -1, 1]], dtype=np.float64)
        local = rch * t / math.sqrt(3.0)
    else:
        raise ValueError(kind)
    for i in range(grid[0]):
        for j in range(grid[1]):
            for k in range(grid[2]):
                c = (np.array([i, j, k], dtype=np.float64) + 0.5) * sp
                rot = random_rotation(rng)
                heavy.append(c)
                for v in local:
                    light.append(c + rot @ v)
    pts = np.concatenate([np.array(heavy), np.array(light)], axis=0)
    types = np.concatenate([np.zeros(len(heavy)), np.ones(len(light))]).astype(np.int32)
    return pts, np.diag([sp * g for g in grid]).astype(np.float64), types


def _alloy(a, cells, ntypes, rng):
    """Random substitutional fcc alloy: every site draws a type; atoms are then listed sorted by type
    (stable), so the types stay spatially random while the layout convention holds."""
    pts, box, _ = _fcc(a, cells)
    t = rng.integers(0, ntypes, size=len(pts))
    order = np.argsort(t, kind="stable")
    return pts[order], box, t[order].astype(np.int32)


def build_lattice(spec: SystemSpec, rng):
    p = spec.params
    if spec.kind == "fcc":
        return _fcc(p["a"], p["cells"])
    if spec.kind == "diamond":
        return _diamond(p["a"], p["cells"])
    if spec.kind == "rocksalt":
        return _rocksalt(p["a"], p["cells"])
    if spec.kind == "hcp":
        return _hcp(p["a"], p["c"], p["cells"])
    if spec.kind in ("water", "ch4"):
        return _molecules(spec.kind, p["n_side"], p["L"], rng)
    if spec.kind == "alloy":
        return _alloy(p["a"], p["cells"], p["ntypes"], rng)
    raise ValueError(spec.kind)


# ----------------------------------------------------------------------------------------------
# Lennard-Jones labels (shifted-force), periodic with explicit image enumeration
# ----------------------------------------------------------------------------------------------
def _lj_pair(r, eps, sig, rc):
    """Shifted-force LJ pair energy and dE/dr for r < rc (labels only; not the method)."""
    def phi(x):
        s6 = (sig / x) ** 6
        return 4.0 * eps * (s6 * s6 - s6)

    def dphi(x):
        s6 = (sig / x) ** 6
        return 4.0 * eps * (-12.0 * s6 * s6 + 6.0 * s6) / x

    e = phi(r) - phi(rc) - (r - rc) * dphi(rc)
    de = dphi(r) - dphi(rc)
    return e, de


def lj_energy_forces(coord, box, types, lj, rc):
    """Total energy, per-atom forces and virial of a periodic configuration."""
    n = coord.shape[0]
    inv = np.linalg.inv(box)
    # number of images needed per lattice direction: face spacing h_k = V / |a_l x a_m|
    vol = abs(np.linalg.det(box))
    m = []
    for k in range(3):
        cr = np.cross(box[(k + 1) % 3], box[(k + 2) % 3])
        m.append(int(math.ceil(rc / (vol / np.linalg.norm(cr)))))
    shifts = np.array([[i, j, k] for i in range(-m[0], m[0] + 1)
                       for j in range(-m[1], m[1] + 1) for k in range(-m[2], m[2] + 1)], dtype=np.float64)
    svec = shifts @ box
    del inv
    energy = 0.0
    force = np.zeros_like(coord)
    virial = np.zeros((3, 3))
    for i in range(n):
        d = coord[None, :, :] - coord[i][None, None, :] + svec[:, None, :]     # [S, n, 3]
        r = np.sqrt((d * d).sum(-1))
        ti = types[i]
        for tj in np.unique(types):
            eps, sig = lj[(min(ti, tj), max(ti, tj))]
            mask = (r < rc) & (r > 1e-8) & (types[None, :] == tj)
            rr = r[mask]
            if rr.size == 0:
                continue
            e, de = _lj_pair(rr, eps, sig, rc)
            energy += 0.5 * e.sum()
            dd = d[mask]
            fvec = (de / rr)[:, None] * dd      # dE/dd_ij ; force on i = +dE/dd
            force[i] += fvec.sum(0)
            virial -= 0.5 * (dd[:, :, None] * fvec[:, None, :]).sum(0)
    return energy, force, virial


# ----------------------------------------------------------------------------------------------
# named workloads (BASELINE.json configs)
# ----------------------------------------------------------------------------------------------
_CU_LJ = {(0, 0): (0.4093, 2.338)}
_WATER_LJ = {(0, 0): (0.0067, 3.166), (0, 1): (0.2, 0.855), (1, 1): (0.05, 1.35)}
_CH4_LJ = {(0, 0): (0.0045, 3.4), (0, 1): (0.2, 0.971), (1, 1): (0.01, 1.6)}
_AL_LJ = {(0, 0): (0.392, 2.551)}                  # minimum at 2^(1/6) sigma = 2.864 A = a/sqrt(2)
_SI_LJ = {(0, 0): (0.30, 2.094)}                   # minimum at the Si-Si bond, 2.351 A
_MG_LJ = {(0, 0): (0.20, 2.860)}                   # minimum at a = 3.21 A
_NACL_LJ = {(0, 0): (0.0115, 2.58), (0, 1): (0.10, 2.512), (1, 1): (0.0128, 4.40)}   # Na-Cl min at a/2


def _lorentz_berthelot(eps, sig):
    """Pair (eps_ij, sigma_ij) = (sqrt(eps_i eps_j), (sigma_i + sigma_j)/2) for every type pair."""
    n = len(eps)
    return {(i, j): (math.sqrt(eps[i] * eps[j]), 0.5 * (sig[i] + sig[j])) for i in range(n) for j in range(i, n)}


_ALLOY_LJ = _lorentz_berthelot([0.40, 0.30, 0.35, 0.45], [2.30, 2.40, 2.45, 2.55])


def _workloads():
    w = {}
    w["c1_cu32"] = Workload(
        "c1_cu32",
        SystemSpec("Cu32", "fcc", {"a": 3.615, "cells": (2, 2, 2)}, sigma=0.10, strain=0.01,
                   lj=_CU_LJ, lj_cut=4.0),
        ModelConfig(1, 4.0, 3.0, [48], [8, 16, 32], 4, [32, 32]),
        batch=4, n_train=64, n_test=16, seed=SEED_BASE + 1)
    w["c2_water64"] = Workload(
        "c2_water64",
        SystemSpec("H2O-64", "water", {"n_side": 4, "L": 12.42}, sigma=0.05, lj=_WATER_LJ, lj_cut=6.0),
        ModelConfig(2, 6.0, 0.5, [46, 92], [25, 50, 100], 16, [240, 240, 240]),
        batch=32, n_train=2048, n_test=256, seed=SEED_BASE + 2)
    w["c3a_cu108"] = Workload(
        "c3a_cu108",
        SystemSpec("Cu108", "fcc", {"a": 3.615, "cells": (3, 3, 3)}, sigma=0.10, lj=_CU_LJ, lj_cut=6.0),
        ModelConfig(1, 6.0, 0.5, [96], [25, 50, 100], 16, [240, 240, 240]),
        batch=64, n_train=4096, n_test=512, seed=SEED_BASE + 3)
    w["c3b_ch4"] = Workload(
        "c3b_ch4",
        SystemSpec("CH4-27", "ch4", {"n_side": 3, "L": 11.96}, sigma=0.05, lj=_CH4_LJ, lj_cut=6.0),
        ModelConfig(2, 6.0, 0.5, [32, 96], [25, 50, 100], 16, [240, 240, 240]),
        batch=64, n_train=4096, n_test=512, seed=SEED_BASE + 4)
    w["paper_cu108"] = Workload(
        "paper_cu108",
        SystemSpec("Cu108", "fcc", {"a": 3.615, "cells": (3, 3, 3)}, sigma=0.10, lj=_CU_LJ, lj_cut=6.0),
        ModelConfig(1, 6.0, 0.5, [96], [25, 25, 25], 16, [50, 50, 50]),
        batch=64, n_train=4096, n_test=512, seed=SEED_BASE + 5)
    # tiny two-type case for fast oracle/kernel tests (ragged sections, multi-image PBC)
    w["t2_tiny"] = Workload(
        "t2_tiny",
        SystemSpec("H2O-8", "water", {"n_side": 2, "L": 6.21}, sigma=0.05, lj=_WATER_LJ, lj_cut=4.0),
        ModelConfig(2, 4.0, 1.0, [12, 24], [4, 8, 16], 3, [16, 16]),
        batch=3, n_train=12, n_test=4, seed=SEED_BASE + 6)
    # ---- C4: the 8-system sweep shaped like the paper's Table 3: atom counts of
    # the paper's datasets, perturbed lattices with LJ (Lorentz-Berthelot) labels, C2's nets
    c2_emb, c2_fit = [25, 50, 100], [240, 240, 240]
    w["c4_al32"] = Workload(
        "c4_al32", SystemSpec("Al32", "fcc", {"a": 4.05, "cells": (2, 2, 2)}, sigma=0.10, lj=_AL_LJ, lj_cut=6.0),
        ModelConfig(1, 6.0, 0.5, [64], c2_emb, 16, c2_fit), batch=32, n_train=4096, n_test=512, seed=SEED_BASE + 11)
    w["c4_si72"] = Workload(     # 3x3x1 diamond cells: orthorhombic, c = 5.43 A < 2 r_c (two image shells)
        "c4_si72", SystemSpec("Si72", "diamond", {"a": 5.43, "cells": (3, 3, 1)}, sigma=0.08, lj=_SI_LJ, lj_cut=6.0),
        ModelConfig(1, 6.0, 0.5, [56], c2_emb, 16, c2_fit), batch=32, n_train=4096, n_test=512, seed=SEED_BASE + 12)
    w["c4_nacl64"] = Workload(
        "c4_nacl64", SystemSpec("NaCl64", "rocksalt", {"a": 5.64, "cells": (2, 2, 2)}, sigma=0.08, lj=_NACL_LJ,
                                lj_cut=6.0),
        ModelConfig(2, 6.0, 0.5, [24, 24], c2_emb, 16, c2_fit), batch=32, n_train=4096, n_test=512,
        seed=SEED_BASE + 13)
    w["c4_mg36"] = Workload(     # hcp 3x3x2: a triclinic (hexagonal) cell
        "c4_mg36", SystemSpec("Mg36", "hcp", {"a": 3.21, "c": 5.21, "cells": (3, 3, 2)}, sigma=0.08, lj=_MG_LJ,
                              lj_cut=6.0),
        ModelConfig(1, 6.0, 0.5, [56], c2_emb, 16, c2_fit), batch=32, n_train=4096, n_test=512, seed=SEED_BASE + 14)
    w["c4_h2o48"] = Workload(    # 16 molecules on a 4x2x2 grid at 1 g/cm^3
        "c4_h2o48", SystemSpec("H2O-48", "water", {"n_side": (4, 2, 2), "L": 12.42}, sigma=0.05, lj=_WATER_LJ,
                               lj_cut=6.0),
        ModelConfig(2, 6.0, 0.5, [46, 92], c2_emb, 16, c2_fit), batch=32, n_train=4096, n_test=512,
        seed=SEED_BASE + 15)
    w["c4_alloy108"] = Workload(  # random 4-type fcc alloy (FEKF_MAX_TYPES types)
        "c4_alloy108", SystemSpec("Alloy108", "alloy", {"a": 3.615, "cells": (3, 3, 3), "ntypes": 4}, sigma=0.10,
                                  lj=_ALLOY_LJ, lj_cut=6.0),
        ModelConfig(4, 6.0, 0.5, [40, 40, 40, 40], c2_emb, 16, c2_fit), batch=32, n_train=4096, n_test=512,
        seed=SEED_BASE + 16)
    # C4 time-to-target variants: the same systems with C1-sized nets and minibatch 4, so the fp64 CPU
    # oracle (dense P blocks) can produce the target trajectory (metric (iii)) in minutes
    for key in ["c4_al32", "c4_si72", "c4_nacl64", "c4_mg36", "c4_h2o48", "c4_alloy108"]:
        base = w[key]
        bm = base.model
        name = key.replace("c4_", "c4s_")
        w[name] = Workload(name, base.system, ModelConfig(bm.ntypes, bm.rcut, bm.rcut_smth, list(bm.sel), [8, 16, 32],
                                                          4, [32, 32]),
                           batch=4, n_train=64, n_test=16, seed=base.seed)
    # perfect lattice (sigma = 0, no strain): exact r^2 ties in every shell (tie-break tests); sel 16 cuts
    # the second fcc shell (6 atoms at r = a) in the middle
    w["t_cu32_perfect"] = Workload(
        "t_cu32_perfect", SystemSpec("Cu32", "fcc", {"a": 3.615, "cells": (2, 2, 2)}, sigma=0.0, lj=_CU_LJ,
                                     lj_cut=4.0),
        ModelConfig(1, 4.0, 3.0, [48], [8, 16, 32], 4, [32, 32]), batch=2, n_train=4, n_test=2, seed=SEED_BASE + 17)
    return w


CONFIGS = _workloads()


def get_config(name) -> Workload:
    return CONFIGS[name]


# ----------------------------------------------------------------------------------------------
# datasets
# ----------------------------------------------------------------------------------------------
def make_dataset(name, n_images=None, seed=None, split="train", labels=True):
    """Perturbed periodic snapshots of workload `name` with shifted-force LJ labels.

    Returns dict(coord, box, types, energy, force) as documented in the module docstring.
    `split` selects a disjoint seed stream for train / test.
    """
    wl = CONFIGS[name]
    if n_images is None:
        n_images = wl.n_train if split == "train" else wl.n_test
    seed = wl.seed if seed is None else seed
    rng = np.random.Generator(np.random.PCG64([seed, 0 if split == "train" else 1]))
    base_pts, base_box, types = build_lattice(wl.system, np.random.Generator(np.random.PCG64([seed, 7])))
    n = len(base_pts)
    coord = np.empty((n_images, n, 3))
    box = np.empty((n_images, 3, 3))
    energy = np.zeros(n_images)
    force = np.zeros((n_images, n, 3))
    for k in range(n_images):
        scale = 1.0 + (rng.uniform(-wl.system.strain, wl.system.strain) if wl.system.strain > 0 else 0.0)
        x = base_pts * scale + rng.normal(0.0, wl.system.sigma, size=base_pts.shape)
        bx = base_box * scale
        # wrap into the cell (fractional coordinates in [0,1))
        fr = x @ np.linalg.inv(bx)
        fr -= np.floor(fr)
        x = fr @ bx
        coord[k] = x
        box[k] = bx
        if labels:
            e, f, _ = lj_energy_forces(x, bx, types, wl.system.lj, wl.system.lj_cut)
            energy[k] = e
            force[k] = f
    return {"coord": coord, "box": box, "types": types.astype(np.int32), "energy": energy, "force": force}


# ----------------------------------------------------------------------------------------------
# parameters (flat vector in the layout order of SURVEY §8c step 1; random init Z17)
# ----------------------------------------------------------------------------------------------
def tensor_shapes(m: ModelConfig):
    """[(name, shape)] in storage order: embedding nets (ti,tj) lexicographic (or per tj with
    type_one_side), then fitting nets."""
    out = []
    nets = [f"{tj}" for tj in range(m.ntypes)] if getattr(m, "type_one_side", 0) else \
        [f"{ti}{tj}" for ti in range(m.ntypes) for tj in range(m.ntypes)]
    for nm in nets:
        prev = 1
        for l, d in enumerate(m.emb):
            out.append((f"emb{nm}.W{l}", (prev, d)))
            out.append((f"emb{nm}.b{l}", (d,)))
            prev = d
    for ti in range(m.ntypes):
        prev = m.M * m.m2
        for l, h in enumerate(m.fit):
            out.append((f"fit{ti}.W{l}", (prev, h)))
            out.append((f"fit{ti}.b{l}", (h,)))
            if l > 0 and h == prev and m.fit_resnet_dt:
                out.append((f"fit{ti}.dt{l}", (h,)))
            prev = h
        out.append((f"fit{ti}.Wout", (prev, 1)))
        out.append((f"fit{ti}.bout", (1,)))
    return out


def init_weights(m: ModelConfig, seed, e_atom_mean=0.0):
    """Seeded initial weights: W ~ N(0, 1/(in+out)), b ~ N(0,1), dt ~ N(0.1, 1e-3), b_out = mean E/atom."""
    rng = np.random.Generator(np.random.PCG64([seed, 11]))
    parts = []
    for name, shp in tensor_shapes(m):
        if name.endswith("bout"):
            parts.append(np.full(shp, e_atom_mean, dtype=np.float64))
        elif ".W" in name:
            parts.append(rng.normal(0.0, 1.0 / math.sqrt(shp[0] + shp[1]), size=shp))
        elif ".dt" in name:
            parts.append(rng.normal(0.1, 1e-3, size=shp))
        else:
            parts.append(rng.normal(0.0, 1.0, size=shp))
    return np.concatenate([p.reshape(-1) for p in parts])


# ----------------------------------------------------------------------------------------------
# schedules: which images form each minibatch, which atoms each force update uses
# ----------------------------------------------------------------------------------------------
def batch_schedule(n_train, batch, step, seed):
    """Image indices of minibatch `step`: epochs are seeded permutations, consumed in order."""
    per_epoch = n_train // batch
    epoch, k = divmod(step, per_epoch)
    perm = np.random.Generator(np.random.PCG64([seed, 101, epoch])).permutation(n_train)
    return perm[k * batch:(k + 1) * batch].astype(np.int64)


def force_groups(n_atoms, step, seed, groups=4, apg=6):
    """[groups, apg] atom indices for the force updates of step `step` (no repeats inside a step
    while n_atoms allows; the same atoms for every image of the minibatch)."""
    rng = np.random.Generator(np.random.PCG64([seed, 202, step]))
    need = groups * apg
    if need <= n_atoms:
        idx = rng.choice(n_atoms, size=need, replace=False)
    else:
        idx = rng.integers(0, n_atoms, size=need)
    return idx.reshape(groups, apg).astype(np.int32)
