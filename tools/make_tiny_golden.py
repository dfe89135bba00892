#!/usr/bin/env python
"""Writes tests/golden/tiny_model.json: per-atom energies of hand-sized DeePMD se_a models, computed
scalar by scalar with the `math` module only (no numpy, no torch, no oracle/), so they pin the oracle's
vectorised model (oracle.model_energy / energy_force_virial) to an independent evaluation of the
paper's formulas:

  R~ row of neighbour j of atom i:  s(r) (1, d_x/r, d_y/r, d_z/r), d = x_j - x_i
      s(r) = sw(u)/r, u = (r - r_cs)/(r_c - r_cs), sw = 1 (r < r_cs),
      quintic u^3(-6u^2 + 15u - 10) + 1 (Z8) or cosine 0.5 cos(pi u) + 0.5 (Z8 flag)
      optional statistics: (row - avg[t_i]) / std[t_i] on valid rows (Z11 flag)
  embedding (Z12):  h0 = tanh(s W0 + b0);  layer 1 doubles the width:
      h1[c] = h0[c mod d0] + tanh(sum_k h0[k] W1[k][c] + b1[c])      (the [h, h] skip)
  descriptor (Z13):  X[a][m] = sum_slots R[a] G[m] / N_m ;  D[m][n] = sum_a X[a][m] X[a][n],
      n < M^<, flattened row-major
  fitting (Z14):  f0 = tanh(D W0 + b0);  f1 = f0 + dt * tanh(f0 W1 + b1) (equal widths);
      E_i = f1 . Wout + bout
  net choice (Z15): embedding per (t_i, t_j), or per t_j with type_one_side; fitting per t_i

The configurations are three atoms in a 20 A cubic box (no periodic image within r_c), with one
neighbour distance inside [r_cs, r_c) so the switch polynomial enters, and N_m = 3 > the 2 neighbours
each atom has, so the padding (excluded) and the 1/N_m scale both matter.

  python tools/make_tiny_golden.py
"""
import json
import math
import os

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

COORD = [[1.0, 1.0, 1.0], [2.5, 1.0, 1.0], [1.0, 3.2, 1.0]]   # |AB| = 1.5, |AC| = 2.2, |BC| = 2.6627
BOX = [[20.0, 0.0, 0.0], [0.0, 20.0, 0.0], [0.0, 0.0, 20.0]]
RC, RCS = 3.0, 2.0
EMB = [2, 4]
M2 = 2
FIT = [2, 2]


def weight(k):
    """Deterministic small weights in [-5/8, 5/8], all exactly representable."""
    return ((7 * k + 3) % 11 - 5) / 8.0


def tensor_list(ntypes, one_side):
    """(name, rows, cols) in storage order."""
    out = []
    nets = [f"{tj}" for tj in range(ntypes)] if one_side else [f"{ti}{tj}" for ti in range(ntypes) for tj in range(ntypes)]
    for nm in nets:
        out += [(f"emb{nm}.W0", 1, EMB[0]), (f"emb{nm}.b0", 1, EMB[0]),
                (f"emb{nm}.W1", EMB[0], EMB[1]), (f"emb{nm}.b1", 1, EMB[1])]
    for ti in range(ntypes):
        out += [(f"fit{ti}.W0", EMB[1] * M2, FIT[0]), (f"fit{ti}.b0", 1, FIT[0]),
                (f"fit{ti}.W1", FIT[0], FIT[1]), (f"fit{ti}.b1", 1, FIT[1]), (f"fit{ti}.dt1", 1, FIT[1]),
                (f"fit{ti}.Wout", FIT[1], 1), (f"fit{ti}.bout", 1, 1)]
    return out


def unpack(ntypes, one_side):
    """Flat weight vector w_k = weight(k) and a dict name -> 2-D list view."""
    flat, views, k = [], {}, 0
    for name, r, c in tensor_list(ntypes, one_side):
        mat = []
        for i in range(r):
            row = []
            for j in range(c):
                row.append(weight(k))
                flat.append(weight(k))
                k += 1
            mat.append(row)
        views[name] = mat
    return flat, views


def sw(r, kind):
    if r < RCS:
        return 1.0
    if r >= RC:
        return 0.0
    u = (r - RCS) / (RC - RCS)
    if kind == 1:
        return 0.5 * math.cos(math.pi * u) + 0.5
    return u * u * u * (-6.0 * u * u + 15.0 * u - 10.0) + 1.0


def energies(types, sel, kind, one_side, avg, std):
    ntypes = len(sel)
    nm_slots = sum(sel)
    flat, W = unpack(ntypes, one_side)
    e_atom = []
    for i in range(3):
        ti = types[i]
        X = [[0.0] * EMB[1] for _ in range(4)]
        for j in range(3):
            if j == i:
                continue
            tj = types[j]
            dx = COORD[j][0] - COORD[i][0]
            dy = COORD[j][1] - COORD[i][1]
            dz = COORD[j][2] - COORD[i][2]
            r = math.sqrt(dx * dx + dy * dy + dz * dz)
            if r >= RC:
                continue
            s = sw(r, kind) / r
            R = [s, s * dx / r, s * dy / r, s * dz / r]
            if avg is not None:
                R = [(R[a] - avg[ti][a]) / std[ti][a] for a in range(4)]
            net = f"emb{tj}" if one_side else f"emb{ti}{tj}"
            h0 = [math.tanh(R[0] * W[net + ".W0"][0][c] + W[net + ".b0"][0][c]) for c in range(EMB[0])]
            h1 = []
            for c in range(EMB[1]):
                z = W[net + ".b1"][0][c]
                for k in range(EMB[0]):
                    z += h0[k] * W[net + ".W1"][k][c]
                h1.append(h0[c % EMB[0]] + math.tanh(z))
            for a in range(4):
                for m in range(EMB[1]):
                    X[a][m] += R[a] * h1[m] / nm_slots
        D = []
        for m in range(EMB[1]):
            for n in range(M2):
                D.append(X[0][m] * X[0][n] + X[1][m] * X[1][n] + X[2][m] * X[2][n] + X[3][m] * X[3][n])
        f = f"fit{ti}"
        f0 = []
        for c in range(FIT[0]):
            z = W[f + ".b0"][0][c]
            for q in range(len(D)):
                z += D[q] * W[f + ".W0"][q][c]
            f0.append(math.tanh(z))
        f1 = []
        for c in range(FIT[1]):
            z = W[f + ".b1"][0][c]
            for k in range(FIT[0]):
                z += f0[k] * W[f + ".W1"][k][c]
            f1.append(f0[c] + W[f + ".dt1"][0][c] * math.tanh(z))
        E = W[f + ".bout"][0][0]
        for k in range(FIT[1]):
            E += f1[k] * W[f + ".Wout"][k][0]
        e_atom.append(E)
    return flat, e_atom


CASES = [
    # name, types, sel, switch_kind, type_one_side, env avg/std (per centre type, 4 components)
    ("one_type", [0, 0, 0], [3], 0, 0, None, None),
    ("one_type_cosine", [0, 0, 0], [3], 1, 0, None, None),
    ("two_type_pair_nets", [0, 1, 1], [1, 2], 0, 0, None, None),
    ("two_type_one_side_stats", [0, 1, 1], [1, 2], 0, 1,
     [[0.25, 0.0, 0.0, 0.0], [-0.125, 0.0, 0.0, 0.0]], [[0.5, 0.75, 0.75, 0.75], [2.0, 1.25, 1.25, 1.25]]),
]


def main():
    out = {"_source": "tools/make_tiny_golden.py (math-module scalar evaluation; no oracle, no CUDA path)",
           "_formulas": "P:L83 (R~, s(r)), P:L84-90 (embedding, [h,h] skip Z12), P:L92/P:L233 (X = R~^T G / N_m, "
                        "D = X^T X^<, Z13), P:L95-103 (fitting with dt, Z14), Z8/Z11/Z15 flags",
           "coord": COORD, "box": BOX, "rcut": RC, "rcut_smth": RCS, "emb": EMB, "m2": M2, "fit": FIT,
           "cases": []}
    for name, types, sel, kind, one_side, avg, std in CASES:
        w, ea = energies(types, sel, kind, one_side, avg, std)
        out["cases"].append({"name": name, "types": types, "sel": sel, "switch_kind": kind,
                             "type_one_side": one_side, "env_avg": avg, "env_std": std,
                             "weights": w, "e_atom": ea})
        print(name, len(w), ea)
    path = os.path.join(ROOT, "tests", "golden", "tiny_model.json")
    with open(path, "w") as f:
        json.dump(out, f, indent=1)
    print("wrote", path)


if __name__ == "__main__":
    main()
