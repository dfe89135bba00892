"""Multi-process (world_size 2, gloo, CPU) checks of the N>1 path's host logic and decomposition:

  * every rank builds the same P shard plan and the ranks' tiles partition the packed P exactly;
  * the early reduction: per-rank gradient/error sums all-reduced over ranks equal the
    single-process sums over the whole minibatch (oracle, fp64);
  * sharded P: per-rank partial u from the rank's own packed tiles (row + transposed contributions),
    all-reduced, equals P g — the exchange the CUDA path does with ncclAllReduce;
  * Naive-EKF over ranks: all-gathered per-sample gradients, all-reduced partial U, per-rank rank-n
    correction of the owned tiles == oracle.NaiveEKF on the global samples.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle as O
from fixtures import get_config, make_dataset, init_weights
import paper_conf_ppopp_huzslmlwtj24_b200 as fk

WORLD = 2
TILE = 64


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _tiles(blocks):
    """Canonical packed tile order: block, strip I, J = I..nt-1 (segments of 32 tiles)."""
    out = []
    for b, n in enumerate(blocks):
        nt = (n + TILE - 1) // TILE
        for I in range(nt):
            for J0 in range(I, nt, 32):
                for J in range(J0, min(nt, J0 + 32)):
                    out.append((b, I, J))
    return out


def _worker(rank, port, q):
    try:
        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
        dist.init_process_group("gloo", rank=rank, world_size=WORLD)
        torch.set_num_threads(2)
        res = {}
        # 1. shard plan
        blocks = [1350, 10240, 9760, 5301]
        tl, bl, owner = fk.plan_shard(blocks, WORLD, rank)
        t = torch.tensor([tl], dtype=torch.int64)
        allt = [torch.zeros(1, dtype=torch.int64) for _ in range(WORLD)]
        dist.all_gather(allt, t)
        o = torch.tensor(owner, dtype=torch.int32)
        o0 = o.clone()
        dist.broadcast(o0, 0)
        res["plan_same"] = bool(torch.equal(o, o0))
        res["plan_counts"] = [int(x) for x in allt] == [owner.count(r) for r in range(WORLD)]
        res["plan_total"] = sum(int(x) for x in allt) == len(owner)

        # 2. early reduction of [g || error sum] over ranks
        name = "t2_tiny"
        wl = get_config(name)
        m = wl.model
        ds = make_dataset(name, 4)
        w = init_weights(m, 3, float(ds["energy"].mean() / len(ds["types"])))
        sl = slice(2 * rank, 2 * rank + 2)
        nl = O.build_nlist(ds["coord"][sl], ds["box"][sl], ds["types"], m.rcut, m.sel)
        g, s, _ = O.energy_grad(w, ds["coord"][sl], ds["box"][sl], ds["types"], nl[0], nl[1], ds["energy"][sl], m)
        buf = torch.tensor(np.concatenate([g, [s]]))
        dist.all_reduce(buf)
        nlf = O.build_nlist(ds["coord"], ds["box"], ds["types"], m.rcut, m.sel)
        gf, sf, _ = O.energy_grad(w, ds["coord"], ds["box"], ds["types"], nlf[0], nlf[1], ds["energy"], m)
        res["early_reduction"] = float(np.abs(buf.numpy()[:-1] - gf).max() / np.abs(gf).max())
        res["err_sum"] = abs(float(buf[-1]) - sf)

        # 3. sharded P: partial u from owned tiles, all-reduced
        blocks = [70, 200, 130]
        rng = np.random.default_rng(3)
        Ps = []
        for n in blocks:
            a = rng.standard_normal((n, n))
            Ps.append(a @ a.T / n + np.eye(n))
        gv = rng.standard_normal(sum(blocks))
        _, _, owner = fk.plan_shard(blocks, WORLD, rank)
        off = np.concatenate([[0], np.cumsum(blocks)])
        u = np.zeros(sum(blocks))
        mine = 0
        for (b, I, J), ow in zip(_tiles(blocks), owner):
            if ow != rank:
                continue
            mine += 1
            n = blocks[b]
            r0, r1 = I * TILE, min(n, (I + 1) * TILE)
            c0, c1 = J * TILE, min(n, (J + 1) * TILE)
            if r0 >= n or c0 >= n:
                continue
            Pt = Ps[b][r0:r1, c0:c1]
            gb = gv[off[b]:off[b + 1]]
            u[off[b] + r0:off[b] + r1] += Pt @ gb[c0:c1]
            if I != J:
                u[off[b] + c0:off[b] + c1] += Pt.T @ gb[r0:r1]
        ut = torch.tensor(u)
        dist.all_reduce(ut)
        ref = np.concatenate([Ps[b] @ gv[off[b]:off[b + 1]] for b in range(len(blocks))])
        res["sharded_u"] = float(np.abs(ut.numpy() - ref).max() / np.abs(ref).max())
        res["mine"] = mine

        # 4. Naive-EKF over ranks (readings N1-N4): each rank's local samples' gradients and
        #    errors are all-gathered, the partial U = P G of the rank's tiles is all-reduced (instead of
        #    the paper's P all-reduce), then every rank applies the same w step and the rank-n correction
        #    to its own tiles; equals oracle.NaiveEKF over the global samples
        lam, L = 0.98, len(blocks)
        Gl = rng.standard_normal((2, sum(blocks))) + rank      # this rank's 2 samples (differ per rank)
        al = np.abs(rng.standard_normal(2)) + 0.1 * rank
        Gt = [torch.zeros(2, sum(blocks), dtype=torch.float64) for _ in range(WORLD)]
        At = [torch.zeros(2, dtype=torch.float64) for _ in range(WORLD)]
        dist.all_gather(Gt, torch.tensor(Gl))
        dist.all_gather(At, torch.tensor(al))
        G = torch.cat(Gt).numpy()
        ab = torch.cat(At).numpy()
        nS = len(G)
        U = np.zeros((sum(blocks), nS))
        for (b, I, J), ow in zip(_tiles(blocks), owner):
            if ow != rank:
                continue
            n = blocks[b]
            r0, r1 = I * TILE, min(n, (I + 1) * TILE)
            c0, c1 = J * TILE, min(n, (J + 1) * TILE)
            if r0 >= n or c0 >= n:
                continue
            Pt = Ps[b][r0:r1, c0:c1]
            U[off[b] + r0:off[b] + r1] += Pt @ G[:, off[b] + c0:off[b] + c1].T
            if I != J:
                U[off[b] + c0:off[b] + c1] += Pt.T @ G[:, off[b] + r0:off[b] + r1].T
        Ut = torch.tensor(U)
        dist.all_reduce(Ut)
        U = Ut.numpy()
        A = 1.0 / (L * lam + np.einsum("pi,ip->i", U, G))
        dw = U @ (ab * A) / nS
        st = O.NaiveEKF(np.zeros(sum(blocks)), blocks, lam=lam, nu=0.9987)
        st.P = [P.copy() for P in Ps]
        A_ref = st.update_naive(list(G), list(ab))
        res["naive_A"] = float(np.abs(A - np.array(A_ref)).max() / np.abs(A_ref).max())
        res["naive_w"] = float(np.abs(dw - st.w).max() / np.abs(st.w).max())
        err = 0.0
        for (b, I, J), ow in zip(_tiles(blocks), owner):
            if ow != rank:
                continue
            n = blocks[b]
            r0, r1 = I * TILE, min(n, (I + 1) * TILE)
            c0, c1 = J * TILE, min(n, (J + 1) * TILE)
            if r0 >= n or c0 >= n:
                continue
            Ub = U[off[b]:off[b + 1]]
            Pn = (Ps[b][r0:r1, c0:c1] - (Ub[r0:r1] * (A / nS)) @ Ub[c0:c1].T) / lam
            err = max(err, float(np.abs(Pn - st.P[b][r0:r1, c0:c1]).max() / np.abs(st.P[b]).max()))
        res["naive_P"] = err
        q.put((rank, res))
        dist.destroy_process_group()
    except Exception as e:  # pragma: no cover
        q.put((rank, {"error": repr(e)}))


def test_gloo_world2():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, port, q)) for r in range(WORLD)]
    for p in ps:
        p.start()
    out = dict(q.get(timeout=300) for _ in range(WORLD))
    for p in ps:
        p.join(60)
    for r in range(WORLD):
        res = out[r]
        assert "error" not in res, res
        assert res["plan_same"] and res["plan_counts"] and res["plan_total"]
        assert res["early_reduction"] < 1e-12
        assert res["err_sum"] < 1e-13
        assert res["sharded_u"] < 1e-12
        assert res["mine"] > 0
        assert res["naive_A"] < 1e-12 and res["naive_w"] < 1e-12 and res["naive_P"] < 1e-12
