"""C-ABI library: loads, exports every symbol include/fekf.h declares, host-only planners agree with
the oracle's layout / block split.  CPU only (no compute calls)."""
import os
import re

import numpy as np
import pytest

import oracle as O
from fixtures import get_config, CONFIGS
import paper_conf_ppopp_huzslmlwtj24_b200 as fk

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    src = open(os.path.join(ROOT, "include", "fekf.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(fekf_[a-z_0-9]+)\s*\(", src)))


def test_library_exports_every_declared_symbol():
    L = fk.lib()
    decl = _declared()
    assert len(decl) >= 30
    for name in decl:
        assert hasattr(L, name), name
    assert set(decl) == set(fk.EXPORTED)
    assert L.fekf_version() == 2


@pytest.mark.parametrize("name", sorted(CONFIGS))
def test_plan_layout_matches_oracle(name):
    m = get_config(name).model
    n, blocks = fk.plan_layout(m, 10240)
    assert n == O.param_count(m)
    sizes = [int(np.prod(s)) for _, s in O.param_tensors(m)]
    assert blocks == O.block_split(sizes, 10240)
    n2, b2 = fk.plan_layout(m, 1024)
    assert n2 == n and b2 == O.block_split(sizes, 1024)


def test_plan_layout_paper_pins():
    m = get_config("paper_cu108").model
    n, blocks = fk.plan_layout(m, 10240)
    assert n == 26651 and blocks == [1350, 10240, 9760, 5301]


@pytest.mark.parametrize("world", [1, 2, 3, 8])
def test_plan_shard_partitions_tiles(world):
    blocks = [1350, 10240, 9760, 5301]
    owners, tiles = None, []
    for r in range(world):
        tl, bl, own = fk.plan_shard(blocks, world, r)
        tiles.append(tl)
        assert bl == tl * 64 * 64 * 8
        if owners is None:
            owners = own
        assert own == owners                       # every rank computes the same plan
    nt = [(n + 63) // 64 for n in blocks]
    assert len(owners) == sum(x * (x + 1) // 2 for x in nt)
    for r in range(world):
        assert owners.count(r) == tiles[r]
    # LPT balance: no rank above the mean by more than one work item (32 tiles)
    assert max(tiles) - sum(tiles) / world <= 32


def test_bad_config_rejected():
    m = dict(ntypes=1, rcut=4.0, rcut_smth=5.0, sel=[10], emb=[4], m2=2, fit=[8])
    with pytest.raises(fk.FekfError):
        fk.plan_layout(m, 100)


def test_opt_defaults_follow_the_paper():
    """P:L221 (lambda, nu; the bs > 1024 preset) and P:L293 (N_b, 4 force updates) from the golden file."""
    import json
    gold = json.load(open(os.path.join(ROOT, "tests", "golden", "paper_model.json")))
    lam = gold["lambda"]
    d = fk.opt_defaults(64)
    assert d["lambda0"] == lam["lambda0"] and d["nu"] == lam["nu"]
    assert d["block_size"] == gold["block_size"]["value"] and d["force_groups"] == 4
    assert fk.opt_defaults(1024)["lambda0"] == lam["lambda0"]
    big = fk.opt_defaults(4096)
    assert big["lambda0"] == lam["lambda0_large"] and big["nu"] == lam["nu_large"]
    with pytest.raises(fk.FekfError):
        fk.opt_defaults(0)


def test_net_precision_knob():
    """fekf_opt_cfg.net_precision (reading Z22): fekf_opt_defaults sets 0 (follow `precision`); the binding
    accepts 0 / 32 / 64 and rejects anything else before any C call."""
    d = fk.opt_defaults(32)
    assert d["precision"] == 64 and d["net_precision"] == 0
    for v in (0, 32, 64):
        assert fk.opt_cfg({**d, "net_precision": v}).net_precision == v
    with pytest.raises(ValueError):
        fk.opt_cfg({**d, "net_precision": 16})
