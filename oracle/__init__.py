"""FEKF / DeePMD se_a ORACLE — test infrastructure, not product code.

Only `tests/`, `__graft_entry__.smoke()` and `bench.py` (its `cpu_baseline` leg and `--impl reference`)
may import this package.  The product path (`paper_conf_ppopp_huzslmlwtj24_b200`) never imports it and
fails loudly when its CUDA library is missing.

Plain, slow, fp64 CPU implementation written from PAPER.md (Hu et al., PPoPP'24).  Citations are
`P:Lnnn` = /root/reference/PAPER.md line nnn.  See `oracle/fekf_oracle.py` for the per-function
citations, and DESIGN.md "Readings" for every place where the paper is silent or garbled.
"""
from .fekf_oracle import *  # noqa: F401,F403
