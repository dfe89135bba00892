"""Seeded synthetic inputs shared by the oracle tests, the CUDA parity tests and bench.py.

This package holds NONE of the method's arithmetic (no neighbour list, no descriptor, no network,
no Kalman filter).  It only produces inputs: periodic lattices shaped like the paper's datasets
(Table 3), Lennard-Jones labels, random initial weights, and the per-step
image / force-atom schedules.
"""
from .synth import *  # noqa: F401,F403
