"""B200-native minibatch FEKF training of DeePMD se_a (Hu et al., PPoPP'24), sm_100a.

The compute path is libfekf.so (csrc/, C ABI in include/fekf.h); `fekf` is its ctypes binding.
"""
from .fekf import (Comm, Context, FekfError, KalmanFilter, lib, model_cfg, opt_cfg, opt_defaults, plan_layout,  # noqa: F401
                   plan_shard, EXPORTED, LIB_PATH)
