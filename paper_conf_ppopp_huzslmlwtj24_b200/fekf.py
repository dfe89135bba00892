"""Thin ctypes binding of libfekf.so (include/fekf.h).  Argument marshalling only: every step of the
FEKF training path runs in the library's sm_100a kernels.  torch is used for device memory, streams
and process groups.  There is no CPU fallback: if the library cannot be loaded, or a tensor is not a
contiguous CUDA tensor of the right dtype, the call raises.
"""
from __future__ import annotations

import ctypes as C
import math
import os

import torch

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libfekf.so")

MAX_TYPES = 4
MAX_LAYERS = 4
TILE = 64

STATUS = {0: "OK", 1: "EINVAL", 2: "ECUDA", 3: "ENCCL", 4: "ENOMEM", 5: "ENLIST_OVERFLOW", 6: "ENONFINITE", 7: "ESTATE"}


class FekfError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"fekf {STATUS.get(status, status)}: {msg}")
        self.status = status


class ModelCfg(C.Structure):
    _fields_ = [("ntypes", C.c_int), ("rcut", C.c_double), ("rcut_smth", C.c_double), ("sel", C.c_int * MAX_TYPES),
                ("n_emb", C.c_int), ("emb", C.c_int * MAX_LAYERS), ("m2", C.c_int), ("n_fit", C.c_int),
                ("fit", C.c_int * MAX_LAYERS), ("fit_resnet_dt", C.c_int), ("switch_kind", C.c_int),
                ("type_one_side", C.c_int)]


class OptCfg(C.Structure):
    _fields_ = [("lambda0", C.c_double), ("nu", C.c_double), ("block_size", C.c_int), ("noise_mode", C.c_int),
                ("grad_reduce", C.c_int), ("force_groups", C.c_int), ("atoms_per_group", C.c_int),
                ("p_defer", C.c_int), ("precision", C.c_int), ("p_mode", C.c_int),
                ("net_precision", C.c_int)]


_lib = None


def lib():
    """Load libfekf.so (built by `python -m paper_conf_ppopp_huzslmlwtj24_b200.build`)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise FekfError(2, f"{LIB_PATH} not built; run `python -m paper_conf_ppopp_huzslmlwtj24_b200.build`")
    L = C.CDLL(LIB_PATH)
    vp, i32, i64, dbl = C.c_void_p, C.c_int, C.c_int64, C.c_double
    sigs = {
        "fekf_last_error": ([], C.c_char_p), "fekf_version": ([], i32),
        "fekf_plan_layout": ([C.POINTER(ModelCfg), i32, C.POINTER(i64), vp, i32, C.POINTER(i32)], i32),
        "fekf_plan_shard": ([vp, i32, i32, i32, C.POINTER(i64), C.POINTER(i64), vp], i32),
        "fekf_get_unique_id": ([vp], i32), "fekf_comm_init": ([i32, i32, vp, C.POINTER(vp)], i32),
        "fekf_comm_destroy": ([vp], i32), "fekf_comm_allreduce_sum": ([vp, vp, i64, vp], i32),
        "fekf_kf_create": ([vp, i32, C.POINTER(OptCfg), vp, C.POINTER(vp)], i32), "fekf_kf_destroy": ([vp], i32),
        "fekf_kf_update": ([vp, vp, vp, dbl, vp, vp], i32), "fekf_kf_flush": ([vp, vp], i32),
        "fekf_opt_defaults": ([i32, C.POINTER(OptCfg)], i32),
        "fekf_kf_create_shard": ([vp, i32, C.POINTER(OptCfg), i32, i32, C.POINTER(vp)], i32),
        "fekf_kf_update_begin": ([vp, vp, vp], i32), "fekf_kf_update_end": ([vp, vp, dbl, vp, vp], i32),
        "fekf_kf_partial_u": ([vp, C.POINTER(vp), C.POINTER(i64)], i32),
        "fekf_kf_get_block": ([vp, i32, vp, vp], i32), "fekf_kf_set_block": ([vp, i32, vp, vp], i32),
        "fekf_kf_get_state": ([vp, C.POINTER(dbl), C.POINTER(dbl), C.POINTER(i32)], i32),
        "fekf_kf_info": ([vp, C.POINTER(i64), C.POINTER(i64), C.POINTER(i64), C.POINTER(i64)], i32),
        "fekf_kf_pass": ([vp, vp, vp], i32),
        "fekf_kf_timing": ([vp, i32, C.POINTER(dbl), C.POINTER(i64), C.POINTER(i64)], i32),
        "fekf_create": ([C.POINTER(ModelCfg), C.POINTER(OptCfg), i32, vp, i32, i32, vp, C.POINTER(vp)], i32),
        "fekf_destroy": ([vp], i32), "fekf_param_count": ([vp, C.POINTER(i64)], i32),
        "fekf_get_kf": ([vp, C.POINTER(vp)], i32), "fekf_set_params": ([vp, vp, vp], i32),
        "fekf_get_params": ([vp, vp, vp], i32),
        "fekf_build_nlist": ([vp, vp, vp, i32, vp, vp, vp, vp], i32),
        "fekf_env_mat": ([vp, vp, vp, vp, vp, i32, vp, vp, vp, vp], i32),
        "fekf_forward": ([vp, vp, vp, i32, vp, vp, vp, vp, vp], i32),
        "fekf_energy_jacobian": ([vp, vp, vp, vp, i32, vp, vp, vp], i32),
        "fekf_force_jacobian": ([vp, vp, vp, vp, vp, i32, i32, vp, vp, vp], i32),
        "fekf_kalman_update": ([vp, vp, vp, i32, i32, vp], i32),
        "fekf_train_step": ([vp, vp, vp, vp, vp, vp, vp, vp], i32),
        "fekf_last_launch_count": ([vp, C.POINTER(i64)], i32),
        "fekf_set_graph_mode": ([vp, i32], i32),
        "fekf_kf_update_naive": ([vp, vp, i64, vp, i32, vp, vp, vp], i32),
        "fekf_kf_timing_parts": ([vp, vp], i32),
        "fekf_kf_update_naive_begin": ([vp, vp, i64, i32, vp], i32),
        "fekf_kf_naive_partial_u": ([vp, C.POINTER(vp), C.POINTER(i64)], i32),
        "fekf_kf_update_naive_end": ([vp, vp, vp, vp, vp], i32),
        "fekf_naive_train_step": ([vp, vp, vp, vp, vp, vp, vp, vp], i32),
        "fekf_set_env_stats": ([vp, vp, vp], i32),
        "fekf_comm_init_loopback": ([i32, vp], i32),
        "fekf_kf_timing_span": ([vp, C.POINTER(dbl)], i32),
    }
    for name, (args, res) in sigs.items():
        f = getattr(L, name)
        f.argtypes = args
        f.restype = res
    _lib = L
    return L


EXPORTED = [
    "fekf_last_error", "fekf_version", "fekf_plan_layout", "fekf_plan_shard", "fekf_get_unique_id",
    "fekf_comm_init", "fekf_comm_destroy", "fekf_comm_allreduce_sum", "fekf_kf_create", "fekf_kf_destroy",
    "fekf_kf_update", "fekf_kf_flush", "fekf_kf_get_block", "fekf_kf_set_block", "fekf_kf_get_state",
    "fekf_opt_defaults", "fekf_kf_create_shard", "fekf_kf_update_begin", "fekf_kf_partial_u", "fekf_kf_update_end",
    "fekf_kf_info", "fekf_kf_pass", "fekf_kf_timing", "fekf_create", "fekf_destroy", "fekf_param_count", "fekf_get_kf",
    "fekf_set_params", "fekf_get_params", "fekf_build_nlist", "fekf_env_mat", "fekf_forward",
    "fekf_energy_jacobian", "fekf_force_jacobian", "fekf_kalman_update", "fekf_train_step",
    "fekf_last_launch_count", "fekf_set_graph_mode", "fekf_kf_update_naive", "fekf_naive_train_step",
    "fekf_kf_timing_parts", "fekf_kf_update_naive_begin", "fekf_kf_naive_partial_u", "fekf_kf_update_naive_end",
    "fekf_set_env_stats", "fekf_comm_init_loopback", "fekf_kf_timing_span",
]


def _check(st):
    if st != 0:
        raise FekfError(st, lib().fekf_last_error().decode(errors="replace"))


def _ptr(t, dtype, name="tensor"):
    if t is None:
        return None
    if not isinstance(t, torch.Tensor) or not t.is_cuda:
        raise FekfError(1, f"{name} must be a CUDA tensor (no CPU fallback)")
    if t.dtype != dtype:
        raise FekfError(1, f"{name} must be {dtype}, got {t.dtype}")
    if not t.is_contiguous():
        raise FekfError(1, f"{name} must be contiguous")
    return C.c_void_p(t.data_ptr())


def _stream(stream=None):
    s = stream if stream is not None else torch.cuda.current_stream()
    return C.c_void_p(s.cuda_stream)


def _get(o, k, default=None):
    if isinstance(o, dict):
        return o.get(k, default)
    return getattr(o, k, default)


def model_cfg(m) -> ModelCfg:
    """ModelCfg from any object/dict with ntypes, rcut, rcut_smth, sel, emb, m2, fit[, fit_resnet_dt]."""
    c = ModelCfg()
    c.ntypes = int(_get(m, "ntypes"))
    c.rcut = float(_get(m, "rcut"))
    c.rcut_smth = float(_get(m, "rcut_smth"))
    sel, emb, fit = list(_get(m, "sel")), list(_get(m, "emb")), list(_get(m, "fit"))
    if len(sel) > MAX_TYPES or len(emb) > MAX_LAYERS or len(fit) > MAX_LAYERS:
        raise FekfError(1, "config exceeds library limits")
    for i, v in enumerate(sel):
        c.sel[i] = int(v)
    c.n_emb = len(emb)
    for i, v in enumerate(emb):
        c.emb[i] = int(v)
    c.m2 = int(_get(m, "m2"))
    c.n_fit = len(fit)
    for i, v in enumerate(fit):
        c.fit[i] = int(v)
    c.fit_resnet_dt = int(_get(m, "fit_resnet_dt", 1))
    c.switch_kind = int(_get(m, "switch_kind", 0) or 0)
    c.type_one_side = int(_get(m, "type_one_side", 0) or 0)
    return c


def opt_cfg(o=None) -> OptCfg:
    c = OptCfg()
    c.lambda0 = float(_get(o, "lambda0", 0.98)) if o is not None else 0.98
    c.nu = float(_get(o, "nu", 0.9987)) if o is not None else 0.9987
    c.block_size = int(_get(o, "block_size", 10240)) if o is not None else 10240
    c.noise_mode = int(_get(o, "noise_mode", 0)) if o is not None else 0
    c.grad_reduce = int(_get(o, "grad_reduce", 0)) if o is not None else 0
    c.force_groups = int(_get(o, "force_groups", 4)) if o is not None else 4
    c.atoms_per_group = int(_get(o, "atoms_per_group", 6)) if o is not None else 6
    c.p_defer = int(_get(o, "p_defer", 15)) if o is not None else 15
    c.precision = int(_get(o, "precision", 64)) if o is not None else 64
    c.p_mode = int(_get(o, "p_mode", 0)) if o is not None else 0
    c.net_precision = int(_get(o, "net_precision", 0) or 0) if o is not None else 0
    if c.net_precision not in (0, 32, 64):
        raise ValueError("net_precision must be 0 (follow precision), 32 or 64")
    if c.p_mode not in (0, 1):
        raise ValueError("p_mode must be 0 (sharded) or 1 (replicated)")
    if c.precision not in (32, 64):
        raise ValueError("precision must be 32 or 64")
    return c


def opt_defaults(global_batch):
    """The paper's optimizer defaults for a global minibatch (lambda/nu 0.98/0.9987, 0.90/0.996
    above 1024 images; N_b 10240, 4 force updates) as a dict for Context / KalmanFilter."""
    c = OptCfg()
    _check(lib().fekf_opt_defaults(int(global_batch), C.byref(c)))
    return {k: getattr(c, k) for k, _ in OptCfg._fields_}


def plan_layout(m, block_size=10240):
    L = lib()
    mc = model_cfg(m)
    n = C.c_int64()
    nb = C.c_int()
    _check(L.fekf_plan_layout(C.byref(mc), block_size, C.byref(n), None, 0, C.byref(nb)))
    arr = (C.c_int32 * nb.value)()
    _check(L.fekf_plan_layout(C.byref(mc), block_size, C.byref(n), arr, nb.value, C.byref(nb)))
    return n.value, list(arr)


def plan_shard(blocks, world, rank):
    L = lib()
    b = (C.c_int32 * len(blocks))(*blocks)
    tl, bl = C.c_int64(), C.c_int64()
    nt = [(n + TILE - 1) // TILE for n in blocks]
    total = sum(x * (x + 1) // 2 for x in nt)
    owner = (C.c_int32 * total)()
    _check(L.fekf_plan_shard(b, len(blocks), world, rank, C.byref(tl), C.byref(bl), owner))
    return tl.value, bl.value, list(owner)


class Comm:
    """Library-owned NCCL communicator; the unique id travels through torch.distributed (any backend)."""

    def __init__(self, rank, world, uid: bytes):
        self.h = C.c_void_p()
        buf = (C.c_ubyte * 128).from_buffer_copy(uid)
        _check(lib().fekf_comm_init(rank, world, buf, C.byref(self.h)))
        self.rank, self.world = rank, world

    @classmethod
    def loopback(cls, world):
        """fekf_comm_init_loopback: `world` rank handles of one in-process group (one GPU, one host thread
        per rank)."""
        arr = (C.c_void_p * world)()
        _check(lib().fekf_comm_init_loopback(world, arr))
        out = []
        for r in range(world):
            c = cls.__new__(cls)
            c.h = C.c_void_p(arr[r])
            c.rank, c.world = r, world
            out.append(c)
        return out

    @staticmethod
    def unique_id() -> bytes:
        buf = (C.c_ubyte * 128)()
        _check(lib().fekf_get_unique_id(buf))
        return bytes(buf)

    @classmethod
    def from_process_group(cls, group=None):
        import torch.distributed as dist
        rank, world = dist.get_rank(group), dist.get_world_size(group)
        uid = cls.unique_id() if rank == 0 else bytes(128)
        t = torch.tensor(list(uid), dtype=torch.uint8)
        if dist.get_backend(group) == "nccl":
            t = t.cuda()
        dist.broadcast(t, 0, group=group)
        return cls(rank, world, bytes(t.cpu().tolist()))

    def allreduce_sum(self, t, stream=None):
        _check(lib().fekf_comm_allreduce_sum(self.h, _ptr(t, torch.float64, "buf"), t.numel(), _stream(stream)))

    def close(self):
        if self.h:
            lib().fekf_comm_destroy(self.h)
            self.h = C.c_void_p()


class KalmanFilter:
    """Blocked FEKF Kalman filter over packed-symmetric P (fekf_kf_*)."""

    def __init__(self, blocks, opt=None, comm: Comm | None = None, _handle=None, _owner=None, shard=None):
        """shard=(world, rank): this rank's P tiles with no communicator; the caller exchanges u
        (update_begin / partial_u / update_end)."""
        self.blocks = list(blocks)
        self._owner = _owner
        self._h = C.c_void_p()
        if _handle is not None:
            if _owner is None:
                self._h = _handle
            self._own = False
        else:
            self.h = C.c_void_p()
            oc = opt_cfg(opt)
            arr = (C.c_int32 * len(self.blocks))(*self.blocks)
            if shard is not None:
                _check(lib().fekf_kf_create_shard(arr, len(self.blocks), C.byref(oc), int(shard[0]), int(shard[1]),
                                                  C.byref(self.h)))
            else:
                _check(lib().fekf_kf_create(arr, len(self.blocks), C.byref(oc), comm.h if comm else None,
                                            C.byref(self.h)))
            self._own = True

    @property
    def h(self):
        # a context's filter follows the context's handle (null once the context is closed)
        return self._owner._kh if self._owner is not None else self._h

    @h.setter
    def h(self, v):
        self._h = v

    def update(self, g, abe, sqrt_bs, w, stream=None):
        _check(lib().fekf_kf_update(self.h, _ptr(g, torch.float64, "g"), _ptr(abe, torch.float64, "abe"),
                                    float(sqrt_bs), _ptr(w, torch.float64, "w"), _stream(stream)))

    def update_naive(self, G, abe, w, A_out=None, stream=None):
        """Naive-EKF update (fekf_kf_update_naive): G [n, ldg] per-sample gradients, abe [n]."""
        if G.dim() != 2 or abe.numel() != G.shape[0]:
            raise FekfError(1, "update_naive: G must be [n, ldg] and abe [n]")
        _check(lib().fekf_kf_update_naive(self.h, _ptr(G, torch.float64, "G"), int(G.stride(0)),
                                          _ptr(abe, torch.float64, "abe"), int(G.shape[0]), _ptr(w, torch.float64, "w"),
                                          _ptr(A_out, torch.float64, "A_out") if A_out is not None else None,
                                          _stream(stream)))

    def update_naive_begin(self, G, stream=None):
        if G.dim() != 2:
            raise FekfError(1, "update_naive_begin: G must be [n, ldg]")
        _check(lib().fekf_kf_update_naive_begin(self.h, _ptr(G, torch.float64, "G"), int(G.stride(0)), int(G.shape[0]),
                                                _stream(stream)))

    def naive_partial_u(self):
        """Zero-copy view of this rank's partial U ([N_pad * roundup8(n)]) between naive begin and end."""
        p, n = C.c_void_p(), C.c_int64()
        _check(lib().fekf_kf_naive_partial_u(self.h, C.byref(p), C.byref(n)))

        class _View:
            __cuda_array_interface__ = {"shape": (n.value,), "typestr": "<f8", "data": (p.value, False),
                                        "version": 2, "strides": None}
        return torch.as_tensor(_View(), device="cuda")

    def update_naive_end(self, abe, w, A_out=None, stream=None):
        _check(lib().fekf_kf_update_naive_end(self.h, _ptr(abe, torch.float64, "abe"), _ptr(w, torch.float64, "w"),
                                              _ptr(A_out, torch.float64, "A_out") if A_out is not None else None,
                                              _stream(stream)))

    def update_begin(self, g, stream=None):
        _check(lib().fekf_kf_update_begin(self.h, _ptr(g, torch.float64, "g"), _stream(stream)))

    def partial_u(self):
        """Zero-copy view of this rank's partial u (padded layout) between update_begin and update_end."""
        p, n = C.c_void_p(), C.c_int64()
        _check(lib().fekf_kf_partial_u(self.h, C.byref(p), C.byref(n)))

        class _View:
            __cuda_array_interface__ = {"shape": (n.value,), "typestr": "<f8", "data": (p.value, False),
                                        "version": 2, "strides": None}
        return torch.as_tensor(_View(), device="cuda")

    def update_end(self, abe, sqrt_bs, w, stream=None):
        _check(lib().fekf_kf_update_end(self.h, _ptr(abe, torch.float64, "abe"), float(sqrt_bs),
                                        _ptr(w, torch.float64, "w"), _stream(stream)))

    def timing_span(self):
        """Summed wall ms of the passes of the last timing window (split passes: early start -> last end)."""
        v = C.c_double()
        _check(lib().fekf_kf_timing_span(self.h, C.byref(v)))
        return v.value

    def timing_parts(self):
        """[early, late, early start -> reverse pass done] summed ms of the last timing window (split pass)."""
        a = (C.c_double * 3)()
        _check(lib().fekf_kf_timing_parts(self.h, a))
        return list(a)

    def pass_only(self, g, stream=None):
        _check(lib().fekf_kf_pass(self.h, _ptr(g, torch.float64, "g"), _stream(stream)))

    def flush(self, stream=None):
        _check(lib().fekf_kf_flush(self.h, _stream(stream)))

    def get_block(self, b, out=None, stream=None):
        n = self.blocks[b]
        if out is None:
            out = torch.zeros(n, n, dtype=torch.float64, device="cuda")
        _check(lib().fekf_kf_get_block(self.h, b, _ptr(out, torch.float64, "out"), _stream(stream)))
        return out

    def set_block(self, b, src, stream=None):
        _check(lib().fekf_kf_set_block(self.h, b, _ptr(src, torch.float64, "src"), _stream(stream)))

    def state(self):
        lam, A = C.c_double(), C.c_double()
        fl = C.c_int()
        _check(lib().fekf_kf_get_state(self.h, C.byref(lam), C.byref(A), C.byref(fl)))
        return {"lambda": lam.value, "A": A.value, "flags": fl.value}

    def info(self):
        a, b, c, d = C.c_int64(), C.c_int64(), C.c_int64(), C.c_int64()
        _check(lib().fekf_kf_info(self.h, C.byref(a), C.byref(b), C.byref(c), C.byref(d)))
        return {"p_bytes_local": a.value, "tiles_local": b.value, "n_pad": c.value, "items_local": d.value}

    def timing(self, enable):
        """enable=True: start recording P-pass kernel times; False: stop, return (total_ms, launches, rw_launches)."""
        ms, n, rw = C.c_double(), C.c_int64(), C.c_int64()
        _check(lib().fekf_kf_timing(self.h, 1 if enable else 0, C.byref(ms), C.byref(n), C.byref(rw)))
        return ms.value, n.value, rw.value

    def close(self):
        if self._own and self.h:
            lib().fekf_kf_destroy(self.h)
        self.h = C.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class Context:
    """Model + optimizer context (fekf_create).  All tensors are CUDA, contiguous; float64 / int32."""

    def __init__(self, model, opt=None, natoms=None, types=None, local_batch=1, global_batch=None,
                 comm: Comm | None = None, graph: bool = True):
        L = lib()
        self.mc = model_cfg(model)
        self.oc = opt_cfg(opt)
        types = [int(t) for t in types]
        self.natoms = natoms if natoms is not None else len(types)
        self.B = int(local_batch)
        self.Bg = int(global_batch if global_batch is not None else local_batch)
        self.nm = int(sum(self.mc.sel[i] for i in range(self.mc.ntypes)))
        arr = (C.c_int32 * len(types))(*types)
        self.h = C.c_void_p()
        _check(L.fekf_create(C.byref(self.mc), C.byref(self.oc), self.natoms, arr, self.B, self.Bg,
                             comm.h if comm else None, C.byref(self.h)))
        n = C.c_int64()
        _check(L.fekf_param_count(self.h, C.byref(n)))
        self.n_params = n.value
        kh = C.c_void_p()
        _check(L.fekf_get_kf(self.h, C.byref(kh)))
        _, blocks = plan_layout(model, self.oc.block_size)
        self._kh, self._blocks = kh, blocks
        self.comm = comm
        if not graph:
            self.set_graph_mode(False)
        if _get(model, "env_avg", None) is not None or _get(model, "env_std", None) is not None:
            self.set_env_stats(_get(model, "env_avg", None), _get(model, "env_std", None))

    def set_env_stats(self, avg=None, std=None):
        """Descriptor statistics per centre type [ntypes][4] (fekf_set_env_stats, reading Z11)."""
        nt = self.mc.ntypes

        def host(a):
            if a is None:
                return None
            flat = [float(v) for row in a for v in row]
            if len(flat) != nt * 4:
                raise FekfError(1, f"env stats must be [{nt}][4]")
            return (C.c_double * len(flat))(*flat)
        _check(lib().fekf_set_env_stats(self.h, host(avg), host(std)))

    @property
    def kf(self):
        """The context's filter (fekf_get_kf).  A fresh wrapper per access that keeps the context alive,
        so the context itself holds no reference cycle and is freed as soon as the caller drops it."""
        return KalmanFilter(self._blocks, _handle=self._kh, _owner=self)

    def set_graph_mode(self, enable: bool):
        """a10: replay each minibatch step as one captured CUDA graph (default) or launch eagerly."""
        _check(lib().fekf_set_graph_mode(self.h, 1 if enable else 0))

    # ---- parameters ----
    def set_params(self, w, stream=None):
        if w.numel() != self.n_params:
            raise FekfError(1, f"expected {self.n_params} parameters, got {w.numel()}")
        _check(lib().fekf_set_params(self.h, _ptr(w, torch.float64, "w"), _stream(stream)))

    def get_params(self, stream=None):
        out = torch.empty(self.n_params, dtype=torch.float64, device="cuda")
        _check(lib().fekf_get_params(self.h, _ptr(out, torch.float64, "w"), _stream(stream)))
        return out

    # ---- pieces of the step ----
    def build_nlist(self, coord, box, stream=None):
        nb = coord.shape[0]
        nj = torch.empty(nb, self.natoms, self.nm, dtype=torch.int32, device="cuda")
        ns = torch.empty_like(nj)
        ov = torch.empty(nb, dtype=torch.int32, device="cuda")
        _check(lib().fekf_build_nlist(self.h, _ptr(coord, torch.float64, "coord"), _ptr(box, torch.float64, "box"),
                                      nb, _ptr(nj, torch.int32), _ptr(ns, torch.int32), _ptr(ov, torch.int32),
                                      _stream(stream)))
        return nj, ns, ov

    def env_mat(self, coord, box, nlist_j, nlist_shift, stream=None):
        nb = coord.shape[0]
        em = torch.empty(nb, self.natoms, self.nm, 4, dtype=torch.float64, device="cuda")
        jac = torch.empty(nb, self.natoms, self.nm, 4, 3, dtype=torch.float64, device="cuda")
        rij = torch.empty(nb, self.natoms, self.nm, 3, dtype=torch.float64, device="cuda")
        _check(lib().fekf_env_mat(self.h, _ptr(coord, torch.float64, "coord"), _ptr(box, torch.float64, "box"),
                                  _ptr(nlist_j, torch.int32, "nlist_j"), _ptr(nlist_shift, torch.int32, "nlist_shift"),
                                  nb, _ptr(em, torch.float64), _ptr(jac, torch.float64), _ptr(rij, torch.float64),
                                  _stream(stream)))
        return em, jac, rij

    def forward(self, coord, box, need_force=True, stream=None):
        nb = coord.shape[0]
        ea = torch.empty(nb, self.natoms, dtype=torch.float64, device="cuda")
        e = torch.empty(nb, dtype=torch.float64, device="cuda")
        f = torch.empty(nb, self.natoms, 3, dtype=torch.float64, device="cuda") if need_force else None
        v = torch.empty(nb, 9, dtype=torch.float64, device="cuda") if need_force else None
        _check(lib().fekf_forward(self.h, _ptr(coord, torch.float64, "coord"), _ptr(box, torch.float64, "box"), nb,
                                  _ptr(ea, torch.float64), _ptr(e, torch.float64), _ptr(f, torch.float64),
                                  _ptr(v, torch.float64), _stream(stream)))
        return ea, e, f, v

    def energy_jacobian(self, coord, box, e_label, stream=None):
        nb = coord.shape[0]
        g = torch.empty(self.n_params, dtype=torch.float64, device="cuda")
        s = torch.empty(1, dtype=torch.float64, device="cuda")
        _check(lib().fekf_energy_jacobian(self.h, _ptr(coord, torch.float64, "coord"), _ptr(box, torch.float64, "box"),
                                          _ptr(e_label, torch.float64, "e_label"), nb, _ptr(g, torch.float64),
                                          _ptr(s, torch.float64), _stream(stream)))
        return g, s

    def force_jacobian(self, coord, box, f_label, atom_idx, stream=None):
        nb = coord.shape[0]
        g = torch.empty(self.n_params, dtype=torch.float64, device="cuda")
        s = torch.empty(1, dtype=torch.float64, device="cuda")
        _check(lib().fekf_force_jacobian(self.h, _ptr(coord, torch.float64, "coord"), _ptr(box, torch.float64, "box"),
                                         _ptr(f_label, torch.float64, "f_label"), _ptr(atom_idx, torch.int32, "atom_idx"),
                                         atom_idx.numel(), nb, _ptr(g, torch.float64), _ptr(s, torch.float64),
                                         _stream(stream)))
        return g, s

    def kalman_update(self, g, abs_sum, kind, n_sel=0, stream=None):
        _check(lib().fekf_kalman_update(self.h, _ptr(g, torch.float64, "g"), _ptr(abs_sum, torch.float64, "abs_sum"),
                                        int(kind), int(n_sel), _stream(stream)))

    def train_step(self, coord, box, e_label, f_label, force_idx, metrics=None, stream=None):
        if metrics is None:
            metrics = torch.empty(8, dtype=torch.float64, device="cuda")
        na = self.natoms
        for t, n, name in ((coord, self.B * na * 3, "coord"), (box, self.B * 9, "box"), (e_label, self.B, "e_label"),
                           (f_label, self.B * na * 3, "f_label"), (metrics, 8, "metrics"),
                           (force_idx, self.oc.force_groups * self.oc.atoms_per_group, "force_idx")):
            if t.numel() != n:
                raise FekfError(1, f"train_step: {name} has {t.numel()} elements, expected {n} (local_batch={self.B})")
        _check(lib().fekf_train_step(self.h, _ptr(coord, torch.float64, "coord"), _ptr(box, torch.float64, "box"),
                                     _ptr(e_label, torch.float64, "e_label"), _ptr(f_label, torch.float64, "f_label"),
                                     _ptr(force_idx, torch.int32, "force_idx"), _ptr(metrics, torch.float64, "metrics"),
                                     _stream(stream)))
        return metrics

    def naive_train_step(self, coord, box, e_label, f_label, force_idx, metrics=None, stream=None):
        """Naive-EKF minibatch (fekf_naive_train_step): per-image gradients, rank-B Kalman updates."""
        if metrics is None:
            metrics = torch.empty(8, dtype=torch.float64, device="cuda")
        na = self.natoms
        for t, n, name in ((coord, self.B * na * 3, "coord"), (box, self.B * 9, "box"), (e_label, self.B, "e_label"),
                           (f_label, self.B * na * 3, "f_label"), (metrics, 8, "metrics"),
                           (force_idx, self.oc.force_groups * self.oc.atoms_per_group, "force_idx")):
            if t.numel() != n:
                raise FekfError(1, f"naive_train_step: {name} has {t.numel()} elements, expected {n}")
        _check(lib().fekf_naive_train_step(self.h, _ptr(coord, torch.float64, "coord"), _ptr(box, torch.float64, "box"),
                                           _ptr(e_label, torch.float64, "e_label"),
                                           _ptr(f_label, torch.float64, "f_label"),
                                           _ptr(force_idx, torch.int32, "force_idx"),
                                           _ptr(metrics, torch.float64, "metrics"), _stream(stream)))
        return metrics

    def last_launch_count(self):
        n = C.c_int64()
        _check(lib().fekf_last_launch_count(self.h, C.byref(n)))
        return n.value

    def close(self):
        if self.h:
            self._kh = C.c_void_p()
            lib().fekf_destroy(self.h)
            self.h = C.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def sqrt_bs(bg):
    return math.sqrt(bg)
