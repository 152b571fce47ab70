"""Thin Python binding of libmcl.so (include/mcl.h, include/mcl_ext.h) -- argument
marshalling only. Every mapping is scored by the library's CUDA kernels; there is no
Python or CPU fallback: if libmcl.so is missing or no CUDA device is usable, calls raise.

Names mirror the C ABI: ``mcl_mapper_create``, ``mcl_map_queues``, ``mcl_mapper_destroy``,
``mcl_status_string`` ... plus a small ``Mapper`` convenience class that accepts torch
tensors (CUDA or CPU) or numpy arrays.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libmcl.so")

MCL_OK, MCL_E_INVAL, MCL_E_RANGE, MCL_E_CUDA, MCL_E_NCCL, MCL_E_NOMEM = 0, -1, -2, -3, -4, -5
PATH_NAMES = {1: "blocked_u32", 2: "blocked_u64", 3: "generic", 4: "small_batched", 5: "flat_u32",
              6: "pruned", 7: "batch_u32", 8: "blocked_u32_lean", 9: "mixed_u32", 10: "mixed_u64",
              11: "mixed_warp_u32", 12: "batch_pool_u32"}

# Every symbol the headers declare (tests check the library exports all of them).
EXPORTED = [
    "mcl_mapper_create", "mcl_map_queues", "mcl_mapper_destroy", "mcl_status_string",
    "mcl_last_error_string", "mcl_last_launch_info", "mcl_version",
    "mcl_set_timing", "mcl_set_timing_hold", "mcl_last_kernel_time", "mcl_force_path", "mcl_set_pipeline_chunks", "mcl_probe_int_rate",
    "mcl_probe_launch_floor",
    "mcl_device_sms",
    "mcl_comm_unique_id", "mcl_comm_init", "mcl_comm_destroy",
    "mcl_map_queues_constrained", "mcl_score_mappings", "mcl_map_queues_pruned",
    "mcl_build_costs", "mcl_map_from_profiles",
    "mcl_peer_export", "mcl_peer_import", "mcl_static_mappings",
    "mcl_resident_start", "mcl_resident_map", "mcl_resident_stop",
]


class mcl_constraints_t(ctypes.Structure):
    _fields_ = [("base_load", ctypes.c_void_p), ("eligible", ctypes.c_void_p)]


class mcl_cost_model_t(ctypes.Structure):
    _fields_ = [
        ("num_kernels", ctypes.c_uint32), ("kernel_profile", ctypes.c_void_p),
        ("offsets", ctypes.c_void_p), ("kernel_ids", ctypes.c_void_p),
        ("num_invocations", ctypes.c_uint64), ("bytes", ctypes.c_void_p),
        ("source", ctypes.c_void_p), ("cached", ctypes.c_void_p), ("num_sizes", ctypes.c_uint32),
        ("sizes", ctypes.c_void_p), ("h2d_bw", ctypes.c_void_p), ("d2h_bw", ctypes.c_void_p),
        ("host_shared", ctypes.c_uint32), ("num_sockets", ctypes.c_uint32), ("host_socket", ctypes.c_void_p),
    ]


class mcl_config_t(ctypes.Structure):
    _fields_ = [
        ("device", ctypes.c_int),
        ("stream", ctypes.c_void_p),
        ("nccl_comm", ctypes.c_void_p),
        ("rank", ctypes.c_int),
        ("world", ctypes.c_int),
    ]


class MclError(RuntimeError):
    def __init__(self, status: int, where: str, detail: str = ""):
        msg = f"{where}: {mcl_status_string(status)}"
        if detail:
            msg += f" ({detail})"
        super().__init__(msg)
        self.status = status


_lib = None


def load_library(path: str | None = None) -> ctypes.CDLL:
    """Load libmcl.so (fails loudly if it has not been built)."""
    global _lib
    if _lib is not None:
        return _lib
    p = path or LIB_PATH
    if not os.path.exists(p):
        raise RuntimeError(
            f"{p} not found: build it with `python -m paper_conf_cluster_ajipbf15_b200.build` "
            "(there is no CPU fallback)"
        )
    lib = ctypes.CDLL(p)
    vp, u32, u64, i32 = ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int
    sig = {
        "mcl_mapper_create": (i32, [ctypes.POINTER(mcl_config_t), ctypes.POINTER(vp)]),
        "mcl_map_queues": (i32, [vp, u32, u32, u64, vp, vp, vp, vp, vp]),
        "mcl_mapper_destroy": (None, [vp]),
        "mcl_status_string": (ctypes.c_char_p, [i32]),
        "mcl_last_error_string": (ctypes.c_char_p, [vp]),
        "mcl_last_launch_info": (i32, [vp, ctypes.POINTER(ctypes.c_int64)]),
        "mcl_version": (ctypes.c_char_p, []),
        "mcl_set_timing": (i32, [vp, i32]),
        "mcl_set_timing_hold": (i32, [vp, u32]),
        "mcl_force_path": (i32, [vp, i32]),
        "mcl_set_pipeline_chunks": (i32, [vp, i32]),
        "mcl_last_kernel_time": (i32, [vp, ctypes.POINTER(ctypes.c_float), ctypes.POINTER(ctypes.c_float)]),
        "mcl_probe_int_rate": (i32, [i32, i32, ctypes.POINTER(ctypes.c_double),
                                     ctypes.POINTER(ctypes.c_double), ctypes.POINTER(ctypes.c_double)]),
        "mcl_probe_launch_floor": (i32, [i32, i32, ctypes.POINTER(ctypes.c_double), ctypes.POINTER(ctypes.c_double)]),
        "mcl_device_sms": (i32, [i32, ctypes.POINTER(i32)]),
        "mcl_comm_unique_id": (i32, [ctypes.c_char_p]),
        "mcl_comm_init": (i32, [i32, i32, i32, ctypes.c_char_p, ctypes.POINTER(vp)]),
        "mcl_comm_destroy": (i32, [vp]),
        "mcl_map_queues_constrained": (i32, [vp, u32, u32, u64, vp, vp,
                                             ctypes.POINTER(mcl_constraints_t), vp, vp, vp]),
        "mcl_score_mappings": (i32, [vp, u32, u32, u64, vp, vp, vp, vp, vp]),
        "mcl_map_queues_pruned": (i32, [vp, u32, u32, u64, vp, vp,
                                        ctypes.POINTER(mcl_constraints_t), vp, vp, vp]),
        "mcl_build_costs": (i32, [vp, u32, u32, u64, ctypes.POINTER(mcl_cost_model_t), vp, vp]),
        "mcl_map_from_profiles": (i32, [vp, u32, u32, u64, ctypes.POINTER(mcl_cost_model_t),
                                        ctypes.POINTER(mcl_constraints_t), vp, vp, vp]),
        "mcl_peer_export": (i32, [vp, u64, ctypes.c_char_p]),
        "mcl_peer_import": (i32, [vp, ctypes.c_char_p, u32]),
        "mcl_static_mappings": (i32, [vp, u32, u32, u64, vp, u32, vp, vp, vp]),
        "mcl_resident_start": (i32, [vp, u32, u32, u32, u32]),
        "mcl_resident_map": (i32, [vp, u64, vp, vp, vp, vp, vp]),
        "mcl_resident_stop": (i32, [vp]),
    }
    for name, (res, args) in sig.items():
        f = getattr(lib, name)
        f.restype = res
        f.argtypes = args
    _lib = lib
    return lib


def mcl_status_string(status: int) -> str:
    return load_library().mcl_status_string(status).decode()


def mcl_version() -> str:
    return load_library().mcl_version().decode()


def mcl_mapper_create(device: int = 0, stream: int | None = None, nccl_comm: int | None = None,
                      rank: int = 0, world: int = 1) -> int:
    lib = load_library()
    cfg = mcl_config_t(device, stream or None, nccl_comm or None, rank, world)
    h = ctypes.c_void_p()
    st = lib.mcl_mapper_create(ctypes.byref(cfg), ctypes.byref(h))
    if st != MCL_OK:
        raise MclError(st, "mcl_mapper_create", lib.mcl_last_error_string(None).decode())
    return h.value


def mcl_mapper_destroy(handle: int | None) -> None:
    load_library().mcl_mapper_destroy(handle)


def mcl_map_queues(handle: int, Q: int, D: int, epochs: int, cost_kernel_ptr: int,
                   cost_xfer_ptr: int, mapping_index_ptr: int, mapping_ptr: int | None,
                   makespan_ptr: int) -> int:
    """Raw call with integer pointers (device or host). Returns the status code."""
    return load_library().mcl_map_queues(handle, Q, D, epochs, cost_kernel_ptr, cost_xfer_ptr,
                                         mapping_index_ptr, mapping_ptr or None, makespan_ptr)


def mcl_last_error_string(handle: int | None) -> str:
    return load_library().mcl_last_error_string(handle).decode()


def mcl_last_launch_info(handle: int) -> list[int]:
    arr = (ctypes.c_int64 * 8)()
    load_library().mcl_last_launch_info(handle, arr)
    return list(arr)


def mcl_probe_launch_floor(device: int, reps: int = 20) -> tuple[float, float]:
    """(empty-kernel event time, events-alone time) in microseconds (mcl_ext.h)."""
    k, e = ctypes.c_double(), ctypes.c_double()
    st = load_library().mcl_probe_launch_floor(device, reps, ctypes.byref(k), ctypes.byref(e))
    if st != MCL_OK:
        raise MclError(st, "mcl_probe_launch_floor", mcl_last_error_string(None))
    return k.value, e.value


def mcl_probe_int_rate(device: int, op: int) -> tuple[float, float, float]:
    r, c, m = ctypes.c_double(), ctypes.c_double(), ctypes.c_double()
    st = load_library().mcl_probe_int_rate(device, op, ctypes.byref(r), ctypes.byref(c), ctypes.byref(m))
    if st != MCL_OK:
        raise MclError(st, "mcl_probe_int_rate", mcl_last_error_string(None))
    return r.value, c.value, m.value


def mcl_device_sms(device: int = 0) -> int:
    n = ctypes.c_int()
    st = load_library().mcl_device_sms(device, ctypes.byref(n))
    if st != MCL_OK:
        raise MclError(st, "mcl_device_sms")
    return n.value


def mcl_comm_unique_id() -> bytes:
    buf = ctypes.create_string_buffer(128)
    st = load_library().mcl_comm_unique_id(buf)
    if st != MCL_OK:
        raise MclError(st, "mcl_comm_unique_id", mcl_last_error_string(None))
    return buf.raw


def mcl_comm_init(device: int, world: int, rank: int, uid: bytes) -> int:
    comm = ctypes.c_void_p()
    st = load_library().mcl_comm_init(device, world, rank, uid, ctypes.byref(comm))
    if st != MCL_OK:
        raise MclError(st, "mcl_comm_init", mcl_last_error_string(None))
    return comm.value


def mcl_comm_destroy(comm: int | None) -> None:
    load_library().mcl_comm_destroy(comm)


_TORCH = None  # (torch.Tensor, {numpy dtype: torch dtype}) once torch is importable


def _torch_types():
    global _TORCH
    if _TORCH is None:
        try:
            import torch
        except ImportError:  # pragma: no cover
            _TORCH = (type(None), {})
        else:
            _TORCH = (torch.Tensor, {np.uint64: torch.uint64, np.uint8: torch.uint8,
                                     np.uint16: torch.uint16, np.uint32: torch.uint32,
                                     np.int32: torch.int32, np.float64: torch.float64})
    return _TORCH


def _ptr_and_keepalive(x, dtype, convert: bool = False):
    """(pointer, owner) for a torch tensor or numpy array of the given numpy dtype. With
    ``convert`` (read-only inputs) a numpy array is first made a contiguous copy of the
    right dtype; outputs must already match."""
    tensor_type, dtypes = _TORCH or _torch_types()
    if isinstance(x, tensor_type):
        want = dtypes[dtype]
        if x.dtype != want or not x.is_contiguous():
            raise TypeError(f"expected a contiguous {want} tensor")
        return x.data_ptr(), x
    a = np.asarray(x)
    if convert:
        a = np.ascontiguousarray(a, dtype=dtype)
    if a.dtype != dtype or not a.flags.c_contiguous:
        raise TypeError(f"expected a C-contiguous {np.dtype(dtype)} array")
    return a.ctypes.data, a


CUDA_STREAM_LEGACY = 1  # cudaStreamLegacy: the legacy default stream, as a stream handle


def _shape(x) -> tuple:
    return tuple(int(s) for s in x.shape)


def _check(name: str, x, want: tuple) -> None:
    """Raise ValueError unless ``x`` has exactly shape ``want`` (caught here, before any
    pointer reaches the library, so a mismatch can never read or write out of bounds)."""
    if x is not None and _shape(x) != want:
        raise ValueError(f"{name}: expected shape {want}, got {_shape(x)}")


def _default_stream(device: int):
    """torch's current stream on ``device`` (the legacy default stream as cudaStreamLegacy),
    so a handle created without an explicit stream is ordered after the torch work that
    produced its CUDA inputs; None (the handle's own stream) without torch or CUDA."""
    try:
        import torch

        if torch.cuda.is_available():
            return torch.cuda.current_stream(device).cuda_stream or CUDA_STREAM_LEGACY
    except Exception:  # pragma: no cover
        pass
    return None


class Mapper:
    """One mapper handle (see include/mcl.h). Use as a context manager or call close().

    ``stream``: None = torch's current stream on ``device`` at creation (so CUDA tensors
    produced there are ready when the search runs, include/mcl.h "Stream order"); an
    integer cudaStream_t otherwise; 0 = a private non-blocking stream of the handle."""

    def __init__(self, device: int = 0, stream: int | None = None, nccl_comm: int | None = None,
                 rank: int = 0, world: int = 1):
        self.device = device
        if stream is None:
            stream = _default_stream(device)
        self.handle = mcl_mapper_create(device, stream, nccl_comm, rank, world)

    def close(self):
        if self.handle:
            mcl_mapper_destroy(self.handle)
            self.handle = None

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()

    def __del__(self):  # pragma: no cover
        try:
            self.close()
        except Exception:
            pass

    def map_queues_into(self, K, X, index, mapping, makespan) -> None:
        """Run the search writing into caller-owned outputs. K, X: [E, Q, D] uint64;
        index, makespan: [E] uint64; mapping: [E, Q] uint8 or None. Tensors may live on the
        handle's CUDA device or on the host."""
        if K.ndim != 3:
            raise ValueError(f"K: expected [E, Q, D], got shape {_shape(K)}")
        E, Q, D = K.shape
        if (X.shape != K.shape or index.shape != (E,) or makespan.shape != (E,)
                or (mapping is not None and mapping.shape != (E, Q))):
            _check("X", X, (E, Q, D))
            _check("index", index, (E,))
            _check("makespan", makespan, (E,))
            _check("mapping", mapping, (E, Q))
        tensor_type, dtypes = _TORCH or _torch_types()
        if type(K) is tensor_type and type(X) is tensor_type and type(index) is tensor_type \
                and type(makespan) is tensor_type and (mapping is None or type(mapping) is tensor_type):
            # fast path for torch tensors (the per-call marshalling is a few us of a ~20 us call)
            u64 = dtypes[np.uint64]
            ok = (K.dtype is u64 and X.dtype is u64 and index.dtype is u64 and makespan.dtype is u64
                  and (mapping is None or mapping.dtype is dtypes[np.uint8])
                  and K.is_contiguous() and X.is_contiguous() and index.is_contiguous()
                  and makespan.is_contiguous() and (mapping is None or mapping.is_contiguous()))
            if ok:
                st = (_lib or load_library()).mcl_map_queues(
                    self.handle, Q, D, E, K.data_ptr(), X.data_ptr(), index.data_ptr(),
                    None if mapping is None else mapping.data_ptr(), makespan.data_ptr())
                if st != MCL_OK:
                    raise MclError(st, "mcl_map_queues", mcl_last_error_string(self.handle))
                return
        pk, _k = _ptr_and_keepalive(K, np.uint64)
        px, _x = _ptr_and_keepalive(X, np.uint64)
        pi, _i = _ptr_and_keepalive(index, np.uint64)
        pm, _m = _ptr_and_keepalive(makespan, np.uint64)
        pmap = None
        if mapping is not None:
            pmap, _mp = _ptr_and_keepalive(mapping, np.uint8)
        st = (_lib or load_library()).mcl_map_queues(self.handle, Q, D, E, pk, px, pi, pmap, pm)
        if st != MCL_OK:
            raise MclError(st, "mcl_map_queues", mcl_last_error_string(self.handle))

    def map_queues(self, K, X, with_mapping: bool = True):
        """Convenience: allocate outputs like K (same device / numpy) and return
        (index[E], mapping[E, Q] or None, makespan[E])."""
        if K.ndim == 2:
            K, X = K[None], X[None]
        if K.ndim != 3:
            raise ValueError(f"K: expected [E, Q, D], got shape {_shape(K)}")
        E, Q, D = (int(s) for s in K.shape)
        try:
            import torch
        except ImportError:  # pragma: no cover
            torch = None
        if torch is not None and isinstance(K, torch.Tensor):
            idx = torch.empty(E, dtype=torch.uint64, device=K.device)
            ms = torch.empty(E, dtype=torch.uint64, device=K.device)
            mp = torch.empty((E, Q), dtype=torch.uint8, device=K.device) if with_mapping else None
        else:
            idx = np.empty(E, dtype=np.uint64)
            ms = np.empty(E, dtype=np.uint64)
            mp = np.empty((E, Q), dtype=np.uint8) if with_mapping else None
        self.map_queues_into(K, X, idx, mp, ms)
        return idx, mp, ms

    @staticmethod
    def _cost_model(model: dict, D: int):
        """mcl_cost_model_t from a dict of arrays (numpy or torch, host or device); returns
        (struct, keepalive list, E, Q)."""
        keep = []

        def p(name, dtype, optional=False):
            v = model.get(name)
            if v is None:
                if optional:
                    return None
                raise KeyError(name)
            ptr, owner = _ptr_and_keepalive(v, dtype, convert=True)
            keep.append(owner)
            return ptr

        nb = model["bytes"]
        if nb.ndim != 2:
            raise ValueError(f"bytes: expected [E, Q], got shape {_shape(nb)}")
        E, Q = int(nb.shape[0]), int(nb.shape[1])
        nk, M = int(model["profile"].shape[0]), int(model["sizes"].shape[0])
        _check("profile", model["profile"], (nk, D))
        _check("offsets", model["offsets"], (E * Q + 1,))
        if model["kernel_ids"].ndim != 1:
            raise ValueError("kernel_ids: expected a 1-D array")
        _check("source", model["source"], (E, Q))
        _check("cached", model.get("cached"), (E, Q))
        _check("sizes", model["sizes"], (M,))
        S = 1 if model["h2d_bw"].ndim == 2 else int(model["h2d_bw"].shape[0])
        for name in ("h2d_bw", "d2h_bw"):
            _check(name, model[name], (D, M) if model[name].ndim == 2 else (S, D, M))
        _check("host_socket", model.get("host_socket"), (E, Q))
        c = mcl_cost_model_t(
            int(model["profile"].shape[0]), p("profile", np.uint64), p("offsets", np.uint64),
            p("kernel_ids", np.uint32) if int(model["kernel_ids"].shape[0]) else None,
            int(model["kernel_ids"].shape[0]), p("bytes", np.uint64), p("source", np.int32),
            p("cached", np.uint16, optional=True), int(model["sizes"].shape[0]), p("sizes", np.uint64),
            p("h2d_bw", np.float64), p("d2h_bw", np.float64), int(model.get("host_shared", 0)),
            S, p("host_socket", np.uint8, optional=True),
        )
        return c, keep, E, Q

    def build_costs(self, model: dict, D: int, device_out: bool = False):
        """Cost tables K, X [E, Q, D] from a cost model (include/mcl.h mcl_build_costs).
        Returns numpy arrays, or CUDA tensors when device_out."""
        c, keep, E, Q = self._cost_model(model, D)
        if device_out:
            import torch

            K = torch.empty((E, Q, D), dtype=torch.uint64, device=f"cuda:{self.device}")
            X = torch.empty_like(K)
        else:
            K = np.empty((E, Q, D), np.uint64)
            X = np.empty((E, Q, D), np.uint64)
        pk, _k = _ptr_and_keepalive(K, np.uint64)
        px, _x = _ptr_and_keepalive(X, np.uint64)
        st = load_library().mcl_build_costs(self.handle, Q, D, E, ctypes.byref(c), pk, px)
        if st != MCL_OK:
            raise MclError(st, "mcl_build_costs", mcl_last_error_string(self.handle))
        return K, X

    def map_from_profiles(self, model: dict, D: int, base=None, eligible=None):
        """Build the cost tables and search in one call (mcl_map_from_profiles); host
        (numpy) outputs (index, mapping, makespan)."""
        c, keep, E, Q = self._cost_model(model, D)
        pb, _b = _ptr_and_keepalive(base, np.uint64) if base is not None else (None, None)
        pe, _e = _ptr_and_keepalive(eligible, np.uint16) if eligible is not None else (None, None)
        cons = mcl_constraints_t(pb, pe)
        idx = np.empty(E, np.uint64)
        ms = np.empty(E, np.uint64)
        mp = np.empty((E, Q), np.uint8)
        st = load_library().mcl_map_from_profiles(self.handle, Q, D, E, ctypes.byref(c), ctypes.byref(cons),
                                                  idx.ctypes.data, mp.ctypes.data, ms.ctypes.data)
        if st != MCL_OK:
            raise MclError(st, "mcl_map_from_profiles", mcl_last_error_string(self.handle))
        return idx, mp, ms

    def map_queues_pruned(self, K, X, base=None, eligible=None, with_mapping: bool = True):
        """Exact search with pruning (include/mcl.h mcl_map_queues_pruned): same result as
        map_queues_constrained, time depends on the instance."""
        return self.map_queues_constrained(K, X, base, eligible, with_mapping, _fn="mcl_map_queues_pruned")

    def map_queues_constrained(self, K, X, base=None, eligible=None, with_mapping: bool = True,
                               _fn: str = "mcl_map_queues_constrained"):
        """Constrained search (include/mcl.h mcl_map_queues_constrained): ``base`` [E, D]
        uint64 device base loads or None, ``eligible`` [E, Q] uint16 device masks (0 = any)
        or None. Outputs are allocated like K; returns (index, mapping or None, makespan)."""
        if K.ndim == 2:
            K, X = K[None], X[None]
            base = None if base is None else base[None]
            eligible = None if eligible is None else eligible[None]
        if K.ndim != 3:
            raise ValueError(f"K: expected [E, Q, D], got shape {_shape(K)}")
        E, Q, D = (int(s) for s in K.shape)
        _check("X", X, (E, Q, D))
        _check("base", base, (E, D))
        _check("eligible", eligible, (E, Q))
        idx, mp, ms = self._alloc_outputs(K, E, Q, with_mapping)
        pk, _k = _ptr_and_keepalive(K, np.uint64)
        px, _x = _ptr_and_keepalive(X, np.uint64)
        pb, _b = _ptr_and_keepalive(base, np.uint64) if base is not None else (None, None)
        pe, _e = _ptr_and_keepalive(eligible, np.uint16) if eligible is not None else (None, None)
        pi, _i = _ptr_and_keepalive(idx, np.uint64)
        pm, _m = _ptr_and_keepalive(ms, np.uint64)
        pmap = _ptr_and_keepalive(mp, np.uint8)[0] if mp is not None else None
        c = mcl_constraints_t(pb, pe)
        st = getattr(load_library(), _fn)(self.handle, Q, D, E, pk, px, ctypes.byref(c), pi, pmap, pm)
        if st != MCL_OK:
            raise MclError(st, _fn, mcl_last_error_string(self.handle))
        return idx, mp, ms

    def score_mappings(self, K, X, mappings, base=None):
        """Makespan of given mappings [E, Q] (uint8 device ids), optional base loads [E, D]."""
        if K.ndim == 2:
            K, X, mappings = K[None], X[None], mappings[None]
            base = None if base is None else base[None]
        if K.ndim != 3:
            raise ValueError(f"K: expected [E, Q, D], got shape {_shape(K)}")
        E, Q, D = (int(s) for s in K.shape)
        _check("X", X, (E, Q, D))
        _check("mappings", mappings, (E, Q))
        _check("base", base, (E, D))
        ms = self._alloc_outputs(K, E, Q, False)[2]
        pk, _k = _ptr_and_keepalive(K, np.uint64)
        px, _x = _ptr_and_keepalive(X, np.uint64)
        pb, _b = _ptr_and_keepalive(base, np.uint64) if base is not None else (None, None)
        pmp, _mp = _ptr_and_keepalive(mappings, np.uint8)
        pm, _m = _ptr_and_keepalive(ms, np.uint64)
        st = load_library().mcl_score_mappings(self.handle, Q, D, E, pk, px, pb, pmp, pm)
        if st != MCL_OK:
            raise MclError(st, "mcl_score_mappings", mcl_last_error_string(self.handle))
        return ms

    def static_mappings(self, hints, device_score, eligible=None):
        """SCHED_AUTO_STATIC policy baseline (include/mcl.h mcl_static_mappings): hints
        [E, Q] uint8 queue classes, device_score [C, D] uint64 (lower is better), eligible
        [E, Q] uint16 or None. Returns mappings [E, Q] uint8 like ``hints`` (torch / numpy)."""
        if hints.ndim != 2 or device_score.ndim != 2:
            raise ValueError("hints: [E, Q]; device_score: [C, D]")
        E, Q = (int(s) for s in hints.shape)
        C, D = (int(s) for s in device_score.shape)
        _check("eligible", eligible, (E, Q))
        try:
            import torch
        except ImportError:  # pragma: no cover
            torch = None
        if torch is not None and isinstance(hints, torch.Tensor):
            out = torch.empty((E, Q), dtype=torch.uint8, device=hints.device)
        else:
            out = np.empty((E, Q), np.uint8)
        ph, _h = _ptr_and_keepalive(hints, np.uint8)
        ps, _s = _ptr_and_keepalive(device_score, np.uint64, convert=True)
        pe, _e = _ptr_and_keepalive(eligible, np.uint16) if eligible is not None else (None, None)
        po, _o = _ptr_and_keepalive(out, np.uint8)
        st = load_library().mcl_static_mappings(self.handle, Q, D, E, ph, C, ps, pe, po)
        if st != MCL_OK:
            raise MclError(st, "mcl_static_mappings", mcl_last_error_string(self.handle))
        return out

    def resident_start(self, Q: int, D: int, max_epochs: int = 1, idle_ms: int = 0) -> None:
        """Leave one warp resident for low-latency decisions (include/mcl.h
        mcl_resident_start): D^Q <= 8192, max_epochs <= 64 per resident_map call. While it is
        resident, device-wide synchronisation waits for it (up to idle_ms): stop it first."""
        st = load_library().mcl_resident_start(self.handle, Q, D, max_epochs, idle_ms)
        if st != MCL_OK:
            raise MclError(st, "mcl_resident_start", mcl_last_error_string(self.handle))
        self._resident = (int(Q), int(D), int(max_epochs))
        self._res_fn = load_library().mcl_resident_map
        self._res_cache = None

    def resident_map(self, K, X, out=None):
        """One decision batch through the resident warp. K, X: HOST arrays [E, Q, D] (or
        [Q, D]) uint64 (numpy, or CPU torch tensors); returns (index [E], mapping [E, Q],
        makespan [E]) numpy arrays, or fills ``out`` = (index, mapping, makespan)."""
        Q, D, cap = getattr(self, "_resident", (0, 0, 0))
        if not Q:
            raise MclError(-1, "mcl_resident_map", "resident mapper not started")
        if K.ndim == 2:
            K, X = K[None], X[None]
        E = int(K.shape[0])
        if out is None:
            out = (np.empty(E, np.uint64), np.empty((E, Q), np.uint8), np.empty(E, np.uint64))
        idx, mp, ms = out
        c = self._res_cache
        if (c is not None and K is c[0] and X is c[1] and idx is c[2] and mp is c[3] and ms is c[4]
                and K.shape == c[5]):
            # the same five arrays as the previous call (kept alive by the cache, so their
            # addresses are still theirs): a decision is a few microseconds, and building an
            # address from a numpy array costs ~1.5 us each
            st = self._res_fn(self.handle, E, *c[6])
        elif (type(K) is np.ndarray and type(X) is np.ndarray and type(idx) is np.ndarray
                and type(ms) is np.ndarray and type(mp) is np.ndarray):
            want = (E, Q, D)
            if (K.shape != want or X.shape != want or idx.shape != (E,) or ms.shape != (E,)
                    or mp.shape != (E, Q)):
                raise ValueError(f"resident_map: expected K, X {want}, outputs ({E},), ({E}, {Q}), ({E},)")
            for a, dt in ((K, np.uint64), (X, np.uint64), (idx, np.uint64), (ms, np.uint64), (mp, np.uint8)):
                if a.dtype != dt or not a.flags.c_contiguous:
                    raise TypeError(f"expected C-contiguous {np.dtype(dt)} arrays")
            ptrs = tuple(a.ctypes.data for a in (K, X, idx, mp, ms))
            self._res_cache = (K, X, idx, mp, ms, K.shape, ptrs)
            st = self._res_fn(self.handle, E, *ptrs)
        else:
            _check("K", K, (E, Q, D))
            _check("X", X, (E, Q, D))
            _check("index", idx, (E,))
            _check("mapping", mp, (E, Q))
            _check("makespan", ms, (E,))
            pk, _k = _ptr_and_keepalive(K, np.uint64)
            px, _x = _ptr_and_keepalive(X, np.uint64)
            pi, _i = _ptr_and_keepalive(idx, np.uint64)
            pm, _m = _ptr_and_keepalive(ms, np.uint64)
            pmap = _ptr_and_keepalive(mp, np.uint8)[0] if mp is not None else None
            st = self._res_fn(self.handle, E, pk, px, pi, pmap, pm)
        if st != MCL_OK:
            raise MclError(st, "mcl_resident_map", mcl_last_error_string(self.handle))
        return idx, mp, ms

    def resident_stop(self) -> None:
        st = load_library().mcl_resident_stop(self.handle)
        self._resident = (0, 0, 0)
        self._res_cache = None
        if st != MCL_OK:
            raise MclError(st, "mcl_resident_stop", mcl_last_error_string(self.handle))

    @staticmethod
    def _alloc_outputs(K, E, Q, with_mapping):
        try:
            import torch
        except ImportError:  # pragma: no cover
            torch = None
        if torch is not None and isinstance(K, torch.Tensor):
            idx = torch.empty(E, dtype=torch.uint64, device=K.device)
            ms = torch.empty(E, dtype=torch.uint64, device=K.device)
            mp = torch.empty((E, Q), dtype=torch.uint8, device=K.device) if with_mapping else None
        else:
            idx = np.empty(E, dtype=np.uint64)
            ms = np.empty(E, dtype=np.uint64)
            mp = np.empty((E, Q), dtype=np.uint8) if with_mapping else None
        return idx, mp, ms

    def launch_info(self) -> dict:
        i = mcl_last_launch_info(self.handle)
        return {"path": PATH_NAMES.get(i[0], str(i[0])), "launches": i[1], "ctas": i[2],
                "threads": i[3], "allreduce": bool(i[4]), "fused_exchange": i[4] == 2,
                "index_bits": i[5], "two_step": bool(i[6]),
                "nodes": i[7] if i[0] == 6 else 0, "chunks": i[7] if i[0] != 6 else 0}

    def peer_export(self, max_epochs: int = 1) -> bytes:
        """Allocate this rank's exchange slab for the fused cross-GPU exchange and return
        its 64-byte CUDA IPC handle (include/mcl.h mcl_peer_export)."""
        buf = ctypes.create_string_buffer(64)
        st = load_library().mcl_peer_export(self.handle, max_epochs, buf)
        if st != MCL_OK:
            raise MclError(st, "mcl_peer_export", mcl_last_error_string(self.handle))
        return buf.raw

    def peer_import(self, handles: list[bytes], timeout_ms: int = 0) -> None:
        """Map every rank's slab (handles in rank order, 64 bytes each); afterwards calls
        of up to max_epochs epochs exchange results inside the search kernel."""
        if any(len(h) != 64 for h in handles):
            raise ValueError("every handle is 64 bytes")
        st = load_library().mcl_peer_import(self.handle, b"".join(handles), timeout_ms)
        if st != MCL_OK:
            raise MclError(st, "mcl_peer_import", mcl_last_error_string(self.handle))

    def connect_peers(self, group=None, max_epochs: int = 1, timeout_ms: int = 0) -> None:
        """Collective over a torch.distributed group: export, all-gather the handles
        (plumbing only), import."""
        import torch.distributed as dist

        mine = self.peer_export(max_epochs)
        world = dist.get_world_size(group)
        got: list = [None] * world
        dist.all_gather_object(got, mine, group=group)
        self.peer_import(got, timeout_ms)

    def set_pipeline_chunks(self, chunks: int) -> None:
        """Pipelined staging of host-resident batches (include/mcl_ext.h
        mcl_set_pipeline_chunks): 0 automatic, 1 off, n > 1 exactly n chunks."""
        st = load_library().mcl_set_pipeline_chunks(self.handle, chunks)
        if st != MCL_OK:
            raise MclError(st, "mcl_set_pipeline_chunks")

    def force_path(self, path: int) -> None:
        """Testing aid: 0 auto, 1 blocked u32 (CTA per epoch), 2 blocked u64, 3 generic,
        4 small batched, 5 flattened batched blocked u32, 6 branch-and-bound kernel in
        map_queues_pruned even for small index spaces, 7 warp-per-epoch batched kernel,
        8 mixed-radix constrained kernel (the default for calls with eligible masks), 9 its
        warp-per-epoch form (the default for batches of them)."""
        st = load_library().mcl_force_path(self.handle, path)
        if st != MCL_OK:
            raise MclError(st, "mcl_force_path")

    def set_timing(self, enable: bool = True, hold_us: int = 0) -> None:
        """CUDA-event timing of the search kernel; hold_us > 0 precedes each timed launch
        with a spin kernel so the events exclude host launch latency (measurement only)."""
        lib = load_library()
        lib.mcl_set_timing(self.handle, 1 if enable else 0)
        lib.mcl_set_timing_hold(self.handle, int(hold_us))

    def last_kernel_time_ms(self) -> tuple[float, float]:
        k, c = ctypes.c_float(), ctypes.c_float()
        load_library().mcl_last_kernel_time(self.handle, ctypes.byref(k), ctypes.byref(c))
        return k.value, c.value
