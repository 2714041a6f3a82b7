"""Thin ctypes binding of libmemxct (include/memxct.h).

Argument marshalling only: every step of the hot path (tracing, ordering, layout, SpMV, CG) runs
in the library's CUDA kernels.  PyTorch is used for device memory and streams.  There is no CPU
fallback: if the CUDA library is missing or there is no GPU, calls raise.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_PKG, "libmemxct.so")

OK = 0
STATUS = {0: "MEMXCT_OK", 1: "MEMXCT_ERR_INVALID_ARG", 2: "MEMXCT_ERR_STATE",
          3: "MEMXCT_ERR_OUT_OF_MEMORY", 4: "MEMXCT_ERR_CUDA", 5: "MEMXCT_ERR_NCCL",
          6: "MEMXCT_ERR_UNSUPPORTED"}
OPT = {"tile_tomo": 0, "tile_sino": 1, "part_rows": 2, "buffer_entries": 3, "precision": 4,
       "canonical": 5, "cg_variant": 6, "vector_order": 7, "slices": 8, "exchange": 9,
       "ray_block": 10, "stage_order": 11}

#: every symbol include/memxct.h declares (checked by tests/test_abi.py)
SYMBOLS = [
    "memxct_plan_create", "memxct_plan_set_option", "memxct_plan_get_option",
    "memxct_plan_set_comm", "memxct_get_unique_id", "memxct_build", "memxct_local_size",
    "memxct_local_indices", "memxct_forward", "memxct_back", "memxct_cg",
    "memxct_forward_host", "memxct_back_host", "memxct_cg_host", "memxct_stats",
    "memxct_layout_info", "memxct_layout_export", "memxct_plan_destroy",
    "memxct_status_string", "memxct_last_error", "memxct_kernel_launch_count",
    "memxct_local_group_create", "memxct_local_group_destroy", "memxct_plan_set_comm_local",
    "memxct_partition_ranges", "memxct_domain_ranges", "memxct_exchange_info",
    "memxct_forward_batch", "memxct_back_batch", "memxct_cg_batch", "memxct_exchange_time",
    "memxct_sirt", "memxct_spmv_time", "memxct_plan_set_shard", "memxct_exchange_counts",
    "memxct_footprint_rays", "memxct_footprint_forward", "memxct_footprint_back", "memxct_layout_rows",
    "memxct_read_ceiling", "memxct_export_coo", "memxct_build_phases", "memxct_plan_set_comm_host", "memxct_host_comm_probe",
]

#: memxct_build_phases order (include/memxct.h)
BUILD_PHASES = ["hilbert", "decompose", "count", "trace_fwd", "sort_fwd", "layout_fwd", "trace_back",
                "transpose", "layout_back", "exchange", "total"]


def read_ceiling(nbytes: int = 11_600_000_000, reps: int = 10, stream=None) -> float:
    """memxct_read_ceiling: achievable HBM read bandwidth of the current device, GB/s."""
    g = ctypes.c_double()
    _check(lib().memxct_read_ceiling(int(nbytes), int(reps), ctypes.byref(g), _stream(stream)),
           "memxct_read_ceiling")
    return g.value


class MemXCTError(RuntimeError):
    def __init__(self, status: int, where: str, detail: str):
        super().__init__(f"{where}: {STATUS.get(status, status)}: {detail}")
        self.status = status


_lib = None


def lib():
    """Load libmemxct.so (raises if it was not built: there is no fallback)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} not built; run `python -m paper_conf_sc_hidayetoglubgrg19_b200"
                              f".build_ext` (the CUDA library is required, there is no CPU path)")
        L = ctypes.CDLL(LIB_PATH)
        i32, i64, vp, st = ctypes.c_int32, ctypes.c_int64, ctypes.c_void_p, ctypes.c_int
        P64 = ctypes.POINTER(ctypes.c_int64)
        sig = {
            "memxct_plan_create": [i32, i32, i32, ctypes.POINTER(vp)],
            "memxct_plan_set_option": [vp, ctypes.c_int, i64],
            "memxct_plan_get_option": [vp, ctypes.c_int, P64],
            "memxct_plan_set_comm": [vp, i32, i32, vp, i32],
            "memxct_get_unique_id": [vp],
            "memxct_build": [vp, vp],
            "memxct_local_size": [vp, i32, P64],
            "memxct_local_indices": [vp, i32, vp],
            "memxct_forward": [vp, vp, vp, vp],
            "memxct_back": [vp, vp, vp, vp],
            "memxct_cg": [vp, vp, vp, i32, vp, vp],
            "memxct_forward_host": [vp, vp, vp, vp],
            "memxct_back_host": [vp, vp, vp, vp],
            "memxct_cg_host": [vp, vp, vp, i32, vp, vp],
            "memxct_stats": [vp, P64, P64, P64, P64],
            "memxct_layout_info": [vp, i32, P64, P64, P64, P64, P64, P64, P64, P64],
            "memxct_layout_export": [vp, i32, i64, i64, vp, vp, vp, vp, vp, vp, vp, vp, P64, P64, P64],
            "memxct_plan_destroy": [vp],
            "memxct_local_group_create": [i32, ctypes.POINTER(vp)],
            "memxct_local_group_destroy": [vp],
            "memxct_plan_set_comm_local": [vp, vp, i32],
            "memxct_partition_ranges": [vp, i64, i32, vp],
            "memxct_domain_ranges": [vp, i32, vp],
            "memxct_exchange_info": [vp, P64, P64, P64, ctypes.POINTER(i32)],
            "memxct_forward_batch": [vp, i32, vp, vp, vp],
            "memxct_back_batch": [vp, i32, vp, vp, vp],
            "memxct_cg_batch": [vp, i32, vp, vp, i32, vp, vp],
            "memxct_sirt": [vp, vp, vp, i32, vp, vp],
            "memxct_exchange_time": [vp, i32, ctypes.POINTER(ctypes.c_double),
                                     ctypes.POINTER(ctypes.c_double), vp],
            "memxct_spmv_time": [vp, i32, ctypes.POINTER(ctypes.c_double),
                                 ctypes.POINTER(ctypes.c_double), vp],
            "memxct_plan_set_shard": [vp, i32, i32, i32],
            "memxct_exchange_counts": [vp, vp, vp],
            "memxct_footprint_rays": [vp, vp],
            "memxct_footprint_forward": [vp, vp, vp, vp],
            "memxct_footprint_back": [vp, vp, vp, vp],
            "memxct_layout_rows": [vp, i32, vp],
            "memxct_read_ceiling": [i64, i32, ctypes.POINTER(ctypes.c_double), vp],
            "memxct_export_coo": [vp, i32, vp, vp, vp, vp],
            "memxct_build_phases": [vp, vp],
            "memxct_plan_set_comm_host": [vp, i32, i32, ctypes.c_char_p, i32],
            "memxct_host_comm_probe": [ctypes.c_char_p, i32, i32, i64, vp],
        }
        for name, args in sig.items():
            f = getattr(L, name)
            f.argtypes = args
            f.restype = st
        L.memxct_status_string.argtypes = [st]
        L.memxct_status_string.restype = ctypes.c_char_p
        L.memxct_last_error.argtypes = []
        L.memxct_last_error.restype = ctypes.c_char_p
        L.memxct_kernel_launch_count.argtypes = []
        L.memxct_kernel_launch_count.restype = i64
        _lib = L
    return _lib


def _check(status: int, where: str):
    if status != OK:
        raise MemXCTError(status, where, lib().memxct_last_error().decode())


def kernel_launch_count() -> int:
    return int(lib().memxct_kernel_launch_count())


def _ptr(t) -> ctypes.c_void_p:
    return ctypes.c_void_p(t.data_ptr())


def _stream(stream):
    import torch
    if stream is None:
        stream = torch.cuda.current_stream()
    return ctypes.c_void_p(stream.cuda_stream)


def get_unique_id() -> bytes:
    buf = ctypes.create_string_buffer(128)
    _check(lib().memxct_get_unique_id(buf), "memxct_get_unique_id")
    return buf.raw


def partition_ranges(weights, parts: int) -> np.ndarray:
    """Host helper of the domain decomposition (memxct_partition_ranges): contiguous ranges of
    about equal weight; returns bounds[0..parts]."""
    w = np.ascontiguousarray(weights, np.int64)
    out = np.empty(parts + 1, np.int64)
    _check(lib().memxct_partition_ranges(w.ctypes.data_as(ctypes.c_void_p), len(w), int(parts),
                                         out.ctypes.data_as(ctypes.c_void_p)), "memxct_partition_ranges")
    return out


class LocalGroup:
    """Virtual ranks in one process (memxct_local_group_create): P plans on one device, each
    driven from its own thread, collectives done by device copies.  For testing the multi-GPU
    path on a single GPU."""

    def __init__(self, nranks: int):
        self.nranks = int(nranks)
        self._h = ctypes.c_void_p()
        _check(lib().memxct_local_group_create(self.nranks, ctypes.byref(self._h)), "memxct_local_group_create")

    def close(self):
        if self._h and self._h.value:
            lib().memxct_local_group_destroy(self._h)
            self._h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def host_comm_probe(name: str, rank: int, nranks: int, value: int) -> np.ndarray:
    """memxct_host_comm_probe: host-only rendezvous + allgather of one int64 per rank."""
    out = np.empty(nranks, np.int64)
    _check(lib().memxct_host_comm_probe(name.encode(), int(rank), int(nranks), int(value),
                                        out.ctypes.data_as(ctypes.c_void_p)), "memxct_host_comm_probe")
    return out


def bootstrap_host_comm_name(rank: int, group=None) -> str:
    """Rank 0 draws a fresh shared-memory segment name for memxct_plan_set_comm_host; every rank
    receives it through torch.distributed (gloo is enough)."""
    import torch.distributed as dist
    import uuid
    obj = ["/memxct-" + uuid.uuid4().hex[:20] if rank == 0 else None]
    dist.broadcast_object_list(obj, src=0, group=group)
    return obj[0]


def bootstrap_unique_id(rank: int, group=None) -> bytes:
    """Rank 0 makes an ncclUniqueId; every rank receives it through torch.distributed."""
    import torch.distributed as dist
    obj = [get_unique_id() if rank == 0 else None]
    dist.broadcast_object_list(obj, src=0, group=group)
    return obj[0]


class MemXCT:
    """A MemXCT plan: geometry (N, M, C), options, built matrices, and the hot-path calls.

    Mirrors memxct_plan_create / set_option / set_comm / build / forward / back / cg / destroy.
    Vectors are torch CUDA tensors (float32 in "fp32" precision, float64 in "mixed").
    """

    def __init__(self, n: int, projections: int, channels: int, *, precision: str = "fp32",
                 canonical: bool = False, vector_order: str = "natural", part_rows: int = None,
                 buffer_entries: int = None, tile_tomo: int = None, tile_sino: int = None,
                 cg_variant: int = 0, rank: int = 0, nranks: int = 1, unique_id: bytes = None,
                 device: int = None, group: "LocalGroup" = None, slices: int = None,
                 exchange: str = None, shard: bool = False, ray_block: int = None,
                 stage_order: int = None, host_comm: str = None):
        self.n, self.m, self.c = int(n), int(projections), int(channels)
        self._h = ctypes.c_void_p()
        _check(lib().memxct_plan_create(self.n, self.m, self.c, ctypes.byref(self._h)),
               "memxct_plan_create")
        self.precision = precision
        opts = {"precision": {"fp32": 0, "mixed": 1}[precision], "canonical": int(bool(canonical)),
                "vector_order": {"natural": 0, "plan": 1}[vector_order], "cg_variant": cg_variant,
                "part_rows": part_rows, "buffer_entries": buffer_entries, "tile_tomo": tile_tomo,
                "tile_sino": tile_sino, "slices": slices, "ray_block": ray_block, "stage_order": stage_order,
                "exchange": None if exchange is None else {"collective": 0, "peer": 1, "dense": 2}[exchange]}
        for k, v in opts.items():
            if v is not None:
                self.set_option(k, v)
        self._group = group  # keep the virtual-rank group alive as long as the plan
        self.rank = int(rank)
        self.nranks = group.nranks if group is not None else int(nranks)
        if shard:
            _check(lib().memxct_plan_set_shard(self._h, self.rank, int(nranks), -1 if device is None else int(device)),
                   "memxct_plan_set_shard")
        elif group is not None:
            _check(lib().memxct_plan_set_comm_local(self._h, group._h, int(rank)), "memxct_plan_set_comm_local")
        elif host_comm is not None:
            _check(lib().memxct_plan_set_comm_host(self._h, self.rank, int(nranks), host_comm.encode(),
                                                   -1 if device is None else int(device)),
                   "memxct_plan_set_comm_host")
        elif nranks > 1 or device is not None or unique_id is not None:
            uid = None if unique_id is None else ctypes.create_string_buffer(unique_id, 128)
            _check(lib().memxct_plan_set_comm(self._h, rank, nranks, uid,
                                              -1 if device is None else int(device)),
                   "memxct_plan_set_comm")
        self.built = False

    # -- options / lifecycle ---------------------------------------------------------------
    def set_option(self, name: str, value: int):
        _check(lib().memxct_plan_set_option(self._h, OPT[name], int(value)), "memxct_plan_set_option")

    def get_option(self, name: str) -> int:
        v = ctypes.c_int64()
        _check(lib().memxct_plan_get_option(self._h, OPT[name], ctypes.byref(v)), "memxct_plan_get_option")
        return v.value

    def build(self, stream=None):
        _check(lib().memxct_build(self._h, _stream(stream)), "memxct_build")
        self.built = True
        return self

    def close(self):
        if self._h and self._h.value:
            lib().memxct_plan_destroy(self._h)
            self._h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    # -- sizes / introspection --------------------------------------------------------------
    @property
    def dtype(self):
        import torch
        return torch.float32 if self.precision == "fp32" else torch.float64

    def build_phases(self) -> dict:
        """Seconds per preprocessing phase of the build (memxct_build_phases)."""
        out = np.empty(len(BUILD_PHASES), np.float64)
        _check(lib().memxct_build_phases(self._h, out.ctypes.data_as(ctypes.c_void_p)), "memxct_build_phases")
        return dict(zip(BUILD_PHASES, out.tolist()))

    def local_size(self, domain: int) -> int:
        v = ctypes.c_int64()
        _check(lib().memxct_local_size(self._h, domain, ctypes.byref(v)), "memxct_local_size")
        return v.value

    def local_indices(self, domain: int) -> np.ndarray:
        out = np.empty(self.local_size(domain), np.int64)
        _check(lib().memxct_local_indices(self._h, domain, out.ctypes.data_as(ctypes.c_void_p)),
               "memxct_local_indices")
        return out

    def stats(self) -> dict:
        v = [ctypes.c_int64() for _ in range(4)]
        _check(lib().memxct_stats(self._h, *[ctypes.byref(x) for x in v]), "memxct_stats")
        return dict(zip(["nnz", "stored_slots", "map_entries", "device_bytes"], [x.value for x in v]))

    def domain_ranges(self, domain: int) -> np.ndarray:
        """Hilbert-index range boundaries of every rank for domain 0 (pixels) / 1 (rays)."""
        out = np.empty(self.nranks + 1, np.int64)
        _check(lib().memxct_domain_ranges(self._h, domain, out.ctypes.data_as(ctypes.c_void_p)),
               "memxct_domain_ranges")
        return out

    def exchange_info(self) -> dict:
        a, b, c = ctypes.c_int64(), ctypes.c_int64(), ctypes.c_int64()
        d = ctypes.c_int32()
        _check(lib().memxct_exchange_info(self._h, ctypes.byref(a), ctypes.byref(b), ctypes.byref(c),
                                          ctypes.byref(d)), "memxct_exchange_info")
        return {"footprint_rays": a.value, "sent": b.value, "received": c.value, "peers": d.value}

    def exchange_counts(self) -> dict:
        """Entries sent to / received from every rank per forward exchange (decomposed plans)."""
        sc = np.empty(self.nranks, np.int64)
        rc = np.empty(self.nranks, np.int64)
        _check(lib().memxct_exchange_counts(self._h, sc.ctypes.data_as(ctypes.c_void_p),
                                            rc.ctypes.data_as(ctypes.c_void_p)), "memxct_exchange_counts")
        return {"send": sc, "recv": rc}

    def footprint_rays(self) -> np.ndarray:
        """Natural indices of this rank's footprint rays (rows of A_p), in A_p row order."""
        out = np.empty(self.exchange_info()["footprint_rays"], np.int64)
        _check(lib().memxct_footprint_rays(self._h, out.ctypes.data_as(ctypes.c_void_p)), "memxct_footprint_rays")
        return out

    def footprint_forward(self, x_local, y_fp=None, stream=None):
        """Partial projection y_fp = A_p x_local (before exchange and reduction)."""
        import torch
        self._vec(x_local, 0, "x_local")
        nfp = self.exchange_info()["footprint_rays"]
        if y_fp is None:
            y_fp = torch.empty(nfp, dtype=self.dtype, device=x_local.device)
        if y_fp.numel() != nfp or y_fp.dtype != self.dtype or not y_fp.is_contiguous():
            raise ValueError(f"y_fp must be a contiguous {self.dtype} tensor of {nfp} elements")
        _check(lib().memxct_footprint_forward(self._h, _ptr(x_local), _ptr(y_fp), _stream(stream)),
               "memxct_footprint_forward")
        return y_fp

    def footprint_back(self, y_fp, x_local=None, stream=None):
        """Partial backprojection x_local = A_p^T y_fp."""
        import torch
        nfp = self.exchange_info()["footprint_rays"]
        if y_fp.numel() != nfp or y_fp.dtype != self.dtype or not y_fp.is_contiguous() or not y_fp.is_cuda:
            raise ValueError(f"y_fp must be a contiguous CUDA {self.dtype} tensor of {nfp} elements")
        if x_local is None:
            x_local = torch.empty(self.local_size(0), dtype=self.dtype, device=y_fp.device)
        self._vec(x_local, 0, "x_local")
        _check(lib().memxct_footprint_back(self._h, _ptr(y_fp), _ptr(x_local), _stream(stream)),
               "memxct_footprint_back")
        return x_local

    def exchange_time(self, reps: int = 20, stream=None) -> dict:
        """Collective: device microseconds of one forward and one back exchange (P > 1)."""
        f, b = ctypes.c_double(), ctypes.c_double()
        _check(lib().memxct_exchange_time(self._h, int(reps), ctypes.byref(f), ctypes.byref(b),
                                          _stream(stream)), "memxct_exchange_time")
        return {"fwd_us": f.value, "back_us": b.value}

    def spmv_time(self, reps: int = 20, stream=None) -> dict:
        """Local: device microseconds of this rank's A_p / A_p^T kernels alone (no exchange)."""
        f, b = ctypes.c_double(), ctypes.c_double()
        _check(lib().memxct_spmv_time(self._h, int(reps), ctypes.byref(f), ctypes.byref(b),
                                      _stream(stream)), "memxct_spmv_time")
        return {"fwd_us": f.value, "back_us": b.value}

    def layout_info(self, direction: int) -> dict:
        v = [ctypes.c_int64() for _ in range(8)]
        _check(lib().memxct_layout_info(self._h, direction, *[ctypes.byref(x) for x in v]),
               "memxct_layout_info")
        return dict(zip(["parts", "stages", "slots", "map_entries", "rows", "nnz", "part_rows", "buffer_entries"],
                        [x.value for x in v]))

    def export_coo(self, direction: int, stream=None):
        """memxct_export_coo: (rows, cols, vals) device tensors, one entry per stored slot
        (padding = (-1, -1, 0)), in the plan's vector order."""
        import torch
        n = self.layout_info(direction)["slots"]
        rows = torch.empty(n, dtype=torch.int32, device="cuda")
        cols = torch.empty(n, dtype=torch.int32, device="cuda")
        vals = torch.empty(n, dtype=torch.float32, device="cuda")
        _check(lib().memxct_export_coo(self._h, int(direction), _ptr(rows), _ptr(cols), _ptr(vals), _stream(stream)),
               "memxct_export_coo")
        return rows, cols, vals

    def layout_rows(self, direction: int) -> np.ndarray:
        """Output position of every layout row (memxct_layout_rows)."""
        out = np.empty(self.layout_info(direction)["rows"], np.int64)
        _check(lib().memxct_layout_rows(self._h, direction, out.ctypes.data_as(ctypes.c_void_p)), "memxct_layout_rows")
        return out

    def layout_export(self, direction: int, p0: int = 0, p1: int = None) -> dict:
        if p1 is None:
            p1 = self.layout_info(direction)["parts"]
        nm, nso, ns = ctypes.c_int64(), ctypes.c_int64(), ctypes.c_int64()
        z = ctypes.c_void_p()
        _check(lib().memxct_layout_export(self._h, direction, p0, p1, z, z, z, z, z, z, z, z,
                                          ctypes.byref(nm), ctypes.byref(nso), ctypes.byref(ns)),
               "memxct_layout_export")
        out = {"stage_base": np.empty(p1 - p0 + 1, np.int64), "map_off": np.empty(p1 - p0 + 1, np.int64),
               "map": np.empty(nm.value, np.int32), "slot_off": np.empty(nso.value, np.int64),
               "ind": np.empty(ns.value, np.uint16), "val": np.empty(ns.value, np.float32),
               "lane_chunks": np.empty(32 * (nso.value - 1), np.uint16),
               "prow0": np.empty(p1 - p0 + 1, np.int64)}
        P = lambda a: a.ctypes.data_as(ctypes.c_void_p)
        _check(lib().memxct_layout_export(self._h, direction, p0, p1, P(out["stage_base"]),
                                          P(out["map_off"]), P(out["map"]), P(out["slot_off"]),
                                          P(out["ind"]), P(out["val"]), P(out["lane_chunks"]), P(out["prow0"]),
                                          ctypes.byref(nm),
                                          ctypes.byref(nso), ctypes.byref(ns)),
               "memxct_layout_export")
        return out

    # -- hot path -------------------------------------------------------------------------
    def _vec(self, t, domain, name):
        import torch
        if not (isinstance(t, torch.Tensor) and t.is_cuda and t.dtype == self.dtype and t.is_contiguous()):
            raise TypeError(f"{name} must be a contiguous CUDA {self.dtype} tensor")
        if t.numel() != self.local_size(domain):
            raise ValueError(f"{name} has {t.numel()} elements, expected {self.local_size(domain)}")
        return t

    def forward(self, x, y=None, stream=None):
        """y = A x (device tensors)."""
        import torch
        self._vec(x, 0, "x")
        if y is None:
            y = torch.empty(self.local_size(1), dtype=self.dtype, device=x.device)
        self._vec(y, 1, "y")
        _check(lib().memxct_forward(self._h, _ptr(x), _ptr(y), _stream(stream)), "memxct_forward")
        return y

    def back(self, y, x=None, stream=None):
        """x = A^T y (device tensors)."""
        import torch
        self._vec(y, 1, "y")
        if x is None:
            x = torch.empty(self.local_size(0), dtype=self.dtype, device=y.device)
        self._vec(x, 0, "x")
        _check(lib().memxct_back(self._h, _ptr(y), _ptr(x), _stream(stream)), "memxct_back")
        return x

    def cg(self, y, iters: int = 30, x=None, residuals: bool = False, stream=None):
        """CGLS from x0 = 0; returns x (and ||r_k||, k = 0..iters, if residuals)."""
        import torch
        self._vec(y, 1, "y")
        if x is None:
            x = torch.empty(self.local_size(0), dtype=self.dtype, device=y.device)
        self._vec(x, 0, "x")
        res = np.empty(iters + 1, np.float64) if residuals else None
        rp = res.ctypes.data_as(ctypes.c_void_p) if residuals else None
        _check(lib().memxct_cg(self._h, _ptr(y), _ptr(x), int(iters), rp, _stream(stream)), "memxct_cg")
        return (x, res) if residuals else x

    def sirt(self, y, iters: int = 45, x=None, residuals: bool = False, stream=None):
        """SIRT from x0 = 0 (memxct_sirt); returns x (and ||y - A x_k||, k = 0..iters)."""
        import torch
        self._vec(y, 1, "y")
        if x is None:
            x = torch.empty(self.local_size(0), dtype=self.dtype, device=y.device)
        self._vec(x, 0, "x")
        res = np.empty(iters + 1, np.float64)
        _check(lib().memxct_sirt(self._h, _ptr(y), _ptr(x), int(iters), res.ctypes.data_as(ctypes.c_void_p),
                                 _stream(stream)), "memxct_sirt")
        return (x, res) if residuals else x

    # -- multi-slice (slice-major [K, n] tensors) ---------------------------------------------
    def _batch(self, t, domain, name):
        import torch
        if not (isinstance(t, torch.Tensor) and t.is_cuda and t.dtype == self.dtype and t.is_contiguous()
                and t.dim() == 2 and t.shape[1] == self.local_size(domain)):
            raise TypeError(f"{name} must be a contiguous CUDA [slices, {self.local_size(domain)}] tensor")
        return t

    def forward_batch(self, x, y=None, stream=None):
        """y[s] = A x[s] for every slice s (one matrix stream per group of up to 8 slices)."""
        import torch
        self._batch(x, 0, "x")
        k = x.shape[0]
        if y is None:
            y = torch.empty(k, self.local_size(1), dtype=self.dtype, device=x.device)
        self._batch(y, 1, "y")
        _check(lib().memxct_forward_batch(self._h, k, _ptr(x), _ptr(y), _stream(stream)), "memxct_forward_batch")
        return y

    def back_batch(self, y, x=None, stream=None):
        import torch
        self._batch(y, 1, "y")
        k = y.shape[0]
        if x is None:
            x = torch.empty(k, self.local_size(0), dtype=self.dtype, device=y.device)
        self._batch(x, 0, "x")
        _check(lib().memxct_back_batch(self._h, k, _ptr(y), _ptr(x), _stream(stream)), "memxct_back_batch")
        return x

    def cg_batch(self, y, iters: int = 30, x=None, residuals: bool = False, stream=None):
        """Independent CGLS solves of every slice of y ([K, local_size(1)])."""
        import torch
        self._batch(y, 1, "y")
        k = y.shape[0]
        if x is None:
            x = torch.empty(k, self.local_size(0), dtype=self.dtype, device=y.device)
        self._batch(x, 0, "x")
        res = np.empty((k, iters + 1), np.float64) if residuals else None
        rp = res.ctypes.data_as(ctypes.c_void_p) if residuals else None
        _check(lib().memxct_cg_batch(self._h, k, _ptr(y), _ptr(x), int(iters), rp, _stream(stream)),
               "memxct_cg_batch")
        return (x, res) if residuals else x

    # host-buffer variants (numpy in, numpy out; copies happen inside the C call)
    def _host(self, a, domain, name):
        dt = np.float32 if self.precision == "fp32" else np.float64
        a = np.ascontiguousarray(a, dt)
        if a.size != self.local_size(domain):
            raise ValueError(f"{name} has {a.size} elements, expected {self.local_size(domain)}")
        return a

    def forward_host(self, x, y=None, stream=None):
        x = self._host(x, 0, "x")
        y = np.empty(self.local_size(1), x.dtype) if y is None else y
        _check(lib().memxct_forward_host(self._h, x.ctypes.data_as(ctypes.c_void_p),
                                         y.ctypes.data_as(ctypes.c_void_p), _stream(stream)),
               "memxct_forward_host")
        return y

    def back_host(self, y, x=None, stream=None):
        y = self._host(y, 1, "y")
        x = np.empty(self.local_size(0), y.dtype) if x is None else x
        _check(lib().memxct_back_host(self._h, y.ctypes.data_as(ctypes.c_void_p),
                                      x.ctypes.data_as(ctypes.c_void_p), _stream(stream)),
               "memxct_back_host")
        return x

    def cg_host_ptr(self, y_ptr: int, x_ptr: int, iters: int = 30, stream=None):
        """memxct_cg_host on raw host addresses (e.g. pinned torch CPU tensors' data_ptr())."""
        _check(lib().memxct_cg_host(self._h, ctypes.c_void_p(y_ptr), ctypes.c_void_p(x_ptr),
                                    int(iters), None, _stream(stream)), "memxct_cg_host")

    def cg_host(self, y, iters: int = 30, x=None, residuals: bool = False, stream=None):
        y = self._host(y, 1, "y")
        x = np.empty(self.local_size(0), y.dtype) if x is None else x
        res = np.empty(iters + 1, np.float64) if residuals else None
        rp = res.ctypes.data_as(ctypes.c_void_p) if residuals else None
        _check(lib().memxct_cg_host(self._h, y.ctypes.data_as(ctypes.c_void_p),
                                    x.ctypes.data_as(ctypes.c_void_p), int(iters), rp,
                                    _stream(stream)), "memxct_cg_host")
        return (x, res) if residuals else x
