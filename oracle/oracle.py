"""ctypes binding of the C oracle (memxct_oracle.c) plus tiny numpy glue.

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).  The glue here does no arithmetic of the
method: it allocates arrays, calls the C functions and reshapes results.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "memxct_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

__all__ = [
    "build_oracle", "lib", "trace_ray", "count_nnz", "row_lengths", "trace_all", "gilbert2d",
    "d2xy", "hilbert_rank", "spmv_coo", "spmv_canonical", "cgls", "dot_canonical",
    "coo_to_csr", "sampled_back_rows", "sirt", "chord", "chords", "sample_rows", "sample_columns",
    "spmv_csr_threaded", "csr_transpose",
]


class _Csr(ctypes.Structure):
    _fields_ = [("nrows", ctypes.c_int64), ("nnz", ctypes.c_int64), ("ptr", ctypes.POINTER(ctypes.c_int64)),
                ("idx", ctypes.POINTER(ctypes.c_int32)), ("len", ctypes.POINTER(ctypes.c_double))]


def build_oracle(force: bool = False) -> str:
    """Compile the oracle with gcc (-O2 -ffp-contract=off; all fmas are explicit)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".{os.getpid()}.tmp"
        subprocess.check_call(["gcc", "-O2", "-ffp-contract=off", "-fPIC", "-shared", "-std=gnu11",
                               "-pthread", "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        build_oracle()
        L = ctypes.CDLL(_LIB)
        i32, i64, dbl, vp = ctypes.c_int32, ctypes.c_int64, ctypes.c_double, ctypes.c_void_p
        L.orc_trace_ray.restype = i64
        L.orc_trace_ray.argtypes = [i32, i32, i32, i64, vp, vp, i64]
        L.orc_count_nnz.restype = i64
        L.orc_count_nnz.argtypes = [i32, i32, i32]
        L.orc_row_lengths.restype = None
        L.orc_row_lengths.argtypes = [i32, i32, i32, vp]
        L.orc_trace_all.restype = i64
        L.orc_trace_all.argtypes = [i32, i32, i32, vp, vp, vp, i64]
        L.orc_gilbert2d.restype = i64
        L.orc_gilbert2d.argtypes = [i32, i32, vp, vp]
        L.orc_d2xy.restype = None
        L.orc_d2xy.argtypes = [i32, i64, ctypes.POINTER(i32), ctypes.POINTER(i32)]
        L.orc_hilbert_rank.restype = ctypes.c_int
        L.orc_hilbert_rank.argtypes = [i32, i32, i32, vp]
        L.orc_spmv_coo.restype = None
        L.orc_spmv_coo.argtypes = [i64, vp, vp, vp, vp, i64, vp]
        L.orc_spmv_canonical.restype = None
        L.orc_spmv_canonical.argtypes = [i64, vp, vp, vp, vp, vp, vp]
        L.orc_cgls.restype = ctypes.c_int
        L.orc_cgls.argtypes = [i64, i64, i64, vp, vp, vp, vp, i32, i32, vp, vp, i64, i64, vp, vp, vp]
        L.orc_sirt.restype = ctypes.c_int
        L.orc_sirt.argtypes = [i64, i64, i64, vp, vp, vp, vp, i32, vp, vp]
        L.orc_dot_canonical.restype = dbl
        L.orc_dot_canonical.argtypes = [i64, vp, vp, vp, i64]
        L.orc_chord.restype = dbl
        L.orc_chord.argtypes = [i32, i32, i32, i64]
        L.orc_chords.restype = None
        L.orc_chords.argtypes = [i32, i32, i32, vp]
        L.orc_sample_rows.restype = ctypes.POINTER(_Csr)
        L.orc_sample_rows.argtypes = [i32, i32, i32, i64, vp, i32]
        L.orc_sample_columns.restype = ctypes.POINTER(_Csr)
        L.orc_sample_columns.argtypes = [i32, i32, i32, i64, vp, i32]
        L.orc_csr_free.restype = None
        L.orc_csr_free.argtypes = [ctypes.POINTER(_Csr)]
        L.orc_csr_transpose.restype = ctypes.POINTER(_Csr)
        L.orc_csr_transpose.argtypes = [i64, vp, vp, vp, i64]
        L.orc_spmv_csr_threaded.restype = i32
        L.orc_spmv_csr_threaded.argtypes = [i64, vp, vp, vp, vp, vp, i32]
        _lib = L
    return _lib


def _p(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


def trace_ray(n: int, m: int, c: int, ray: int):
    """(pixels int32, lengths float64) of one ray in trace order."""
    cap = 2 * n + 4
    pix = np.empty(cap, np.int32)
    ln = np.empty(cap, np.float64)
    k = lib().orc_trace_ray(n, m, c, ray, _p(pix), _p(ln), cap)
    assert k >= 0
    return pix[:k].copy(), ln[:k].copy()


def count_nnz(n: int, m: int, c: int) -> int:
    return int(lib().orc_count_nnz(n, m, c))


def row_lengths(n: int, m: int, c: int) -> np.ndarray:
    out = np.empty(m * c, np.int32)
    lib().orc_row_lengths(n, m, c, _p(out))
    return out


def trace_all(n: int, m: int, c: int):
    """Whole A as COO (rows int32, cols int32, vals float64), ray-major trace order."""
    nnz = int(row_lengths(n, m, c).astype(np.int64).sum())
    rows = np.empty(max(nnz, 1), np.int32)
    cols = np.empty(max(nnz, 1), np.int32)
    vals = np.empty(max(nnz, 1), np.float64)
    k = lib().orc_trace_all(n, m, c, _p(rows), _p(cols), _p(vals), nnz)
    assert k == nnz
    return rows[:nnz], cols[:nnz], vals[:nnz]


def gilbert2d(w: int, h: int):
    xs = np.empty(w * h, np.int32)
    ys = np.empty(w * h, np.int32)
    k = lib().orc_gilbert2d(w, h, _p(xs), _p(ys))
    assert k == w * h
    return xs, ys


def d2xy(n: int, d: int):
    x, y = ctypes.c_int32(), ctypes.c_int32()
    lib().orc_d2xy(n, d, ctypes.byref(x), ctypes.byref(y))
    return x.value, y.value


def hilbert_rank(h: int, w: int, t: int) -> np.ndarray:
    """rank[i*w + j] = two-level pseudo-Hilbert position of cell (row i, col j)."""
    out = np.empty(h * w, np.int64)
    rc = lib().orc_hilbert_rank(h, w, t, _p(out))
    if rc != 0:
        raise ValueError(f"orc_hilbert_rank failed ({rc})")
    return out


def spmv_coo(rows, cols, vals, x, nrows: int) -> np.ndarray:
    rows = np.ascontiguousarray(rows, np.int32)
    cols = np.ascontiguousarray(cols, np.int32)
    vals = np.ascontiguousarray(vals, np.float64)
    x = np.ascontiguousarray(x, np.float64)
    y = np.empty(nrows, np.float64)
    lib().orc_spmv_coo(len(rows), _p(rows), _p(cols), _p(vals), _p(x), nrows, _p(y))
    return y


def coo_to_csr(rows, cols, vals, nrows: int):
    """Stable CSR (entry order preserved inside each row).  Pure index bookkeeping."""
    order = np.argsort(rows, kind="stable")
    ptr = np.zeros(nrows + 1, np.int64)
    np.add.at(ptr, rows.astype(np.int64) + 1, 1)
    ptr = np.cumsum(ptr)
    return ptr, np.ascontiguousarray(cols[order], np.int32), np.ascontiguousarray(vals[order], np.float64)


def spmv_canonical(rows, cols, vals, col_key, x, nrows: int) -> np.ndarray:
    ptr, c, v = coo_to_csr(np.asarray(rows), np.asarray(cols), np.asarray(vals), nrows)
    col_key = np.ascontiguousarray(col_key, np.int64)
    x = np.ascontiguousarray(x, np.float64)
    y = np.empty(nrows, np.float64)
    lib().orc_spmv_canonical(nrows, _p(ptr), _p(c), _p(v), _p(col_key), _p(x), _p(y))
    return y


def dot_canonical(a, b, key, chunk: int) -> float:
    a = np.ascontiguousarray(a, np.float64)
    b = np.ascontiguousarray(b, np.float64)
    key = np.ascontiguousarray(key, np.int64)
    return float(lib().orc_dot_canonical(len(a), _p(a), _p(b), _p(key), chunk))


def cgls(rows, cols, vals, y, nrows: int, ncols: int, iters: int, canonical: bool = False,
         row_key=None, col_key=None, chunk_rows: int = 0, chunk_cols: int = 0):
    """CGLS from x0 = 0.  Returns (x, res[iters+1], true_res[iters+1], iterations_done)."""
    rows = np.ascontiguousarray(rows, np.int32)
    cols = np.ascontiguousarray(cols, np.int32)
    vals = np.ascontiguousarray(vals, np.float64)
    y = np.ascontiguousarray(y, np.float64)
    x = np.empty(ncols, np.float64)
    res = np.empty(iters + 1, np.float64)
    tres = np.empty(iters + 1, np.float64)
    if canonical:
        row_key = np.ascontiguousarray(row_key, np.int64)
        col_key = np.ascontiguousarray(col_key, np.int64)
        rk, ck = _p(row_key), _p(col_key)
    else:
        rk = ck = None
    done = lib().orc_cgls(nrows, ncols, len(rows), _p(rows), _p(cols), _p(vals), _p(y), iters,
                          1 if canonical else 0, rk, ck, chunk_rows, chunk_cols,
                          _p(x), _p(res), _p(tres))
    return x, res, tres, int(done)


def sirt(rows, cols, vals, y, nrows: int, ncols: int, iters: int):
    """SIRT from x0 = 0.  Returns (x, res[iters+1] = ||y - A x_k||)."""
    rows = np.ascontiguousarray(rows, np.int32)
    cols = np.ascontiguousarray(cols, np.int32)
    vals = np.ascontiguousarray(vals, np.float64)
    y = np.ascontiguousarray(y, np.float64)
    x = np.empty(ncols, np.float64)
    res = np.empty(iters + 1, np.float64)
    lib().orc_sirt(nrows, ncols, len(rows), _p(rows), _p(cols), _p(vals), _p(y), iters, _p(x), _p(res))
    return x, res


def chord(n: int, m: int, c: int, ray: int) -> float:
    """Closed-form length of ray `ray` inside the grid square."""
    return float(lib().orc_chord(n, m, c, int(ray)))


def chords(n: int, m: int, c: int) -> np.ndarray:
    """Closed-form chord of every ray (natural order, M*C doubles) = the row sums of A."""
    out = np.empty(m * c, np.float64)
    lib().orc_chords(n, m, c, _p(out))
    return out


def _take_csr(ptr):
    if not ptr:
        raise ValueError("oracle sampled function failed (repeated pixels?)")
    s = ptr.contents
    nr, nz = int(s.nrows), int(s.nnz)
    rp = np.ctypeslib.as_array(s.ptr, shape=(nr + 1,)).copy()
    idx = np.ctypeslib.as_array(s.idx, shape=(max(nz, 1),))[:nz].copy()
    ln = np.ctypeslib.as_array(s.len, shape=(max(nz, 1),))[:nz].copy()
    lib().orc_csr_free(ptr)
    return rp, idx, ln


def sample_rows(n: int, m: int, c: int, rays, threads: int = 0):
    """Rows of A for natural ray indices `rays` (orc_sample_rows): (ptr, pixels int32, lengths)."""
    r = np.ascontiguousarray(rays, np.int64)
    return _take_csr(lib().orc_sample_rows(n, m, c, len(r), _p(r), int(threads)))


def sample_columns(n: int, m: int, c: int, pixels, threads: int = 0):
    """Columns of A for distinct natural pixel indices (orc_sample_columns): (ptr, rays int32
    ascending, lengths) per pixel."""
    p = np.ascontiguousarray(pixels, np.int64)
    return _take_csr(lib().orc_sample_columns(n, m, c, len(p), _p(p), int(threads)))


def csr_transpose(ptr, idx, vals, ncols: int):
    """Stable CSR transpose (orc_csr_transpose): (ptr, row indices, values) per column."""
    ptr = np.ascontiguousarray(ptr, np.int64)
    idx = np.ascontiguousarray(idx, np.int32)
    vals = np.ascontiguousarray(vals, np.float64)
    return _take_csr(lib().orc_csr_transpose(len(ptr) - 1, _p(ptr), _p(idx), _p(vals), int(ncols)))


def spmv_csr_threaded(ptr, cols, vals, x, threads: int = 0):
    """Threaded CSR y = A x (orc_spmv_csr_threaded); returns (y, threads used)."""
    ptr = np.ascontiguousarray(ptr, np.int64)
    cols = np.ascontiguousarray(cols, np.int32)
    vals = np.ascontiguousarray(vals, np.float64)
    x = np.ascontiguousarray(x, np.float64)
    y = np.empty(len(ptr) - 1, np.float64)
    nt = lib().orc_spmv_csr_threaded(len(ptr) - 1, _p(ptr), _p(cols), _p(vals), _p(x), _p(y), int(threads))
    return y, int(nt)


def sampled_back_rows(n: int, m: int, c: int, pixels, threads: int = 0):
    """Rows of A^T for distinct pixels (orc_sample_columns): a list of (ray indices int64,
    lengths float64) per pixel, rays ascending."""
    ptr, rays, ln = sample_columns(n, m, c, pixels, threads)
    return [(rays[ptr[q]:ptr[q + 1]].astype(np.int64), ln[ptr[q]:ptr[q + 1]]) for q in range(len(ptr) - 1)]
