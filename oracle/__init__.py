"""CPU oracle for the distance similarity self-join -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this package.  The product
(``paper_conf_ipps_galletg19_b200``) never imports it and shares no code with it.

The arithmetic lives in ``oracle.c`` (plain C, binary64, ``-ffp-contract=off``):

* ``bf_*``   -- O1, the definition written out: every ordered (i, j), i != j, with
               s(i, j) <= fl(eps*eps) (§II-A; "two nested loops").
* ``grid_*`` -- O2, a CPU eps-grid with a hash map of integer cell tuples and a full
               3^n neighbourhood scan (§II-B1).

This wrapper only marshals numpy arrays.  Parity status of each function is in
the header of oracle.c and in DESIGN.md §3.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

# Spinning OpenMP workers starve each other on CPU-quota-limited containers (measured here:
# 0.2 s vs 7 ms for the same C1 call); the oracle always runs with passive waiting.
os.environ.setdefault("OMP_WAIT_POLICY", "PASSIVE")

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_lib = None

_u64p = ctypes.POINTER(ctypes.c_uint64)
_u32p = ctypes.POINTER(ctypes.c_uint32)
_i64p = ctypes.POINTER(ctypes.c_int64)
_dblp = ctypes.POINTER(ctypes.c_double)


class OracleError(RuntimeError):
    pass


def build(force: bool = False) -> str:
    """Compile liboracle.so with the oracle's own Makefile (gcc, -ffp-contract=off)."""
    src = os.path.join(_HERE, "oracle.c")
    if force or not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < os.path.getmtime(src):
        subprocess.run(["make", "-C", _HERE, "-s", "-B" if force else "liboracle.so"], check=True)
    return _LIB_PATH


def _load():
    global _lib
    if _lib is not None:
        return _lib
    build()
    lib = ctypes.CDLL(_LIB_PATH)
    c = ctypes
    lib.orc_bf_count.argtypes = [_dblp, c.c_uint64, c.c_int, c.c_double, _u64p, _u64p]
    lib.orc_bf_rows.argtypes = [_dblp, c.c_uint64, c.c_int, c.c_double, _u32p, c.c_uint64, _u64p, _u32p, c.c_uint64]
    lib.orc_bf_pairs.argtypes = [_dblp, c.c_uint64, c.c_int, c.c_double, _u32p, c.c_uint64, _u64p]
    lib.orc_grid_count.argtypes = [_dblp, c.c_uint64, c.c_int, c.c_double, _u64p, _u64p, _u64p, _u64p]
    lib.orc_grid_rows.argtypes = [_dblp, c.c_uint64, c.c_int, c.c_double, _u32p, c.c_uint64, _u64p, _u32p, c.c_uint64]
    lib.orc_grid_pairs.argtypes = [_dblp, c.c_uint64, c.c_int, c.c_double, _u32p, c.c_uint64, _u64p]
    lib.orc_grid_cells.argtypes = [_dblp, c.c_uint64, c.c_int, c.c_double, _i64p, _u64p, _u32p, _u64p]
    lib.orc_grid_new.argtypes = [_dblp, c.c_uint64, c.c_int, c.c_double, c.POINTER(c.c_int)]
    lib.orc_grid_new.restype = c.c_void_p
    lib.orc_grid_delete.argtypes = [c.c_void_p]
    lib.orc_grid_delete.restype = None
    lib.orc_grid_rows_range.argtypes = [c.c_void_p, c.c_uint64, c.c_uint64, _u64p, _u32p, c.c_uint64]
    lib.orc_grid_rows_range.restype = c.c_int
    lib.orc_hash_pairs.argtypes = [_u32p, c.c_uint64]
    lib.orc_hash_pairs.restype = c.c_uint64
    lib.orc_num_threads.restype = c.c_int
    lib.orc_set_threads.argtypes = [c.c_int]
    for name in ("orc_bf_count", "orc_bf_rows", "orc_bf_pairs", "orc_grid_count", "orc_grid_rows",
                 "orc_grid_pairs", "orc_grid_cells"):
        getattr(lib, name).restype = c.c_int
    _lib = lib
    return lib


def _pts(points) -> np.ndarray:
    p = np.ascontiguousarray(points, dtype=np.float64)
    if p.ndim != 2:
        raise ValueError("points must be (N, dim)")
    return p


def _ptr(a, t):
    return a.ctypes.data_as(t)


def _check(rc: int, what: str):
    if rc != 0:
        raise OracleError(f"{what} failed with code {rc}")


def num_threads() -> int:
    return _load().orc_num_threads()


def set_threads(t: int) -> None:
    _load().orc_set_threads(int(t))


# ----------------------------------------------------------------------------- O1

def bf_count(points, eps: float):
    """O1 pair count and multiset hash: (count, hash)."""
    p = _pts(points)
    lib = _load()
    cnt, h = ctypes.c_uint64(), ctypes.c_uint64()
    _check(lib.orc_bf_count(_ptr(p, _dblp), p.shape[0], p.shape[1], float(eps), ctypes.byref(cnt), ctypes.byref(h)),
           "orc_bf_count")
    return int(cnt.value), int(h.value)


def bf_pairs(points, eps: float) -> np.ndarray:
    """O1 pair set, canonical (i, j) order, as an (M, 2) uint32 array."""
    p = _pts(points)
    lib = _load()
    cnt = ctypes.c_uint64()
    _check(lib.orc_bf_pairs(_ptr(p, _dblp), p.shape[0], p.shape[1], float(eps), None, 0, ctypes.byref(cnt)),
           "orc_bf_pairs(size)")
    out = np.empty((max(int(cnt.value), 1), 2), dtype=np.uint32)
    _check(lib.orc_bf_pairs(_ptr(p, _dblp), p.shape[0], p.shape[1], float(eps), _ptr(out, _u32p), out.shape[0],
                            ctypes.byref(cnt)), "orc_bf_pairs")
    return out[: int(cnt.value)]


def _rows(fn, points, eps, rows):
    p = _pts(points)
    r = np.ascontiguousarray(rows, dtype=np.uint32)
    lib = _load()
    off = np.zeros(r.shape[0] + 1, dtype=np.uint64)
    f = getattr(lib, fn)
    _check(f(_ptr(p, _dblp), p.shape[0], p.shape[1], float(eps), _ptr(r, _u32p), r.shape[0], _ptr(off, _u64p),
             None, 0), fn + "(size)")
    cols = np.empty(max(int(off[-1]), 1), dtype=np.uint32)
    _check(f(_ptr(p, _dblp), p.shape[0], p.shape[1], float(eps), _ptr(r, _u32p), r.shape[0], _ptr(off, _u64p),
             _ptr(cols, _u32p), cols.shape[0]), fn)
    return off, cols[: int(off[-1])]


def bf_rows(points, eps: float, rows):
    """O1 neighbour rows of the given query ids: (offsets[len+1], cols) with each row ascending."""
    return _rows("orc_bf_rows", points, eps, rows)


# ----------------------------------------------------------------------------- O2

def grid_count(points, eps: float, with_hash: bool = True):
    """O2: dict(count, calcs (full 3^n scan, j != i), hash, ncells)."""
    p = _pts(points)
    lib = _load()
    cnt, calcs, h, nc = ctypes.c_uint64(), ctypes.c_uint64(), ctypes.c_uint64(), ctypes.c_uint64()
    _check(lib.orc_grid_count(_ptr(p, _dblp), p.shape[0], p.shape[1], float(eps), ctypes.byref(cnt),
                              ctypes.byref(calcs), ctypes.byref(h) if with_hash else None, ctypes.byref(nc)),
           "orc_grid_count")
    return {"count": int(cnt.value), "calcs": int(calcs.value), "hash": int(h.value) if with_hash else None,
            "ncells": int(nc.value)}


def grid_pairs(points, eps: float) -> np.ndarray:
    """O2 pair set, canonical (i, j) order, (M, 2) uint32."""
    p = _pts(points)
    lib = _load()
    cnt = ctypes.c_uint64()
    _check(lib.orc_grid_pairs(_ptr(p, _dblp), p.shape[0], p.shape[1], float(eps), None, 0, ctypes.byref(cnt)),
           "orc_grid_pairs(size)")
    out = np.empty((max(int(cnt.value), 1), 2), dtype=np.uint32)
    _check(lib.orc_grid_pairs(_ptr(p, _dblp), p.shape[0], p.shape[1], float(eps), _ptr(out, _u32p), out.shape[0],
                              ctypes.byref(cnt)), "orc_grid_pairs")
    return out[: int(cnt.value)]


def grid_rows(points, eps: float, rows):
    """O2 neighbour rows of the given query ids: (offsets, cols), rows ascending."""
    return _rows("orc_grid_rows", points, eps, rows)


class Grid:
    """A persistent O2 grid (built once) whose rows are read in blocks of query ids:
    ``rows_range(lo, hi)`` -> (offsets[hi-lo+1], cols), each row ascending, i.e. the
    canonical (i, j) order of the queries lo .. hi-1.  Context manager."""

    def __init__(self, points, eps: float):
        self.p = _pts(points)  # kept alive: the C grid points into it
        lib = _load()
        rc = ctypes.c_int(0)
        self.g = lib.orc_grid_new(_ptr(self.p, _dblp), self.p.shape[0], self.p.shape[1], float(eps),
                                  ctypes.byref(rc))
        if not self.g:
            raise OracleError(f"orc_grid_new failed with code {rc.value}")

    def rows_range(self, lo: int, hi: int):
        lib = _load()
        off = np.zeros(hi - lo + 1, dtype=np.uint64)
        _check(lib.orc_grid_rows_range(self.g, int(lo), int(hi), _ptr(off, _u64p), None, 0), "orc_grid_rows_range")
        cols = np.empty(max(int(off[-1]), 1), dtype=np.uint32)
        _check(lib.orc_grid_rows_range(self.g, int(lo), int(hi), _ptr(off, _u64p), _ptr(cols, _u32p), cols.shape[0]),
               "orc_grid_rows_range")
        return off, cols[: int(off[-1])]

    def keys_range(self, lo: int, hi: int) -> np.ndarray:
        """The pairs of queries lo .. hi-1 as canonical uint64 keys i << 32 | j (ascending)."""
        off, cols = self.rows_range(lo, hi)
        i = np.repeat(np.arange(lo, hi, dtype=np.uint64), np.diff(off).astype(np.int64))
        return (i << np.uint64(32)) | cols.astype(np.uint64)

    def close(self):
        if getattr(self, "g", None):
            _load().orc_grid_delete(self.g)
            self.g = None

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def grid_cells(points, eps: float):
    """The oracle's grid: (coords[M, dim] int64, first[M+1], ids[N]) in first-seen cell order."""
    p = _pts(points)
    lib = _load()
    nc = ctypes.c_uint64()
    _check(lib.orc_grid_cells(_ptr(p, _dblp), p.shape[0], p.shape[1], float(eps), None, None, None,
                              ctypes.byref(nc)), "orc_grid_cells(size)")
    m = int(nc.value)
    coords = np.empty((max(m, 1), p.shape[1]), dtype=np.int64)
    first = np.empty(m + 1, dtype=np.uint64)
    ids = np.empty(max(p.shape[0], 1), dtype=np.uint32)
    _check(lib.orc_grid_cells(_ptr(p, _dblp), p.shape[0], p.shape[1], float(eps), _ptr(coords, _i64p),
                              _ptr(first, _u64p), _ptr(ids, _u32p), ctypes.byref(nc)), "orc_grid_cells")
    return coords[:m], first, ids[: p.shape[0]]


def hash_pairs(pairs) -> int:
    """The oracle's order-independent multiset hash of an (M, 2) uint32 pair array."""
    a = np.ascontiguousarray(pairs, dtype=np.uint32).reshape(-1, 2)
    return int(_load().orc_hash_pairs(_ptr(a, _u32p), a.shape[0]))


def canonical(pairs) -> np.ndarray:
    """Sort an (M, 2) uint32 pair array by (i, j) (test helper)."""
    a = np.ascontiguousarray(pairs, dtype=np.uint32).reshape(-1, 2)
    key = (a[:, 0].astype(np.uint64) << np.uint64(32)) | a[:, 1].astype(np.uint64)
    key.sort()
    out = np.empty((key.shape[0], 2), dtype=np.uint32)
    out[:, 0] = (key >> np.uint64(32)).astype(np.uint32)
    out[:, 1] = (key & np.uint64(0xFFFFFFFF)).astype(np.uint32)
    return out
