"""ctypes marshalling for libsj.so (include/sj.h).  No computation happens here."""
from __future__ import annotations

import ctypes
import os
import re
import sys

_HERE = os.path.dirname(os.path.abspath(__file__))
_ROOT = os.path.dirname(_HERE)
lib_path = os.environ.get("SJ_LIB_PATH") or os.path.join(_HERE, "libsj.so")  # override: experiments only
HEADER = os.path.join(_ROOT, "include", "sj.h")

SJ_OK, SJ_MORE, SJ_EINVAL, SJ_ENOMEM, SJ_ECUDA, SJ_EGRID, SJ_ESTATE = 0, 1, -1, -2, -3, -4, -5
SJ_PATTERN_LID_UNICOMP, SJ_PATTERN_GCG, SJ_PATTERN_UNICOMP = 0, 1, 2
SJ_ORDER_WORKLOAD, SJ_ORDER_CELL, SJ_ORDER_INPUT = 0, 1, 2
PATTERNS = {"lid_unicomp": SJ_PATTERN_LID_UNICOMP, "gcg": SJ_PATTERN_GCG, "unicomp": SJ_PATTERN_UNICOMP}
ORDERS = {"workload": SJ_ORDER_WORKLOAD, "cell": SJ_ORDER_CELL, "input": SJ_ORDER_INPUT}
(SJ_OPT_K, SJ_OPT_BATCH_PAIRS, SJ_OPT_STREAMS, SJ_OPT_SAMPLE_PPM, SJ_OPT_GRAB, SJ_OPT_COUNT_CALCS,
 SJ_OPT_BLOCKS_PER_SM, SJ_OPT_FAST_PATH, SJ_OPT_EXACT, SJ_OPT_QUEUE, SJ_OPT_OUT_BLOCKS) = range(1, 12)
_NAMES = {0: "SJ_OK", 1: "SJ_MORE", -1: "SJ_EINVAL", -2: "SJ_ENOMEM", -3: "SJ_ECUDA", -4: "SJ_EGRID",
          -5: "SJ_ESTATE"}


class SJError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"{_NAMES.get(code, code)}: {msg}")
        self.code = code


class SJStats(ctypes.Structure):
    _fields_ = [
        ("n", ctypes.c_uint64), ("dim", ctypes.c_uint32), ("key_bits", ctypes.c_uint32),
        ("n_cells", ctypes.c_uint64), ("fwd_runs", ctypes.c_uint64), ("dist_calcs", ctypes.c_uint64),
        ("calcs_measured", ctypes.c_uint64), ("pairs", ctypes.c_uint64), ("est_pairs", ctypes.c_uint64),
        ("batches", ctypes.c_uint32), ("retries", ctypes.c_uint32), ("join_launches", ctypes.c_uint32),
        ("k", ctypes.c_uint32), ("max_cell_load", ctypes.c_uint64),
        ("ms_build", ctypes.c_double), ("ms_estimate", ctypes.c_double), ("ms_join", ctypes.c_double),
        ("ms_join_sum", ctypes.c_double), ("ms_transfer", ctypes.c_double), ("ms_total", ctypes.c_double),
        ("fast_path", ctypes.c_uint32), ("nc", ctypes.c_uint32 * 8), ("n_chunks", ctypes.c_uint64),
        ("tiled_min", ctypes.c_uint32), ("pattern", ctypes.c_uint32), ("order", ctypes.c_uint32),
        ("est_fused", ctypes.c_uint32), ("lookup_hash", ctypes.c_uint32),
    ]

    def as_dict(self) -> dict:
        d = {f[0]: getattr(self, f[0]) for f in self._fields_}
        d["nc"] = list(self.nc)[: self.dim]
        return d


if not os.path.exists(lib_path):
    raise ImportError(f"{lib_path} is not built: run `python -c 'import __graft_entry__ as g; g.build()'` "
                      "(the CUDA path has no CPU fallback)")

_lib = ctypes.CDLL(lib_path)
_vp, _u64, _i64, _int, _dbl = ctypes.c_void_p, ctypes.c_uint64, ctypes.c_int64, ctypes.c_int, ctypes.c_double
_sig = {
    "sj_abi_version": (_int, []),
    "sj_kernel_launches": (_u64, []),
    "sj_last_error": (ctypes.c_char_p, []),
    "sj_create": (_vp, [_vp, _u64, _int, _dbl]),
    "sj_create_ex": (_vp, [_vp, _u64, _int, _dbl, _int, _int]),
    "sj_self_join": (_int, [_vp, _vp, _u64, ctypes.POINTER(_u64)]),
    "sj_destroy": (None, [_vp]),
    "sj_set_option": (_int, [_vp, _int, _i64]),
    "sj_set_slice": (_int, [_vp, _int, _int]),
    "sj_get_stats": (_int, [_vp, ctypes.POINTER(SJStats)]),
    "sj_export_index": (_int, [_vp, _vp, _u64, ctypes.POINTER(_u64)]),
    "sj_create_from_index": (_vp, [_vp, _u64]),
    "sj_create_from_index_view": (_vp, [_vp, _u64]),
    "sj_create_part": (_vp, [_vp, _vp, _u64, _u64, _int, _dbl, _vp]),
    "sj_forward_offsets": (_int, [_int, _vp, _u64]),
    "sj_slice_chunks": (_i64, [_u64, _int, _int, _vp, _u64]),
    "sj_batch_chunks": (_i64, [_u64, _u64, _u64, _int, _vp, _u64]),
    "sj_measure_fp64": (_int, [ctypes.POINTER(_dbl), ctypes.POINTER(_dbl)]),
    "sj_measure_atomics": (_int, [ctypes.POINTER(_dbl), ctypes.POINTER(_dbl)]),
    "sj_neighbor_csr": (_int, [_vp, _vp, _vp, _u64, ctypes.POINTER(_u64)]),
    "sj_set_stream": (None, [_vp]),
    "sj_part_bounds": (_int, [_vp, _u64, _int, _vp, _vp]),
    "sj_part_columns": (_i64, [_dbl, _dbl, _dbl]),
    "sj_part_histogram": (_int, [_vp, _u64, _int, _dbl, _dbl, _u64, _vp]),
    "sj_part_pack": (_int, [_vp, _vp, _u64, _int, _dbl, _dbl, _vp, _u64, _int, _vp, _vp, _vp, _vp, _vp, _vp]),
}
for _n, (_r, _a) in _sig.items():
    if os.environ.get("SJ_LIB_PATH") and not hasattr(_lib, _n):
        continue  # an older experimental build (SJ_LIB_PATH) may lack newer entry points
    _f = getattr(_lib, _n)
    _f.restype = _r
    _f.argtypes = _a


def header_functions() -> list:
    """Function names declared in include/sj.h (for the symbol-export test)."""
    txt = open(HEADER).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(sj_[a-z0-9_]+)\s*\(", txt)))


def _ptr(x) -> int:
    """Raw address of a numpy array, torch tensor, ctypes buffer or int (None -> 0)."""
    if x is None:
        return 0
    if isinstance(x, int):
        return x
    if hasattr(x, "data_ptr"):
        return int(x.data_ptr())
    if hasattr(x, "ctypes"):
        return int(x.ctypes.data)
    return ctypes.addressof(x)


def _order_after_torch() -> None:
    """Name torch's current CUDA stream as the caller's stream (sj_set_stream), so the library
    orders its work after whatever torch queued there (inputs still being written, buffers
    still in use).  Argument marshalling only: no device work happens here."""
    torch = sys.modules.get("torch")
    if torch is None or not torch.cuda.is_available() or not torch.cuda.is_initialized():
        _lib.sj_set_stream(None)
        return
    _lib.sj_set_stream(torch.cuda.current_stream().cuda_stream or None)


def _err(code: int) -> SJError:
    return SJError(code, (_lib.sj_last_error() or b"").decode())


def _check(code: int) -> int:
    if code < 0:
        raise _err(code)
    return code


# ------------------------------------------------------------------ same-name wrappers

def sj_abi_version() -> int:
    return _lib.sj_abi_version()


def sj_set_stream(stream) -> None:
    """stream: a torch.cuda.Stream, a raw cudaStream_t (int) or None (legacy default stream)."""
    raw = getattr(stream, "cuda_stream", stream)
    _lib.sj_set_stream(raw or None)


def sj_kernel_launches() -> int:
    return int(_lib.sj_kernel_launches())


def sj_last_error() -> str:
    return (_lib.sj_last_error() or b"").decode()


def _shape(points, n, dim, eps):
    if eps is None:  # (points, eps) form
        eps = n
        shape = tuple(points.shape)
        if len(shape) != 2:
            raise ValueError("points must be (N, dim)")
        n, dim = shape
        if hasattr(points, "dtype") and str(points.dtype) not in ("float64", "torch.float64"):
            raise TypeError("points must be float64")
        if hasattr(points, "is_contiguous") and not points.is_contiguous():
            raise ValueError("points must be contiguous")
        if hasattr(points, "flags") and not points.flags["C_CONTIGUOUS"]:
            raise ValueError("points must be C-contiguous")
    return n, dim, eps


def sj_create(points, n: int | None = None, dim: int | None = None, eps: float | None = None) -> int:
    """sj_create(points, eps) or sj_create(ptr, n, dim, eps).  Returns the raw handle (int)."""
    n, dim, eps = _shape(points, n, dim, eps)
    _order_after_torch()
    h = _lib.sj_create(_ptr(points), int(n), int(dim), float(eps))
    if not h:
        raise SJError(SJ_EINVAL, sj_last_error())
    return h


def sj_create_ex(points, n=None, dim=None, eps=None, pattern: int = 0, order: int = 0) -> int:
    """sj_create_ex(points, eps, pattern=, order=) or (ptr, n, dim, eps, pattern, order)."""
    n, dim, eps = _shape(points, n, dim, eps)
    _order_after_torch()
    h = _lib.sj_create_ex(_ptr(points), int(n), int(dim), float(eps), int(pattern), int(order))
    if not h:
        raise SJError(SJ_EINVAL, sj_last_error())
    return h


def sj_create_part(points, ids, n_query: int, eps: float, origin) -> int:
    """sj_create_part(points (n, dim) float64, ids (n,) uint32 or None, n_query, eps, origin (dim,)):
    a partition of a larger join -- the first n_query rows are its queries, the rest its halo."""
    import numpy as np

    n, dim, eps = _shape(points, eps, None, None)
    org = np.ascontiguousarray(np.asarray(origin, dtype=np.float64).reshape(-1))
    if org.shape[0] != dim:
        raise SJError(SJ_EINVAL, f"origin needs {dim} values")
    _order_after_torch()
    h = _lib.sj_create_part(_ptr(points), _ptr(ids), int(n), int(n_query), int(dim), float(eps), org.ctypes.data)
    if not h:
        raise SJError(SJ_EINVAL, sj_last_error())
    return h


def sj_create_from_index(blob, nbytes: int) -> int:
    _order_after_torch()
    h = _lib.sj_create_from_index(_ptr(blob), int(nbytes))
    if not h:
        raise SJError(SJ_EINVAL, sj_last_error())
    return h


def sj_create_from_index_view(blob, nbytes: int) -> int:
    """Zero copy: the handle's index arrays alias the (device) blob, which must outlive it."""
    _order_after_torch()
    h = _lib.sj_create_from_index_view(_ptr(blob), int(nbytes))
    if not h:
        raise SJError(SJ_EINVAL, sj_last_error())
    return h


def sj_self_join(h: int, out, cap: int):
    """Returns (status, count) with status SJ_OK or SJ_MORE; raises SJError on error."""
    cnt = _u64(0)
    _order_after_torch()
    rc = _lib.sj_self_join(h, _ptr(out), int(cap), ctypes.byref(cnt))
    _check(rc)
    return rc, int(cnt.value)


def sj_neighbor_csr(h: int, row_off, nbrs, cap: int) -> int:
    """Fills row_off (uint64[n+1]) and, if nbrs is given, nbrs (uint32[cap]); returns the
    total number of neighbour entries.  Raises SJError on error (incl. cap < total)."""
    tot = _u64(0)
    _order_after_torch()
    _check(_lib.sj_neighbor_csr(h, _ptr(row_off), _ptr(nbrs), int(cap), ctypes.byref(tot)))
    return int(tot.value)


def sj_destroy(h: int) -> None:
    _lib.sj_destroy(h)


def sj_set_option(h: int, opt: int, value: int) -> None:
    _check(_lib.sj_set_option(h, int(opt), int(value)))


def sj_set_slice(h: int, rank: int, world: int) -> None:
    _check(_lib.sj_set_slice(h, int(rank), int(world)))


def sj_get_stats(h: int) -> dict:
    st = SJStats()
    _check(_lib.sj_get_stats(h, ctypes.byref(st)))
    return st.as_dict()


def sj_export_index(h: int, dst=None, cap: int = 0) -> int:
    nbytes = _u64(0)
    _order_after_torch()
    _check(_lib.sj_export_index(h, _ptr(dst), int(cap), ctypes.byref(nbytes)))
    return int(nbytes.value)


def sj_forward_offsets(dim: int):
    import numpy as np

    f = _check(_lib.sj_forward_offsets(int(dim), None, 0))
    out = np.zeros((f, dim), dtype=np.int8)
    _check(_lib.sj_forward_offsets(int(dim), out.ctypes.data, out.size))
    return out


def sj_slice_chunks(n_chunks: int, rank: int, world: int):
    import numpy as np

    cnt = _check(_lib.sj_slice_chunks(int(n_chunks), int(rank), int(world), None, 0))
    out = np.zeros(max(cnt, 1), dtype=np.uint32)
    _check(_lib.sj_slice_chunks(int(n_chunks), int(rank), int(world), out.ctypes.data, out.size))
    return out[:cnt]


def sj_batch_chunks(n_chunks: int, n_batches: int, batch: int, queue: int = 1):
    import numpy as np

    cnt = _check(_lib.sj_batch_chunks(int(n_chunks), int(n_batches), int(batch), int(queue), None, 0))
    out = np.zeros(max(cnt, 1), dtype=np.uint32)
    _check(_lib.sj_batch_chunks(int(n_chunks), int(n_batches), int(batch), int(queue), out.ctypes.data, out.size))
    return out[:cnt]


# ------------------------------------------------------------------ slab partition (sj_part_*)

def _part_points(points):
    n, dim, _ = _shape(points, 0.0, None, None)
    if not (hasattr(points, "is_cuda") and points.is_cuda):
        raise SJError(SJ_EINVAL, "sj_part_*: points must be a CUDA float64 tensor")
    return n, dim


def sj_part_bounds(points):
    """(min list, max list) per dimension of a CUDA (n, dim) float64 tensor."""
    import numpy as np

    n, dim = _part_points(points)
    mn, mx = np.empty(dim), np.empty(dim)
    _order_after_torch()
    _check(_lib.sj_part_bounds(_ptr(points), n, dim, mn.ctypes.data, mx.ctypes.data))
    return mn.tolist(), mx.tolist()


def sj_part_columns(origin0: float, max0: float, eps: float) -> int:
    return int(_check(_lib.sj_part_columns(float(origin0), float(max0), float(eps))))


def sj_part_histogram(points, origin0: float, eps: float, ncol: int):
    """Column histogram (CUDA int64 tensor of ncol counts) of the local points."""
    import torch

    n, dim = _part_points(points)
    hist = torch.empty(ncol, dtype=torch.int64, device=points.device)
    _order_after_torch()
    _check(_lib.sj_part_histogram(_ptr(points), n, dim, float(origin0), float(eps), int(ncol), _ptr(hist)))
    return hist


def sj_part_pack(points, ids, origin0: float, eps: float, hist, world: int):
    """Rows packed per destination: (own_pts, own_ids, own_counts, halo_pts, halo_ids, halo_counts);
    the point / id tensors are CUDA (n, dim) float64 / (n,) int32 (uint32 bits), counts lists."""
    import numpy as np
    import torch

    n, dim = _part_points(points)
    dev = points.device
    if ids is not None and (ids.dtype != torch.int32 or ids.numel() != n or not ids.is_contiguous()):
        raise SJError(SJ_EINVAL, "sj_part_pack: ids must be a contiguous int32 tensor of n global ids")
    own_p = torch.empty((max(n, 1), dim), dtype=torch.float64, device=dev)
    own_i = torch.empty(max(n, 1), dtype=torch.int32, device=dev)
    halo_p = torch.empty((max(n, 1), dim), dtype=torch.float64, device=dev)
    halo_i = torch.empty(max(n, 1), dtype=torch.int32, device=dev)
    oc = np.zeros(world, dtype=np.uint64)
    hc = np.zeros(world, dtype=np.uint64)
    _order_after_torch()
    _check(_lib.sj_part_pack(_ptr(points), _ptr(ids), n, dim, float(origin0), float(eps), _ptr(hist), hist.numel(),
                             int(world), _ptr(own_p), _ptr(own_i), oc.ctypes.data, _ptr(halo_p), _ptr(halo_i),
                             hc.ctypes.data))
    return own_p, own_i, [int(x) for x in oc], halo_p, halo_i, [int(x) for x in hc]


def sj_measure_fp64():
    r, ms = _dbl(0), _dbl(0)
    _check(_lib.sj_measure_fp64(ctypes.byref(r), ctypes.byref(ms)))
    return r.value, ms.value


def sj_measure_atomics():
    r, ms = _dbl(0), _dbl(0)
    _check(_lib.sj_measure_atomics(ctypes.byref(r), ctypes.byref(ms)))
    return r.value, ms.value


# ------------------------------------------------------------------ RAII convenience

class Handle:
    """Owning wrapper of an sj_handle*."""

    def __init__(self, points=None, eps: float | None = None, *, raw: int | None = None, pattern=None, order=None,
                 part=None, **options):
        if raw is not None:
            self.h = raw
        elif part is not None:  # (ids, n_query, origin): a partition (sj_create_part)
            ids, n_query, origin = part
            self.h = sj_create_part(points, ids, n_query, eps, origin)
        elif pattern is None and order is None:
            self.h = sj_create(points, eps)
        else:
            pat = PATTERNS.get(pattern, pattern) if pattern is not None else 0
            odr = ORDERS.get(order, order) if order is not None else 0
            self.h = sj_create_ex(points, eps, pattern=pat, order=odr)
        for k, v in options.items():
            self.set_option(k, v)

    @classmethod
    def from_index(cls, blob, nbytes: int, view: bool = False) -> "Handle":
        """A handle from an exported index blob; view=True aliases a device blob (zero copy: the
        blob must stay alive and unchanged while the handle exists -- the handle keeps a
        reference to the object passed)."""
        if view:
            h = cls(raw=sj_create_from_index_view(blob, nbytes))
            h._blob = blob
            return h
        return cls(raw=sj_create_from_index(blob, nbytes))

    _OPTS = {"k": SJ_OPT_K, "batch_pairs": SJ_OPT_BATCH_PAIRS, "streams": SJ_OPT_STREAMS,
             "sample_ppm": SJ_OPT_SAMPLE_PPM, "grab": SJ_OPT_GRAB, "count_calcs": SJ_OPT_COUNT_CALCS,
             "blocks_per_sm": SJ_OPT_BLOCKS_PER_SM, "fast_path": SJ_OPT_FAST_PATH, "exact": SJ_OPT_EXACT,
             "queue": SJ_OPT_QUEUE, "out_blocks": SJ_OPT_OUT_BLOCKS}

    def set_option(self, name, value) -> None:
        sj_set_option(self.h, self._OPTS[name] if isinstance(name, str) else name, int(value))

    def set_slice(self, rank: int, world: int) -> None:
        sj_set_slice(self.h, rank, world)

    def self_join(self, out=None, cap: int = 0):
        return sj_self_join(self.h, out, cap)

    def count(self) -> int:
        return sj_self_join(self.h, None, 0)[1]

    def stats(self) -> dict:
        return sj_get_stats(self.h)

    def neighbor_csr(self, device: str = "cuda"):
        """Device-resident CSR (needs pattern="gcg"): (row_off int64 (n+1,), nbrs int32 (total,))
        torch tensors holding the uint64 offsets / uint32 input ids, on `device` ("cpu":
        pinned host memory)."""
        import torch

        n = self.stats()["n"]
        pin = device == "cpu"
        kw = dict(pin_memory=True) if pin else dict(device=device)
        row_off = torch.empty(n + 1, dtype=torch.int64, **kw)
        total = sj_neighbor_csr(self.h, row_off, None, 0)
        nbrs = torch.empty(max(total, 1), dtype=torch.int32, **kw)
        sj_neighbor_csr(self.h, row_off, nbrs, max(total, 1))
        return row_off, nbrs[:total]

    def export_index(self, dst=None, cap: int = 0) -> int:
        return sj_export_index(self.h, dst, cap)

    def close(self) -> None:
        if getattr(self, "h", None):
            sj_destroy(self.h)
            self.h = None

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def self_join_pairs(handle: Handle, device: str = "cuda", total: int | None = None):
    """All pairs as a torch int32 tensor (M, 2) holding the uint32 ids (count-only call
    first to size the buffer, then one sj_self_join into it)."""
    import torch

    if total is None:
        total = handle.count()
    if device == "cpu":
        out = torch.empty((max(total, 1), 2), dtype=torch.int32, pin_memory=True)
    else:
        out = torch.empty((max(total, 1), 2), dtype=torch.int32, device=device)
    got, rc = 0, SJ_MORE
    rc, got = handle.self_join(out, max(total, 1))
    if rc != SJ_OK:
        raise SJError(rc, "unexpected SJ_MORE with an exactly sized buffer")
    return out[:got]
