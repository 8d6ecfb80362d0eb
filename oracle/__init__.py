"""oracle — TEST INFRASTRUCTURE ONLY.

Plain CPU implementation of the OLAP hot path (Malik et al., IPDPSW 2012,
/root/reference/PAPER.md), used to prove parity of the CUDA path.  Only
``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this package.  It shares no code with
``paper_conf_ipps_malikrse12_b200`` and never imports it.

Functions (all cite the passage they follow in oracle.cpp):
  query()      Eq. 1 / Eq. 3 / PAPER.md:25 — odometer sub-cube aggregation.
  Dict         PAPER.md:252-256 — one std::map dictionary per text column.
  factscan()   PAPER.md:206-208 — filtered aggregation over a fact table.
  factbuild()  PAPER.md:101 — the cube built from fact rows (row loop; float: fp64 per cell, one rounding).
  rollup(), convert_range()  PAPER.md:103-136, Fig. 1, Eq. 1-2 — multi-resolution cube set.
  tablescan()  Eq. 11-12, PAPER.md:206-216 — the paper's GPU query Q_D over a column store.
  fill()       the counter-based cell generator (independent re-implementation).
  sched.Fig10  Fig. 10 / Eq. 4-18 — the CPU/GPU scheduling algorithm,
               plain Python (oracle/sched.py), for the dispatcher.

Parity of every function is pinned in tests/test_oracle_*.py against brute
force (numpy slicing), an independent summed-area-table algorithm, the affine
closed form, hand-worked examples (tests/golden/) and invariants; none is "parity unpinned".
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.cpp")
def _host_tag() -> str:
    """The build is -march=native: one library per host CPU model + flags (the GPU box's host is
    not this one, and an AVX-512 build must never load on a CPU without it)."""
    import hashlib
    sig = ""
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith(("model name", "flags")):
                    sig += line
                if line.strip() == "":
                    break
    except OSError:
        pass
    return hashlib.sha1(sig.encode()).hexdigest()[:10]


_LIB = os.path.join(_HERE, f"liboracle-{_host_tag()}.so")
# -O3 -march=native for the timed CPU baseline; -ffp-contract=off keeps every
# a*b+c a separate multiply and add (no FMA contraction), so the arithmetic is the source's,
# bit for bit, whatever the host's ISA.  GCC never reassociates fp sums without -ffast-math.
CFLAGS = ["-O3", "-march=native", "-ffp-contract=off", "-std=c++17", "-fopenmp", "-shared", "-fPIC"]

INT32, FLOAT32 = 1, 2
SUM, COUNT, MIN, MAX, AVG = 0, 1, 2, 3, 4
GEN_UNIFORM, GEN_AFFINE = 1, 2
RESULT_EMPTY = 1

RESULT_DTYPE = np.dtype([("i", "<i8"), ("d", "<f8"), ("flags", "<u4"), ("pad", "<u4")])


def build(force: bool = False) -> str:
    """Compile oracle.cpp -> liboracle-<host>.so (g++ CFLAGS, OpenMP)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        cmd = ["g++", *CFLAGS, _SRC, "-o", _LIB + ".tmp"]
        subprocess.check_call(cmd)
        os.replace(_LIB + ".tmp", _LIB)
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        L = ctypes.CDLL(build())
        c_i64p = ctypes.POINTER(ctypes.c_int64)
        L.oracle_splitmix64.restype = ctypes.c_uint64
        L.oracle_splitmix64.argtypes = [ctypes.c_uint64, ctypes.c_uint64]
        L.oracle_fill.restype = ctypes.c_int
        L.oracle_fill.argtypes = [ctypes.c_int, c_i64p, ctypes.c_int, ctypes.c_int, ctypes.c_uint64,
                                  ctypes.c_void_p, ctypes.c_int64, ctypes.c_int64, ctypes.c_void_p]
        L.oracle_query.restype = ctypes.c_int
        L.oracle_query.argtypes = [ctypes.c_int, c_i64p, ctypes.c_int, ctypes.c_void_p,
                                   ctypes.c_int, ctypes.c_uint64, ctypes.c_void_p,
                                   ctypes.c_int64, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p,
                                   ctypes.c_int, c_i64p]
        L.oracle_max_threads.restype = ctypes.c_int
        L.oracle_dict_build.restype = ctypes.c_void_p
        L.oracle_dict_build.argtypes = [ctypes.c_char_p, c_i64p, ctypes.c_int64]
        L.oracle_dict_size.restype = ctypes.c_int64
        L.oracle_dict_size.argtypes = [ctypes.c_void_p]
        L.oracle_dict_translate.restype = ctypes.c_int64
        L.oracle_dict_translate.argtypes = [ctypes.c_void_p, ctypes.c_char_p, c_i64p, ctypes.c_int64,
                                            ctypes.c_void_p]
        L.oracle_dict_bound.restype = ctypes.c_int64
        L.oracle_dict_bound.argtypes = [ctypes.c_void_p, ctypes.c_char_p, ctypes.c_int64, ctypes.c_int]
        L.oracle_dict_lookup.restype = ctypes.c_int
        L.oracle_dict_lookup.argtypes = [ctypes.c_void_p, ctypes.c_int32,
                                         ctypes.POINTER(ctypes.c_char_p), c_i64p]
        L.oracle_dict_destroy.restype = None
        L.oracle_dict_destroy.argtypes = [ctypes.c_void_p]
        L.oracle_factscan.restype = ctypes.c_int
        L.oracle_factscan.argtypes = [ctypes.c_int64, ctypes.c_int, ctypes.c_void_p, ctypes.c_int,
                                      ctypes.c_void_p, ctypes.c_int64, ctypes.c_void_p,
                                      ctypes.c_void_p, ctypes.c_void_p]
        L.oracle_factbuild.restype = ctypes.c_int
        L.oracle_factbuild.argtypes = [ctypes.c_int, c_i64p, ctypes.c_int, ctypes.c_int64, ctypes.c_void_p,
                                       ctypes.c_void_p, ctypes.c_void_p]
        L.oracle_tablescan.restype = ctypes.c_int
        L.oracle_tablescan.argtypes = [ctypes.c_int64, ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int64,
                                       ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p,
                                       ctypes.c_void_p, ctypes.c_int]
        L.oracle_rollup.restype = ctypes.c_int
        L.oracle_rollup.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int,
                                    ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int, ctypes.c_void_p,
                                    ctypes.c_void_p, ctypes.c_int]
        L.oracle_convert_range.restype = ctypes.c_int
        L.oracle_convert_range.argtypes = [ctypes.c_int, ctypes.c_int64, ctypes.c_void_p, ctypes.c_int, ctypes.c_int,
                                           ctypes.c_int64, ctypes.c_int64, c_i64p, c_i64p]
        _lib = L
    return _lib


def _i64(a):
    a = np.ascontiguousarray(a, dtype=np.int64)
    return a, a.ctypes.data_as(ctypes.POINTER(ctypes.c_int64))


def _dtype_code(dt) -> int:
    dt = np.dtype(dt)
    if dt == np.int32:
        return INT32
    if dt == np.float32:
        return FLOAT32
    raise ValueError(f"unsupported cube dtype {dt}")


def splitmix64(seed: int, idx: int) -> int:
    return int(lib().oracle_splitmix64(seed, idx))


def fill(extents, dtype, gen: int, seed: int = 0, params=None, first: int = 0, count: int | None = None):
    """Cells [first, first+count) of a procedural cube, row-major."""
    ext, ext_p = _i64(extents)
    n = int(np.prod(ext)) if count is None else int(count)
    out = np.empty(n, dtype=np.dtype(dtype))
    par = np.ascontiguousarray(params if params is not None else np.zeros(len(ext) + 1), dtype=np.float64)
    rc = lib().oracle_fill(len(ext), ext_p, _dtype_code(dtype), gen, seed, par.ctypes.data,
                           first, n, out.ctypes.data)
    if rc:
        raise ValueError("oracle_fill failed")
    return out


def query(extents, ranges, ops, cells=None, *, dtype=None, gen: int = 0, seed: int = 0,
          params=None, nthreads: int = 1):
    """Answer queries on a host cube (cells: ndarray, row-major) or a procedural one.

    ranges: int64 array (nq, nd, 2) of inclusive [lo, hi]; ops: int32 (nq,).
    Returns a structured array with fields i, d, flags (RESULT_DTYPE).
    """
    ext, ext_p = _i64(extents)
    nd = len(ext)
    rng = np.ascontiguousarray(ranges, dtype=np.int64).reshape(-1, nd, 2)
    nq = rng.shape[0]
    opa = np.ascontiguousarray(ops, dtype=np.int32).reshape(nq)
    out = np.zeros(nq, dtype=RESULT_DTYPE)
    if cells is not None:
        cells = np.ascontiguousarray(cells)
        dt = _dtype_code(cells.dtype)
        if cells.size != int(np.prod(ext)):
            raise ValueError("cells size does not match extents")
        cptr = cells.ctypes.data
    else:
        dt = _dtype_code(dtype)
        cptr = None
    par = np.ascontiguousarray(params if params is not None else np.zeros(nd + 1), dtype=np.float64)
    bad = ctypes.c_int64(-1)
    rc = lib().oracle_query(nd, ext_p, dt, cptr, gen, seed, par.ctypes.data, nq, rng.ctypes.data,
                            opa.ctypes.data, out.ctypes.data, nthreads, ctypes.byref(bad))
    if rc == -2:
        raise IndexError(f"query {bad.value} out of bounds")
    if rc:
        raise ValueError("oracle_query: invalid arguments")
    return out


def max_threads() -> int:
    return int(lib().oracle_max_threads())


def _pack(keys):
    keys = [k.encode() if isinstance(k, str) else bytes(k) for k in keys]
    offs = np.zeros(len(keys) + 1, dtype=np.int64)
    if keys:
        offs[1:] = np.cumsum([len(k) for k in keys])
    return b"".join(keys), offs


class Dict:
    """std::map text-to-integer dictionary of one text column."""

    def __init__(self, keys):
        blob, offs = _pack(keys)
        self._h = lib().oracle_dict_build(blob, offs.ctypes.data_as(ctypes.POINTER(ctypes.c_int64)),
                                          len(offs) - 1)

    def __len__(self):
        return int(lib().oracle_dict_size(self._h))

    def translate(self, keys):
        blob, offs = _pack(keys)
        ids = np.empty(len(offs) - 1, dtype=np.int32)
        lib().oracle_dict_translate(self._h, blob, offs.ctypes.data_as(ctypes.POINTER(ctypes.c_int64)),
                                    len(ids), ids.ctypes.data)
        return ids

    def bound(self, key, upper: bool = False) -> int:
        k = key.encode() if isinstance(key, str) else bytes(key)
        return int(lib().oracle_dict_bound(self._h, k, len(k), 1 if upper else 0))

    def lookup(self, i: int) -> bytes:
        p = ctypes.c_char_p()
        n = ctypes.c_int64()
        if lib().oracle_dict_lookup(self._h, i, ctypes.byref(p), ctypes.byref(n)):
            raise KeyError(i)
        return ctypes.string_at(p, n.value)

    def close(self):
        if self._h:
            lib().oracle_dict_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def factbuild(extents, ids, values=None, cells=None, dtype=None):
    """The cube built from fact rows (oracle_factbuild): ids (nd, nrows) int32,
    values (nrows,) of the cube's dtype or None (+1 per row), added into `cells` (a copy of
    the row-major host cube; zeros of `dtype` when None).  Returns the new cells."""
    ext, ext_p = _i64(extents)
    ids = np.ascontiguousarray(ids, dtype=np.int32)
    nd, nrows = ids.shape
    dt = np.dtype(dtype if dtype is not None else (values.dtype if values is not None else cells.dtype))
    out = np.zeros(int(np.prod(ext)), dt) if cells is None else np.array(cells, dtype=dt).reshape(-1).copy()
    v = None if values is None else np.ascontiguousarray(values, dtype=dt)
    lib().oracle_factbuild(nd, ext_p, _dtype_code(dt), nrows, ids.ctypes.data, None if v is None else v.ctypes.data,
                           out.ctypes.data)
    return out


def factscan(dims, data, ranges):
    """SUM and fact COUNT over rows of dims (nd, nrows) int32 whose values lie in ranges (nq, nd, 2)."""
    dims = np.ascontiguousarray(dims, dtype=np.int32)
    nd, nrows = dims.shape
    data = np.ascontiguousarray(data)
    rng = np.ascontiguousarray(ranges, dtype=np.int64).reshape(-1, nd, 2)
    nq = rng.shape[0]
    s = np.zeros(nq, dtype=np.int64)
    c = np.zeros(nq, dtype=np.int64)
    lib().oracle_factscan(nrows, nd, dims.ctypes.data, _dtype_code(data.dtype), data.ctypes.data, nq,
                          rng.ctypes.data, s.ctypes.data, c.ctypes.data)
    if data.dtype == np.float32:
        s = s.view(np.float64)
    return s, c


COND_DTYPE = np.dtype([("col", "<i4"), ("pad", "<i4"), ("lo", "<i8"), ("hi", "<i8")])


def tablescan(columns, queries, nthreads: int = 1):
    """Q_D (Eq. 11) over a column-store fact table.

    columns: list of 1-D int32 / float32 arrays (equal length).  queries: list of
    (conds, data_col, op) with conds a list of (col, lo, hi).  Returns RESULT_DTYPE array."""
    cols = [np.ascontiguousarray(c) for c in columns]
    nrows = len(cols[0])
    ptrs = (ctypes.c_void_p * len(cols))(*[c.ctypes.data for c in cols])
    dts = np.array([_dtype_code(c.dtype) for c in cols], dtype=np.int32)
    off = np.zeros(len(queries) + 1, dtype=np.int64)
    flat = []
    for i, (conds, _dc, _op) in enumerate(queries):
        flat += list(conds)
        off[i + 1] = len(flat)
    ca = np.zeros(max(len(flat), 1), dtype=COND_DTYPE)
    for k, (c, lo, hi) in enumerate(flat):
        ca[k] = (c, 0, lo, hi)
    dcol = np.array([q[1] for q in queries], dtype=np.int32)
    ops = np.array([q[2] for q in queries], dtype=np.int32)
    out = np.zeros(len(queries), dtype=RESULT_DTYPE)
    rc = lib().oracle_tablescan(nrows, len(cols), ctypes.cast(ptrs, ctypes.c_void_p), dts.ctypes.data, len(queries),
                                off.ctypes.data, ca.ctypes.data, dcol.ctypes.data, ops.ctypes.data, out.ctypes.data,
                                nthreads)
    if rc:
        raise ValueError("oracle_tablescan: invalid arguments")
    return out


def _levels_ptrs(level_ids):
    """level_ids: list over dims of lists over levels of int32 arrays (finest-member -> level id)."""
    arrs = [np.ascontiguousarray(a, dtype=np.int32) for dim in level_ids for a in dim]
    ptrs = (ctypes.c_void_p * len(arrs))(*[a.ctypes.data for a in arrs])
    return arrs, ptrs


def rollup(level_ids, fine, rf, rc, op=SUM):
    """Aggregate the level-rf cube `fine` (ndarray, shape = level-rf extents) to level rc."""
    nd, L = len(level_ids), len(level_ids[0])
    n_fin = np.array([len(level_ids[d][-1]) for d in range(nd)], dtype=np.int64)
    arrs, ptrs = _levels_ptrs(level_ids)
    ext_f = np.array(fine.shape, dtype=np.int64)
    ext_c = np.array([int(level_ids[d][rc].max()) + 1 for d in range(nd)], dtype=np.int64)
    f = np.ascontiguousarray(fine)
    out = np.empty(tuple(ext_c), dtype=f.dtype)
    rc_ = lib().oracle_rollup(nd, L, n_fin.ctypes.data, ctypes.cast(ptrs, ctypes.c_void_p), _dtype_code(f.dtype), rf,
                              ext_f.ctypes.data, f.ctypes.data, rc, ext_c.ctypes.data, out.ctypes.data, op)
    if rc_:
        raise ValueError("oracle_rollup failed")
    return out


def convert_range(ids_of_dim, r, R, f, t):
    """[f, t] at level r -> [lo, hi] at level R (lo > hi if empty)."""
    arrs = [np.ascontiguousarray(a, dtype=np.int32) for a in ids_of_dim]
    ptrs = (ctypes.c_void_p * len(arrs))(*[a.ctypes.data for a in arrs])
    lo, hi = ctypes.c_int64(), ctypes.c_int64()
    lib().oracle_convert_range(len(arrs), len(arrs[-1]), ctypes.cast(ptrs, ctypes.c_void_p), r, R, f, t,
                               ctypes.byref(lo), ctypes.byref(hi))
    return lo.value, hi.value
