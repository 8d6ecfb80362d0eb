"""paper_conf_ipps_malikrse12_b200 — B200-native OLAP sub-cube query hot path.

Thin ctypes binding over ``libolap_b200.so`` whose C-ABI is ``include/olap.h``
(Malik, Riha, Shea, El-Ghazawi, IPDPSW 2012; Eq. 1, Eq. 3, §III-F).
This module only marshals arguments: every step of the path (planning,
range-reduce, combine, finalize, dictionary translation) runs in the library's
CUDA kernels.  There is no CPU fallback: if the library is missing, importing
this package raises; if no GPU is usable, the compute calls raise OlapError.

torch is used only for device memory and streams (tensors are passed by
``data_ptr()``; streams by ``torch.cuda.Stream.cuda_stream``).
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

__all__ = ["Cube", "Dict", "OlapError", "translate", "shard_local_rows", "combine_partials_device",
           "finalize_device", "translate_device", "RESULT_DTYPE", "lib", "LIB_PATH",
           "INT32", "FLOAT32", "SUM", "COUNT", "MIN", "MAX", "AVG", "GEN_UNIFORM", "GEN_AFFINE",
           "RESULT_EMPTY", "RESULT_INVALID", "EXPORTS", "text_ranges", "text_ranges_device", "pack_text_conditions", "text_ranges_packed",
           "COND_ALL", "COND_EQ", "COND_RANGE", "COND_IDS", "Table", "COND_DTYPE", "Hierarchy", "CubeSet",
           "TablePart", "Scheduler", "PART_CUBE", "PART_TABLE", "SCHED_PART_DTYPE", "SCHED_QUERY_DTYPE",
           "SCHED_DECISION_DTYPE", "perf_fn", "Comm", "comm_unique_id", "nccl_version", "exchange_partials_device",
           "E_NCCL"]

LIB_PATH = os.path.join(os.path.dirname(os.path.abspath(__file__)), "libolap_b200.so")
if os.environ.get("OLAP_LIB"):          # development only: A/B a differently-tuned build of the same sources
    LIB_PATH = os.path.abspath(os.environ["OLAP_LIB"])

INT32, FLOAT32 = 1, 2
SUM, COUNT, MIN, MAX, AVG = 0, 1, 2, 3, 4
LAYOUT_ROWMAJOR, LAYOUT_BRICK, LAYOUT_BRICK3 = 0, 1, 2  # olap.h OLAP_LAYOUT_*
GEN_UNIFORM, GEN_AFFINE = 1, 2
RESULT_EMPTY, RESULT_INVALID = 1, 2
COND_ALL, COND_EQ, COND_RANGE, COND_IDS = 0, 1, 2, 3

OK, E_INVALID, E_RANGE, E_NOMEM, E_CUDA, E_NCCL, E_STATE, E_UNSUPPORTED = 0, -1, -2, -3, -4, -5, -6, -7

PART_CUBE, PART_TABLE = 0, 1

# olap_sched_partition / olap_sched_query / olap_sched_decision (include/olap.h, dispatcher)
_PERF = [("x_split", "<f8"), ("a1", "<f8"), ("p1", "<f8"), ("b1", "<f8"), ("a2", "<f8"), ("p2", "<f8"), ("b2", "<f8")]
SCHED_PART_DTYPE = np.dtype([("kind", "<i4"), ("needs_translation", "<i4")] + _PERF)
SCHED_QUERY_DTYPE = np.dtype([("t_arrival", "<f8"), ("cube_mb", "<f8"), ("col_frac", "<f8"), ("t_trans", "<f8")])
SCHED_DECISION_DTYPE = np.dtype([("partition", "<i4"), ("translated", "<i4"), ("t_response", "<f8"),
                                 ("t_deadline", "<f8"), ("t_est", "<f8")])

# olap_result: {int64 i; double d; uint32 flags; uint32 _pad}
RESULT_DTYPE = np.dtype([("i", "<i8"), ("d", "<f8"), ("flags", "<u4"), ("pad", "<u4")])

_p = ctypes.c_void_p
_i64 = ctypes.c_int64
_i64p = ctypes.POINTER(ctypes.c_int64)
_int = ctypes.c_int

# every function declared in include/olap.h: name -> (restype, argtypes)
EXPORTS = {
    "olap_cube_create": (_int, [_int, _i64p, _int, _p, _int, ctypes.POINTER(_p)]),
    "olap_cube_create_layout": (_int, [_int, _i64p, _int, _p, _int, _int, ctypes.POINTER(_p)]),
    "olap_cube_info": (_int, [_p, _i64p, _i64p, ctypes.POINTER(_p)]),
    "olap_cube_load": (_int, [_p, _p, _i64]),
    "olap_cube_load_rows": (_int, [_p, _i64, _i64, _p]),
    "olap_cube_fill": (_int, [_p, _int, ctypes.c_uint64, _p]),
    "olap_cube_destroy": (_int, [_p]),
    "olap_query_batch": (_int, [_p, _i64, _p, _p, _p]),
    "olap_query_batch_device": (_int, [_p, _i64, _p, _p, _p, _p]),
    "olap_query_partials_device": (_int, [_p, _i64, _p, _p, _p, _p, _p]),
    "olap_partials_combine_device": (_int, [_int, _i64, _p, _p, _p, _p, _p]),
    "olap_finalize_device": (_int, [_int, _i64p, _int, _i64, _p, _p, _p, _p, _p, _p]),
    "olap_shard_local_rows": (_int, [_i64, _p, _i64, _i64, _i64p, _i64p]),
    "olap_cube_profile": (_int, [_p, _int]),
    "olap_cube_profile_read": (_int, [_p, ctypes.POINTER(ctypes.c_double), _i64p, _i64p]),
    "olap_dict_build": (_int, [_p, _i64p, _i64, _int, ctypes.POINTER(_p)]),
    "olap_dict_size": (_int, [_p, _i64p]),
    "olap_dict_translate": (_int, [_p, _int, _p, _p, _i64p, _i64, _p, _i64p]),
    "olap_dict_translate_device": (_int, [_p, _int, _p, _p, _p, _i64, _p, _p, _p]),
    "olap_dict_bound": (_int, [_p, _p, _i64p, _i64, _int, _p]),
    "olap_dict_lookup": (_int, [_p, ctypes.c_int32, ctypes.POINTER(ctypes.c_char_p), _i64p]),
    "olap_text_ranges": (_int, [_p, _int, _i64p, _i64, _p, _p, _p, _i64p, _i64, _p, _i64p]),
    "olap_text_ranges_device": (_int, [_p, _int, _i64p, _i64, _p, _p, _p, _p, _p, _i64, _p, _p, _p]),
    "olap_cube_add_facts_device": (_int, [_p, _i64, _p, _p, _p]),
    "olap_dict_destroy": (_int, [_p]),
    "olap_cube_stats": (_int, [_p, _i64p, ctypes.POINTER(_int)]),
    "olap_table_create": (_int, [_i64, _int, _p, _int, ctypes.POINTER(_p)]),
    "olap_table_load_column": (_int, [_p, _int, _p]),
    "olap_table_column_device": (_int, [_p, _int, ctypes.POINTER(_p)]),
    "olap_table_query_batch": (_int, [_p, _i64, _p, _p, _p, _p, _p]),
    "olap_table_query_batch_device": (_int, [_p, _i64, _p, _p, _p, _p, _p, _p]),
    "olap_table_destroy": (_int, [_p]),
    "olap_table_profile": (_int, [_p, _int]),
    "olap_table_profile_read": (_int, [_p, ctypes.POINTER(ctypes.c_double), _i64p]),
    "olap_table_part_create": (_int, [_p, _int, ctypes.POINTER(_p)]),
    "olap_table_part_sms": (_int, [_p, ctypes.POINTER(_int), ctypes.POINTER(_int)]),
    "olap_table_part_query_device": (_int, [_p, _i64, _p, _p, _p, _p, _p, _p]),
    "olap_table_part_query_boxes_device": (_int, [_p, _i64, _int, _p, _p, _p, _p, _p, _p, _p]),
    "olap_table_part_destroy": (_int, [_p]),
    "olap_sched_create": (_int, [_int, _p, ctypes.c_double, ctypes.POINTER(_p)]),
    "olap_sched_submit": (_int, [_p, _i64, _p, _p]),
    "olap_sched_complete": (_int, [_p, _int, ctypes.c_double, ctypes.c_double]),
    "olap_sched_queues": (_int, [_p, _p]),
    "olap_sched_destroy": (_int, [_p]),
    "olap_hier_create": (_int, [_int, _int, _p, _p, ctypes.POINTER(_p)]),
    "olap_hier_extents": (_int, [_p, _int, _p]),
    "olap_hier_convert": (_int, [_p, _i64, _p, _p, _int, _p]),
    "olap_cube_rollup": (_int, [_p, _p, _int, _p, _int, _int]),
    "olap_hier_destroy": (_int, [_p]),
    "olap_cubeset_create": (_int, [_p, ctypes.POINTER(_p)]),
    "olap_cubeset_add": (_int, [_p, _int, _p]),
    "olap_cubeset_query": (_int, [_p, _i64, _p, _p, _p, _p, _p]),
    "olap_cubeset_destroy": (_int, [_p]),
    "olap_finalize_launches": (_i64, []),
    "olap_cube_tile_stats": (_int, [_p, ctypes.POINTER(_int), ctypes.POINTER(_i64), ctypes.POINTER(_i64),
                                    ctypes.POINTER(_int)]),
    "olap_cube_create_multi": (_int, [_int, _i64p, _int, _p, ctypes.POINTER(_p)]),
    "olap_comm_unique_id": (_int, [_p]),
    "olap_comm_init_rank": (_int, [_p, _int, _int, _int, ctypes.POINTER(_p)]),
    "olap_comm_info": (_int, [_p, ctypes.POINTER(_int), ctypes.POINTER(_int), ctypes.POINTER(_int)]),
    "olap_comm_check": (_int, [_p]),
    "olap_comm_destroy": (_int, [_p]),
    "olap_cube_attach_comm": (_int, [_p, _p]),
    "olap_exchange_partials_device": (_int, [_p, _int, _i64, _p, _p, _p]),
    "olap_nccl_version": (_int, [ctypes.POINTER(_int)]),
    "olap_query_stream": (_int, [_p, _i64, _p, _p, _p, _i64]),
    "olap_last_error": (ctypes.c_char_p, []),
    "olap_version": (ctypes.c_char_p, []),
}


def _load():
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is missing: build it with `python -m paper_conf_ipps_malikrse12_b200.build` "
                          "(there is no CPU fallback)")
    L = ctypes.CDLL(LIB_PATH)
    for name, (res, args) in EXPORTS.items():
        f = getattr(L, name)
        f.restype = res
        f.argtypes = args
    L.olap_selftest_fastdiv.restype = _int
    L.olap_selftest_fastdiv.argtypes = [ctypes.c_uint32, _p, _i64, _p]
    L.olap_selftest_hash.restype = ctypes.c_uint64
    L.olap_selftest_hash.argtypes = [ctypes.c_char_p, _i64]
    return L


lib = _load()


class OlapError(RuntimeError):
    def __init__(self, status: int, where: str):
        self.status = status
        msg = lib.olap_last_error().decode(errors="replace")
        super().__init__(f"{where}: status {status}: {msg}")


def _check(rc: int, where: str):
    if rc != OK:
        raise OlapError(rc, where)


def _ptr(x):
    """device or host address of a torch tensor / numpy array / int / None"""
    if x is None:
        return None
    if isinstance(x, int):
        return x
    if isinstance(x, np.ndarray):
        return x.ctypes.data
    return x.data_ptr()


def _stream(stream):
    if stream is None:
        import torch
        return torch.cuda.current_stream().cuda_stream
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream


def _dtype_code(dtype) -> int:
    if isinstance(dtype, int):
        return dtype
    if isinstance(dtype, (type, np.dtype)):
        dt = np.dtype(dtype)
    else:
        dt = np.dtype(str(dtype).replace("torch.", ""))
    if dt == np.int32:
        return INT32
    if dt == np.float32:
        return FLOAT32
    raise ValueError(f"unsupported cell dtype {dtype}")


class _Shard(ctypes.Structure):
    _fields_ = [("nshards", ctypes.c_int64), ("shard", ctypes.c_int64), ("block", ctypes.c_int64)]


def _shard(shard):
    if shard is None:
        return None
    G, g, b = shard
    return _Shard(G, g, b)


def _i64arr(a):
    a = np.ascontiguousarray(a, dtype=np.int64)
    return a, a.ctypes.data_as(_i64p)


class _CubeOpts(ctypes.Structure):
    _fields_ = [("ndevices", ctypes.c_int32), ("shards_per_device", ctypes.c_int32),
                ("devices", ctypes.POINTER(ctypes.c_int32)), ("shard_block", ctypes.c_int64),
                ("layout", ctypes.c_int32), ("pad", ctypes.c_int32)]


class Cube:
    """A dense cube (or one block-cyclic dim-0 shard of it) resident in one GPU's HBM.

    devices=[d0, d1, ...] (and/or shards_per_device > 1) makes a group handle
    (olap_cube_create_multi): the cube sharded over those GPUs of this process, answered
    through the library's NCCL exchange."""

    def __init__(self, extents, dtype, shard=None, device: int = 0, layout: int = LAYOUT_ROWMAJOR,
                 devices=None, shards_per_device: int = 1, shard_block: int = 1):
        self.extents = tuple(int(e) for e in extents)
        self.layout = int(layout)
        self.ndims = len(self.extents)
        self.dtype_code = _dtype_code(dtype)
        self.np_dtype = np.int32 if self.dtype_code == INT32 else np.float32
        self.shard = tuple(shard) if shard is not None else (1, 0, 1)
        self.device = device if devices is None else int(devices[0])
        self._comm = None
        ext, extp = _i64arr(self.extents)
        h = ctypes.c_void_p()
        if devices is not None or shards_per_device > 1:
            devs = np.ascontiguousarray(devices if devices is not None else [device], dtype=np.int32)
            o = _CubeOpts(len(devs), int(shards_per_device), devs.ctypes.data_as(ctypes.POINTER(ctypes.c_int32)),
                          int(shard_block), self.layout, 0)
            _check(lib.olap_cube_create_multi(self.ndims, extp, self.dtype_code, ctypes.byref(o), ctypes.byref(h)),
                   "olap_cube_create_multi")
            self.shard = (len(devs) * int(shards_per_device), 0, int(shard_block))
            self.devices = tuple(int(d) for d in devs)
        else:
            sh = _shard(shard)
            _check(lib.olap_cube_create_layout(self.ndims, extp, self.dtype_code, ctypes.byref(sh) if sh else None,
                                               device, self.layout, ctypes.byref(h)), "olap_cube_create_layout")
            self.devices = (int(device),)
        self._h = h

    @property
    def handle(self):
        return self._h

    def info(self):
        rows, cells, ptr = ctypes.c_int64(), ctypes.c_int64(), ctypes.c_void_p()
        _check(lib.olap_cube_info(self._h, ctypes.byref(rows), ctypes.byref(cells), ctypes.byref(ptr)),
               "olap_cube_info")
        return rows.value, cells.value, ptr.value

    def load(self, cells: np.ndarray):
        cells = np.ascontiguousarray(cells, dtype=self.np_dtype).reshape(-1)
        _check(lib.olap_cube_load(self._h, cells.ctypes.data, cells.size), "olap_cube_load")

    def load_rows(self, row_lo: int, row_hi: int, cells: np.ndarray):
        cells = np.ascontiguousarray(cells, dtype=self.np_dtype).reshape(-1)
        _check(lib.olap_cube_load_rows(self._h, row_lo, row_hi, cells.ctypes.data), "olap_cube_load_rows")

    def fill(self, generator: int = GEN_UNIFORM, seed: int = 0, params=None):
        par = None
        if params is not None:
            par = np.ascontiguousarray(params, dtype=np.float64)
        _check(lib.olap_cube_fill(self._h, generator, seed & 0xFFFFFFFFFFFFFFFF,
                                  par.ctypes.data if par is not None else None), "olap_cube_fill")

    def query(self, ranges, ops, out: np.ndarray | None = None) -> np.ndarray:
        """Host-buffer path (olap_query_batch): ranges (nq, ndims, 2) int64, ops (nq,) int32."""
        rng = np.ascontiguousarray(ranges, dtype=np.int64).reshape(-1, self.ndims, 2)
        nq = rng.shape[0]
        opa = np.ascontiguousarray(ops, dtype=np.int32).reshape(nq)
        res = out if out is not None else np.zeros(nq, dtype=RESULT_DTYPE)
        _check(lib.olap_query_batch(self._h, nq, rng.ctypes.data, opa.ctypes.data, res.ctypes.data),
               "olap_query_batch")
        return res

    def query_stream(self, ranges, ops, batch: int = 0, out: np.ndarray | None = None) -> np.ndarray:
        """olap_query_stream: a stream of queries answered in pipelined batches of `batch`."""
        rng = np.ascontiguousarray(ranges, dtype=np.int64).reshape(-1, self.ndims, 2)
        nq = rng.shape[0]
        opa = np.ascontiguousarray(ops, dtype=np.int32).reshape(nq)
        res = out if out is not None else np.zeros(nq, dtype=RESULT_DTYPE)
        _check(lib.olap_query_stream(self._h, nq, rng.ctypes.data, opa.ctypes.data, res.ctypes.data, int(batch)),
               "olap_query_stream")
        return res

    def attach_comm(self, comm: "Comm | None"):
        """olap_cube_attach_comm: this shard's batches become collectives over `comm` (None detaches)."""
        _check(lib.olap_cube_attach_comm(self._h, comm.handle if comm is not None else None), "olap_cube_attach_comm")
        self._comm = comm  # the cube borrows it

    def query_device(self, d_ranges, d_ops, d_results, nq: int | None = None, stream=None):
        nq = d_ops.numel() if nq is None else nq
        _check(lib.olap_query_batch_device(self._h, nq, _ptr(d_ranges), _ptr(d_ops), _ptr(d_results),
                                           _stream(stream)), "olap_query_batch_device")

    def partials_device(self, d_ranges, d_ops, d_sum, d_ext, nq: int | None = None, stream=None):
        nq = d_ops.numel() if nq is None else nq
        _check(lib.olap_query_partials_device(self._h, nq, _ptr(d_ranges), _ptr(d_ops), _ptr(d_sum), _ptr(d_ext),
                                              _stream(stream)), "olap_query_partials_device")

    def add_facts_device(self, d_ids, d_values=None, nrows: int | None = None, stream=None):
        """Scatter-add fact rows into their cells (d_ids: (ndims, nrows) int32 device tensor)."""
        nrows = d_ids.shape[-1] if nrows is None else nrows
        _check(lib.olap_cube_add_facts_device(self._h, nrows, _ptr(d_ids), _ptr(d_values), _stream(stream)),
               "olap_cube_add_facts_device")

    def profile(self, enable: bool = True):
        _check(lib.olap_cube_profile(self._h, 1 if enable else 0), "olap_cube_profile")

    def profile_read(self):
        ms, n, b = ctypes.c_double(), ctypes.c_int64(), ctypes.c_int64()
        _check(lib.olap_cube_profile_read(self._h, ctypes.byref(ms), ctypes.byref(n), ctypes.byref(b)),
               "olap_cube_profile_read")
        return ms.value, n.value, b.value

    def stats(self):
        """(kernel launches so far, L2-aware order active)"""
        n, o = ctypes.c_int64(), ctypes.c_int()
        _check(lib.olap_cube_stats(self._h, ctypes.byref(n), ctypes.byref(o)), "olap_cube_stats")
        return n.value, bool(o.value)

    def tile_stats(self):
        """(tile path enabled, cells per tile, tiles, last batch used it)"""
        en, tc, nt, lu = _int(), ctypes.c_int64(), ctypes.c_int64(), _int()
        _check(lib.olap_cube_tile_stats(self._h, ctypes.byref(en), ctypes.byref(tc), ctypes.byref(nt),
                                        ctypes.byref(lu)), "olap_cube_tile_stats")
        return bool(en.value), tc.value, nt.value, bool(lu.value)

    def close(self):
        if getattr(self, "_h", None):
            lib.olap_cube_destroy(self._h)
            self._h = None
        self._comm = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class Comm:
    """One rank of a NCCL communicator owned by the library (olap_comm_init_rank)."""

    def __init__(self, unique_id: bytes, nranks: int, rank: int, device: int = 0):
        if len(unique_id) != 128:
            raise ValueError("a communicator id is 128 bytes (olap_comm_unique_id)")
        buf = ctypes.create_string_buffer(bytes(unique_id), 128)
        h = ctypes.c_void_p()
        _check(lib.olap_comm_init_rank(buf, int(nranks), int(rank), int(device), ctypes.byref(h)),
               "olap_comm_init_rank")
        self._h = h
        self.nranks, self.rank, self.device = int(nranks), int(rank), int(device)

    @property
    def handle(self):
        return self._h

    def check(self):
        _check(lib.olap_comm_check(self._h), "olap_comm_check")

    def close(self):
        if getattr(self, "_h", None):
            lib.olap_comm_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def comm_unique_id() -> bytes:
    """olap_comm_unique_id: 128 bytes that rank 0 passes to every rank."""
    buf = ctypes.create_string_buffer(128)
    _check(lib.olap_comm_unique_id(buf), "olap_comm_unique_id")
    return buf.raw


def nccl_version() -> int:
    v = _int()
    _check(lib.olap_nccl_version(ctypes.byref(v)), "olap_nccl_version")
    return v.value


def exchange_partials_device(comm: Comm, dtype, nq: int, d_sum, d_ext, stream=None):
    """olap_exchange_partials_device: all-reduce partials in place over the library's communicator."""
    _check(lib.olap_exchange_partials_device(comm.handle, _dtype_code(dtype), nq, _ptr(d_sum), _ptr(d_ext),
                                             _stream(stream)), "olap_exchange_partials_device")


def combine_partials_device(dtype, nq: int, sum_in, ext_in, sum_acc, ext_acc, stream=None):
    _check(lib.olap_partials_combine_device(_dtype_code(dtype), nq, _ptr(sum_in), _ptr(ext_in), _ptr(sum_acc),
                                            _ptr(ext_acc), _stream(stream)), "olap_partials_combine_device")


def finalize_device(extents, dtype, nq: int, d_ranges, d_ops, d_sum, d_ext, d_results, stream=None):
    ext, extp = _i64arr(extents)
    _check(lib.olap_finalize_device(len(ext), extp, _dtype_code(dtype), nq, _ptr(d_ranges), _ptr(d_ops),
                                    _ptr(d_sum), _ptr(d_ext), _ptr(d_results), _stream(stream)),
           "olap_finalize_device")


def shard_local_rows(n0: int, shard, lo: int, hi: int):
    """(llo, lhi) local dim-0 range of global rows [lo, hi]; llo > lhi if the shard owns none."""
    a, b = ctypes.c_int64(), ctypes.c_int64()
    sh = _shard(shard)
    _check(lib.olap_shard_local_rows(n0, ctypes.byref(sh) if sh else None, lo, hi, ctypes.byref(a), ctypes.byref(b)),
           "olap_shard_local_rows")
    return a.value, b.value


def _pack(keys):
    keys = [k.encode() if isinstance(k, str) else bytes(k) for k in keys]
    offs = np.zeros(len(keys) + 1, dtype=np.int64)
    if keys:
        offs[1:] = np.cumsum([len(k) for k in keys])
    blob = b"".join(keys)
    buf = np.frombuffer(blob, dtype=np.uint8) if blob else np.zeros(1, np.uint8)
    return np.ascontiguousarray(buf), offs


class Dict:
    """One text column's dictionary, resident on a GPU."""

    def __init__(self, keys, device: int = 0):
        buf, offs = _pack(keys)
        h = ctypes.c_void_p()
        _check(lib.olap_dict_build(buf.ctypes.data, offs.ctypes.data_as(_i64p), len(offs) - 1, device,
                                   ctypes.byref(h)), "olap_dict_build")
        self._h = h
        self.device = device

    @property
    def handle(self):
        return self._h

    def __len__(self):
        n = ctypes.c_int64()
        _check(lib.olap_dict_size(self._h, ctypes.byref(n)), "olap_dict_size")
        return n.value

    def translate(self, keys):
        """(ids, n_missing) of keys in this dictionary; -1 = absent."""
        return translate([self], None, keys)

    def bound(self, keys, upper: bool = False) -> np.ndarray:
        buf, offs = _pack(keys)
        out = np.empty(len(offs) - 1, dtype=np.int32)
        _check(lib.olap_dict_bound(self._h, buf.ctypes.data, offs.ctypes.data_as(_i64p), len(out),
                                   1 if upper else 0, out.ctypes.data), "olap_dict_bound")
        return out

    def lookup(self, i: int) -> bytes:
        p, n = ctypes.c_char_p(), ctypes.c_int64()
        _check(lib.olap_dict_lookup(self._h, i, ctypes.byref(p), ctypes.byref(n)), "olap_dict_lookup")
        return ctypes.string_at(p, n.value)

    def close(self):
        if getattr(self, "_h", None):
            lib.olap_dict_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def _dict_array(dicts):
    arr = (ctypes.c_void_p * len(dicts))(*[d.handle.value for d in dicts])
    return arr


def translate(dicts, dict_of_key, keys):
    """ids[i] of key i in dicts[dict_of_key[i]] (-1 if absent) and the number of misses."""
    buf, offs = _pack(keys)
    n = len(offs) - 1
    ids = np.empty(n, dtype=np.int32)
    dk = None if dict_of_key is None else np.ascontiguousarray(dict_of_key, dtype=np.int32)
    miss = ctypes.c_int64()
    _check(lib.olap_dict_translate(_dict_array(dicts), len(dicts), dk.ctypes.data if dk is not None else None,
                                   buf.ctypes.data, offs.ctypes.data_as(_i64p), n, ids.ctypes.data,
                                   ctypes.byref(miss)), "olap_dict_translate")
    return ids, miss.value


def translate_device(dicts, d_dict_of_key, d_bytes, d_offsets, n: int, d_ids, d_n_missing=None, stream=None):
    _check(lib.olap_dict_translate_device(_dict_array(dicts), len(dicts), _ptr(d_dict_of_key), _ptr(d_bytes),
                                          _ptr(d_offsets), n, _ptr(d_ids), _ptr(d_n_missing), _stream(stream)),
           "olap_dict_translate_device")


def _dict_or_null_array(dicts):
    return (ctypes.c_void_p * len(dicts))(*[(d.handle.value if d is not None else None) for d in dicts])


def pack_text_conditions(conditions, nd: int):
    """Marshal per-(query, dimension) text conditions into the C-ABI arrays:
    kinds (nq*nd int32), first_key (nq*nd int64), ranges_in (nq, nd, 2), key blob, key offsets."""
    kinds = np.zeros(len(conditions) * nd, dtype=np.int32)
    first = np.zeros(len(conditions) * nd, dtype=np.int64)
    rin = np.zeros((len(conditions), nd, 2), dtype=np.int64)
    keys = []
    for qi, cond in enumerate(conditions):
        for d in range(nd):
            c = cond[d]
            i = qi * nd + d
            first[i] = len(keys)
            if c is None:
                kinds[i] = COND_ALL
            elif isinstance(c, tuple) and len(c) == 3 and c[0] == "ids":
                kinds[i] = COND_IDS
                rin[qi, d] = (c[1], c[2])
            elif isinstance(c, tuple):
                kinds[i] = COND_RANGE
                keys += [c[0], c[1]]
            else:
                kinds[i] = COND_EQ
                keys.append(c)
    buf, offs = _pack(keys)
    return kinds, first, rin, buf, offs


def text_ranges_packed(dicts, extents, nq: int, kinds, rin, buf, offs):
    """olap_text_ranges on conditions already in the C-ABI layout (see pack_text_conditions)."""
    ext, extp = _i64arr(extents)
    out = np.zeros((nq, len(dicts), 2), dtype=np.int64)
    miss = ctypes.c_int64()
    _check(lib.olap_text_ranges(_dict_or_null_array(dicts), len(dicts), extp, nq, kinds.ctypes.data, rin.ctypes.data,
                                buf.ctypes.data, offs.ctypes.data_as(_i64p), len(offs) - 1, out.ctypes.data,
                                ctypes.byref(miss)), "olap_text_ranges")
    return out, miss.value


def text_ranges(dicts, extents, conditions, ranges_in=None):
    """Text conditions -> ranges (olap_text_ranges).

    dicts: one Dict (or None) per dimension; conditions: nq lists of ndims entries, each
    None (whole dimension), a str/bytes key (equality), a (s1, s2) tuple (string range),
    or an int pair [lo, hi] given as ('ids', lo, hi).  Returns (ranges (nq, ndims, 2), n_missing)."""
    nd = len(dicts)
    k, _first, rin, buf, offs = pack_text_conditions(conditions, nd)
    ext, extp = _i64arr(extents)
    out = np.zeros((len(conditions), nd, 2), dtype=np.int64)
    miss = ctypes.c_int64()
    _check(lib.olap_text_ranges(_dict_or_null_array(dicts), nd, extp, len(conditions), k.ctypes.data, rin.ctypes.data,
                                buf.ctypes.data, offs.ctypes.data_as(_i64p), len(offs) - 1, out.ctypes.data,
                                ctypes.byref(miss)), "olap_text_ranges")
    return out, miss.value


def text_ranges_device(dicts, extents, nq: int, d_kinds, d_first_key, d_ranges_in, d_bytes, d_offsets, nkeys: int,
                       d_ranges_out, d_n_missing=None, stream=None):
    ext, extp = _i64arr(extents)
    _check(lib.olap_text_ranges_device(_dict_or_null_array(dicts), len(ext), extp, nq, _ptr(d_kinds),
                                       _ptr(d_first_key), _ptr(d_ranges_in), _ptr(d_bytes), _ptr(d_offsets), nkeys,
                                       _ptr(d_ranges_out), _ptr(d_n_missing), _stream(stream)),
           "olap_text_ranges_device")


# olap_cond: {int32 col; int32 _pad; int64 lo, hi}
COND_DTYPE = np.dtype([("col", "<i4"), ("pad", "<i4"), ("lo", "<i8"), ("hi", "<i8")])


def pack_table_queries(queries):
    """queries: list of (conds, data_col, op), conds a list of (col, lo, hi) ->
    (cond_offsets int64[nq+1], conds COND_DTYPE[], data_cols int32[nq], ops int32[nq])."""
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
    return off, ca, dcol, ops


class Table:
    """A column-store fact table in GPU memory (the paper's GPU data structure)."""

    def __init__(self, nrows: int, dtypes, device: int = 0):
        self.nrows = int(nrows)
        self.dtypes = [_dtype_code(d) for d in dtypes]
        dt = np.array(self.dtypes, dtype=np.int32)
        h = ctypes.c_void_p()
        _check(lib.olap_table_create(self.nrows, len(dt), dt.ctypes.data, device, ctypes.byref(h)),
               "olap_table_create")
        self._h = h
        self.device = device

    def load_column(self, col: int, values: np.ndarray):
        v = np.ascontiguousarray(values, dtype=np.int32 if self.dtypes[col] == INT32 else np.float32)
        if v.size != self.nrows:
            raise ValueError("column length != nrows")
        _check(lib.olap_table_load_column(self._h, col, v.ctypes.data), "olap_table_load_column")

    def column_device(self, col: int) -> int:
        p = ctypes.c_void_p()
        _check(lib.olap_table_column_device(self._h, col, ctypes.byref(p)), "olap_table_column_device")
        return p.value

    def query(self, queries) -> np.ndarray:
        off, ca, dcol, ops = pack_table_queries(queries)
        out = np.zeros(len(queries), dtype=RESULT_DTYPE)
        _check(lib.olap_table_query_batch(self._h, len(queries), off.ctypes.data, ca.ctypes.data, dcol.ctypes.data,
                                          ops.ctypes.data, out.ctypes.data), "olap_table_query_batch")
        return out

    def query_device(self, nq: int, d_off, d_conds, d_dcol, d_ops, d_results, stream=None):
        _check(lib.olap_table_query_batch_device(self._h, nq, _ptr(d_off), _ptr(d_conds), _ptr(d_dcol), _ptr(d_ops),
                                                 _ptr(d_results), _stream(stream)), "olap_table_query_batch_device")

    def profile(self, enable: bool = True):
        _check(lib.olap_table_profile(self._h, 1 if enable else 0), "olap_table_profile")

    def profile_read(self):
        ms, n = ctypes.c_double(), ctypes.c_int64()
        _check(lib.olap_table_profile_read(self._h, ctypes.byref(ms), ctypes.byref(n)), "olap_table_profile_read")
        return ms.value, n.value

    def close(self):
        if getattr(self, "_h", None):
            lib.olap_table_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class TablePart:
    """A GPU partition of `sm_count` SMs for fact-table queries (Fig. 7)."""

    def __init__(self, table: "Table", sm_count: int = 0):
        h = ctypes.c_void_p()
        _check(lib.olap_table_part_create(table._h, int(sm_count), ctypes.byref(h)), "olap_table_part_create")
        self._h = h
        self.table = table  # keeps the table alive
        sm, bl = _int(), _int()
        _check(lib.olap_table_part_sms(h, ctypes.byref(sm), ctypes.byref(bl)), "olap_table_part_sms")
        self.sm_count, self.blocks = sm.value, bl.value

    def query_device(self, nq: int, d_off, d_conds, d_dcol, d_ops, d_results, stream=None):
        _check(lib.olap_table_part_query_device(self._h, nq, _ptr(d_off), _ptr(d_conds), _ptr(d_dcol), _ptr(d_ops),
                                                _ptr(d_results), _stream(stream)), "olap_table_part_query_device")

    def query_boxes_device(self, nq: int, dim_cols, extents, d_boxes, d_dcol, d_ops, d_results, stream=None):
        dc = np.ascontiguousarray(dim_cols, dtype=np.int32)
        ex = np.ascontiguousarray(extents, dtype=np.int64)
        _check(lib.olap_table_part_query_boxes_device(self._h, nq, len(dc), dc.ctypes.data, ex.ctypes.data,
                                                      _ptr(d_boxes), _ptr(d_dcol), _ptr(d_ops), _ptr(d_results),
                                                      _stream(stream)), "olap_table_part_query_boxes_device")

    def close(self):
        if getattr(self, "_h", None):
            lib.olap_table_part_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def perf_fn(a1, p1=1.0, b1=0.0, x_split=float("inf"), a2=0.0, p2=1.0, b2=0.0):
    """Eq. 4 performance function: a1*x^p1 + b1 below x_split, a2*x^p2 + b2 from it on."""
    return (x_split, a1, p1, b1, a2, p2, b2)


class Scheduler:
    """Fig. 10's dispatcher in the library (host code).

    partitions: [(kind PART_CUBE / PART_TABLE, needs_translation, perf_fn(...))] in FOR-loop
    order (slow -> fast); t_c: T_C in seconds."""

    def __init__(self, partitions, t_c: float):
        arr = np.zeros(len(partitions), dtype=SCHED_PART_DTYPE)
        for i, (kind, needs, fn) in enumerate(partitions):
            arr[i]["kind"], arr[i]["needs_translation"] = kind, int(bool(needs))
            for k, v in zip(("x_split", "a1", "p1", "b1", "a2", "p2", "b2"), fn):
                arr[i][k] = v
        h = ctypes.c_void_p()
        _check(lib.olap_sched_create(len(arr), arr.ctypes.data, float(t_c), ctypes.byref(h)), "olap_sched_create")
        self._h = h
        self.nparts = len(arr)

    def submit(self, queries) -> np.ndarray:
        """queries: SCHED_QUERY_DTYPE array or [(t_arrival, cube_mb, col_frac, t_trans)]."""
        q = queries if isinstance(queries, np.ndarray) and queries.dtype == SCHED_QUERY_DTYPE else \
            np.array([tuple(map(float, x)) for x in queries], dtype=SCHED_QUERY_DTYPE)
        q = np.ascontiguousarray(q)
        out = np.zeros(len(q), dtype=SCHED_DECISION_DTYPE)
        _check(lib.olap_sched_submit(self._h, len(q), q.ctypes.data, out.ctypes.data), "olap_sched_submit")
        return out

    def complete(self, partition: int, t_est: float, t_real: float):
        _check(lib.olap_sched_complete(self._h, int(partition), float(t_est), float(t_real)), "olap_sched_complete")

    def queues(self):
        out = np.zeros(self.nparts + 1, dtype=np.float64)
        _check(lib.olap_sched_queues(self._h, out.ctypes.data), "olap_sched_queues")
        return out

    def close(self):
        if getattr(self, "_h", None):
            lib.olap_sched_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class Hierarchy:
    """Resolution levels per dimension (Fig. 1).

    level_ids: list over dimensions of lists over levels (coarsest first) of int32 arrays
    mapping each finest member to its level-r member."""

    def __init__(self, level_ids):
        self.nd, self.L = len(level_ids), len(level_ids[0])
        self._arrs = [np.ascontiguousarray(a, dtype=np.int32) for dim in level_ids for a in dim]
        ptrs = (ctypes.c_void_p * len(self._arrs))(*[a.ctypes.data for a in self._arrs])
        nf = np.array([len(level_ids[d][-1]) for d in range(self.nd)], dtype=np.int64)
        h = ctypes.c_void_p()
        _check(lib.olap_hier_create(self.nd, self.L, nf.ctypes.data, ctypes.cast(ptrs, ctypes.c_void_p),
                                    ctypes.byref(h)), "olap_hier_create")
        self._h = h

    @property
    def handle(self):
        return self._h

    def extents(self, level: int):
        e = np.zeros(self.nd, dtype=np.int64)
        _check(lib.olap_hier_extents(self._h, level, e.ctypes.data), "olap_hier_extents")
        return tuple(int(v) for v in e)

    def convert(self, ranges, levels, target: int):
        r = np.ascontiguousarray(ranges, dtype=np.int64).reshape(-1, self.nd, 2)
        lv = np.ascontiguousarray(levels, dtype=np.int32).reshape(-1, self.nd)
        out = np.zeros_like(r)
        _check(lib.olap_hier_convert(self._h, r.shape[0], r.ctypes.data, lv.ctypes.data, target, out.ctypes.data),
               "olap_hier_convert")
        return out

    def rollup(self, fine: "Cube", fine_level: int, coarse: "Cube", coarse_level: int, op: int = SUM):
        _check(lib.olap_cube_rollup(self._h, fine.handle, fine_level, coarse.handle, coarse_level, op),
               "olap_cube_rollup")

    def close(self):
        if getattr(self, "_h", None):
            lib.olap_hier_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class CubeSet:
    """Cubes at several resolutions; queries routed by Eq. 2."""

    def __init__(self, hier: Hierarchy):
        self.hier = hier
        self._cubes = {}
        h = ctypes.c_void_p()
        _check(lib.olap_cubeset_create(hier.handle, ctypes.byref(h)), "olap_cubeset_create")
        self._h = h

    def add(self, level: int, cube: "Cube"):
        _check(lib.olap_cubeset_add(self._h, level, cube.handle), "olap_cubeset_add")
        self._cubes[level] = cube   # keep alive (the set borrows it)

    def query(self, ranges, levels, ops):
        r = np.ascontiguousarray(ranges, dtype=np.int64).reshape(-1, self.hier.nd, 2)
        lv = np.ascontiguousarray(levels, dtype=np.int32).reshape(-1, self.hier.nd)
        o = np.ascontiguousarray(ops, dtype=np.int32).reshape(-1)
        out = np.zeros(len(o), dtype=RESULT_DTYPE)
        used = np.zeros(len(o), dtype=np.int32)
        _check(lib.olap_cubeset_query(self._h, len(o), r.ctypes.data, lv.ctypes.data, o.ctypes.data, out.ctypes.data,
                                      used.ctypes.data), "olap_cubeset_query")
        return out, used

    def close(self):
        if getattr(self, "_h", None):
            lib.olap_cubeset_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
