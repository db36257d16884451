"""ctypes binding of libgpl.so (include/gpl.h) — argument marshalling only.

Every step of the hot path runs in the library's sm_100a kernels; this module
converts Python/numpy/torch arguments to C types and C results to Python ints.
There is no fallback: if the shared library is missing, importing
`Context` raises.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass, field

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "lib", "libgpl.so")

# status codes (gpl.h)
GPL_OK, GPL_E_ARG, GPL_E_CUDA, GPL_E_NOMEM, GPL_E_STATE, GPL_E_DUPKEY, GPL_E_CAPACITY, \
    GPL_E_OVERFLOW, GPL_E_DOMAIN, GPL_E_NODEV, GPL_E_PLAN = range(11)
STATUS_NAMES = {0: "GPL_OK", 1: "GPL_E_ARG", 2: "GPL_E_CUDA", 3: "GPL_E_NOMEM", 4: "GPL_E_STATE",
                5: "GPL_E_DUPKEY", 6: "GPL_E_CAPACITY", 7: "GPL_E_OVERFLOW", 8: "GPL_E_DOMAIN",
                9: "GPL_E_NODEV", 10: "GPL_E_PLAN"}
GPL_I32, GPL_I64, GPL_DATE32, GPL_DEC64, GPL_DICT32 = 1, 2, 3, 4, 5
GPL_COPY, GPL_BORROW = 0, 1

EXPORTED = ["gpl_create", "gpl_destroy", "gpl_load_columns", "gpl_build_hash", "gpl_run_plan",
            "gpl_run_plan_kbe", "gpl_fetch_result", "gpl_fetch_partials", "gpl_decode_partials",
            "gpl_merge_partials", "gpl_sync", "gpl_choose_tile_rows", "gpl_set_option",
            "gpl_check_plan", "gpl_compile_plan", "gpl_run_query", "gpl_autotune", "gpl_calibrate",
            "gpl_set_calibration", "gpl_fetch_groups", "gpl_merge_groups", "gpl_last_error", "gpl_version"]


class GplError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{STATUS_NAMES.get(status, status)}: {msg}")
        self.status = status
        self.msg = msg


class _Column(ctypes.Structure):
    _fields_ = [("name", ctypes.c_char_p), ("type", ctypes.c_int32), ("scale", ctypes.c_int32),
                ("data", ctypes.c_void_p), ("on_device", ctypes.c_int32), ("reserved", ctypes.c_int32),
                ("capacity_rows", ctypes.c_int64)]


class _Stats(ctypes.Structure):
    _fields_ = [("rows_scanned", ctypes.c_int64), ("tile_rows_used", ctypes.c_int64),
                ("stage_rows", ctypes.c_int32), ("ring_depth", ctypes.c_int32),
                ("consumer_warps", ctypes.c_int32), ("grid", ctypes.c_int32), ("n_ops", ctypes.c_int32),
                ("probe_split", ctypes.c_int32), ("op_pass", ctypes.c_int64 * 16),
                ("kernel_ms", ctypes.c_double), ("predicted_ms", ctypes.c_double),
                ("bytes_scanned", ctypes.c_double), ("agg_mode", ctypes.c_int32), ("kbe", ctypes.c_int32),
                ("jit", ctypes.c_int32), ("reserved", ctypes.c_int32), ("intermediate_bytes", ctypes.c_double),
                ("bytes_full_scan", ctypes.c_double), ("lazy_columns", ctypes.c_int32), ("packets", ctypes.c_int32),
                ("groups_total", ctypes.c_int64), ("hash_slots", ctypes.c_int64), ("drain_warps", ctypes.c_int32),
                ("launches", ctypes.c_int32)]


class _Result(ctypes.Structure):
    _fields_ = [("cap_groups", ctypes.c_int32), ("n_groups", ctypes.c_int32), ("n_keys", ctypes.c_int32),
                ("n_aggs", ctypes.c_int32), ("keys", ctypes.c_void_p), ("aggs", ctypes.c_void_p),
                ("stats", _Stats), ("n_ratios", ctypes.c_int32), ("reserved", ctypes.c_int32),
                ("ratios", ctypes.c_void_p)]


class _Model(ctypes.Structure):
    _fields_ = [("tile_rows", ctypes.c_int64), ("stage_rows", ctypes.c_int32), ("ring_depth", ctypes.c_int32),
                ("consumer_warps", ctypes.c_int32), ("grid", ctypes.c_int32), ("predicted_ms", ctypes.c_double),
                ("t_stream_ms", ctypes.c_double), ("t_probe_ms", ctypes.c_double), ("t_tail_ms", ctypes.c_double),
                ("t_launch_ms", ctypes.c_double), ("bw_gbs", ctypes.c_double), ("smem_bytes", ctypes.c_int32),
                ("feasible", ctypes.c_int32), ("ctas_per_sm", ctypes.c_int32), ("candidates", ctypes.c_int32),
                ("measured_ms", ctypes.c_double), ("probe_split", ctypes.c_int32), ("builds_tuned", ctypes.c_int32),
                ("build_ms_model", ctypes.c_double), ("build_ms", ctypes.c_double)]


class _Gamma(ctypes.Structure):  # gpl_gamma_point
    _fields_ = [("ring_depth", ctypes.c_int32), ("stage_rows", ctypes.c_int32), ("ctas_per_sm", ctypes.c_int32),
                ("consumer_warps", ctypes.c_int32), ("rows", ctypes.c_int64), ("bytes", ctypes.c_double),
                ("ms", ctypes.c_double), ("t0_ms", ctypes.c_double), ("gbs", ctypes.c_double)]


_lib = None


def load_library():
    """Load libgpl.so (raises if it was not built — there is no CPU fallback)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise RuntimeError(f"{LIB_PATH} is missing: build it with `make` (or __graft_entry__.build()); "
                           "the GPL hot path has no CPU fallback")
    lib = ctypes.CDLL(LIB_PATH)
    P, I32, I64, S = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64, ctypes.c_size_t
    sig = {
        "gpl_create": ([ctypes.c_int, P, ctypes.POINTER(P)], I32),
        "gpl_destroy": ([P], None),
        "gpl_load_columns": ([P, ctypes.c_char_p, I64, I32, ctypes.POINTER(_Column), ctypes.c_uint32], I32),
        "gpl_build_hash": ([P, ctypes.c_char_p, ctypes.POINTER(I32)], I32),
        "gpl_run_plan": ([P, ctypes.c_char_p, I64], I32),
        "gpl_run_plan_kbe": ([P, ctypes.c_char_p], I32),
        "gpl_fetch_result": ([P, ctypes.POINTER(_Result)], I32),
        "gpl_fetch_partials": ([P, P, I32, S, ctypes.POINTER(S)], I32),
        "gpl_decode_partials": ([P, P, S, ctypes.POINTER(_Result)], I32),
        "gpl_merge_partials": ([P, I32, S, P], I32),
        "gpl_sync": ([P], I32),
        "gpl_choose_tile_rows": ([P, ctypes.c_char_p, I64, ctypes.POINTER(_Model)], I32),
        "gpl_set_option": ([P, ctypes.c_char_p, I64], I32),
        "gpl_check_plan": ([P, ctypes.c_char_p], I32),
        "gpl_compile_plan": ([P, ctypes.c_char_p, I64], I32),
        "gpl_run_query": ([P, ctypes.c_char_p, I64], I32),
        "gpl_autotune": ([P, ctypes.c_char_p, I32, ctypes.POINTER(_Model)], I32),
        "gpl_calibrate": ([P, ctypes.POINTER(I64), I32, ctypes.POINTER(_Gamma), I32, ctypes.POINTER(I32)], I32),
        "gpl_set_calibration": ([P, ctypes.POINTER(_Gamma), I32], I32),
        "gpl_fetch_groups": ([P, ctypes.POINTER(I64), I64, ctypes.POINTER(I64), ctypes.POINTER(I32)], I32),
        "gpl_merge_groups": ([P, ctypes.c_char_p, ctypes.POINTER(I64), I64, ctypes.POINTER(_Result)], I32),
        "gpl_last_error": ([P], ctypes.c_char_p),
        "gpl_version": ([], ctypes.c_char_p),
    }
    for name, (args, res) in sig.items():
        f = getattr(lib, name)
        f.argtypes = args
        f.restype = res
    _lib = lib
    return lib


def version() -> str:
    return load_library().gpl_version().decode()


def _i128(lo: int, hi: int) -> int:
    return ((int(hi) << 64) | (int(lo) & ((1 << 64) - 1)))


@dataclass
class Result:
    """Rows as gpl_fetch_result returns them: the plan's ORDER BY order (else key order),
    decoded keys, exact int128 aggregates, ratio columns (None = SQL NULL)."""
    keys: list
    aggs: list
    stats: dict = field(default_factory=dict)
    ratios: list = field(default_factory=list)

    def as_dict(self):
        return {k: a for k, a in zip(self.keys, self.aggs)}

    def by_key(self) -> "Result":
        """The same rows in group-key order (for comparisons with key-ordered results)."""
        order = sorted(range(len(self.keys)), key=lambda i: self.keys[i])
        return Result([self.keys[i] for i in order], [self.aggs[i] for i in order], self.stats,
                      [self.ratios[i] for i in order] if self.ratios else [])


def _stats_dict(s: _Stats) -> dict:
    d = {k: getattr(s, k) for k, _ in _Stats._fields_ if k != "op_pass"}
    d["op_pass"] = [int(s.op_pass[i]) for i in range(max(0, s.n_ops))]
    return d


def _ptr_and_device(data):
    """(pointer, on_device, nrows, dtype, keepalive) of a numpy array or torch tensor."""
    try:
        import torch
        if isinstance(data, torch.Tensor):
            if not data.is_contiguous():
                data = data.contiguous()
            return data.data_ptr(), int(data.is_cuda), data.numel(), str(data.dtype).replace("torch.", ""), data
    except ImportError:  # pragma: no cover
        pass
    a = np.ascontiguousarray(data)
    return a.ctypes.data, 0, a.size, str(a.dtype), a


class Context:
    """One device + one stream (include/gpl.h `gpl_ctx`)."""

    def __init__(self, device: int = 0, stream=None):
        self._lib = load_library()
        self._h = ctypes.c_void_p()
        if stream is not None and not isinstance(stream, int):
            stream = stream.cuda_stream
            if stream == 0:
                raise ValueError("pass a non-default CUDA stream (torch.cuda.Stream()): the legacy default "
                                 "stream would make libgpl create its own unsynchronised stream")
        st = self._lib.gpl_create(device, ctypes.c_void_p(stream or 0), ctypes.byref(self._h))
        if st:
            raise GplError(st, self._lib.gpl_last_error(None).decode())
        self.device = device
        self._keep = {}

    # -- plumbing
    def _check(self, st):
        if st:
            raise GplError(st, self._lib.gpl_last_error(self._h).decode())

    def close(self):
        if self._h:
            self._lib.gpl_destroy(self._h)
            self._h = ctypes.c_void_p()
            self._keep.clear()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    # -- API
    def set_option(self, key: str, value: int):
        self._check(self._lib.gpl_set_option(self._h, key.encode(), int(value)))

    def load_columns(self, table: str, columns: dict, types: dict | None = None, borrow: bool = False,
                     scales: dict | None = None):
        """columns: name -> numpy array / torch tensor (host or device, int32/int64)."""
        types = types or {}
        scales = scales or {}
        arr = (_Column * len(columns))()
        keep = []
        nrows = None
        for i, (name, data) in enumerate(columns.items()):
            ptr, on_dev, n, dt, ka = _ptr_and_device(data)
            keep.append(ka)
            if nrows is None:
                nrows = n
            elif n != nrows:
                raise ValueError(f"column {name}: {n} rows, expected {nrows}")
            t = types.get(name)
            if t is None:
                t = {"int32": GPL_I32, "int64": GPL_I64}.get(dt)
                if t is None:
                    raise ValueError(f"column {name}: unsupported dtype {dt}")
            cap = 0
            if borrow and on_dev:
                cap = getattr(ka, "_gpl_capacity_rows", 0) or n
            arr[i] = _Column(name.encode(), t, int(scales.get(name, 0)), ptr, on_dev, 0, cap)
        self._check(self._lib.gpl_load_columns(self._h, table.encode(), nrows or 0, len(columns), arr,
                                               GPL_BORROW if borrow else GPL_COPY))
        # borrowed memory must outlive the runs; a copied source must stay alive until the
        # next planning call waits for the (unsynchronised) load: kept until the table is reloaded
        self._keep[table] = keep

    def build_hash(self, segment: str) -> int:
        hid = ctypes.c_int32(-1)
        self._check(self._lib.gpl_build_hash(self._h, segment.encode(), ctypes.byref(hid)))
        return hid.value

    def run_plan(self, segment: str, tile_rows: int = 0):
        self._check(self._lib.gpl_run_plan(self._h, segment.encode(), int(tile_rows)))

    def run_query(self, plan: str, tile_rows: int = 0):
        """All segments of a plan (builds then the probe segment); replays a CUDA graph once warm."""
        self._check(self._lib.gpl_run_query(self._h, plan.encode(), int(tile_rows)))

    def autotune(self, plan: str, max_candidates: int = 0) -> dict:
        """Measure the model's shortlist of pipeline shapes for this query and pin the fastest."""
        m = _Model()
        self._check(self._lib.gpl_autotune(self._h, plan.encode(), int(max_candidates), ctypes.byref(m)))
        return {k: getattr(m, k) for k, _ in _Model._fields_}

    def calibrate(self, rows=None) -> list:
        """Γ, the channel calibration (Eq 1): ring throughput per shape and data size.
        The points are applied to the A9 model and returned as dicts."""
        arr = (ctypes.c_int64 * len(rows))(*rows) if rows else None
        cap = 256
        out = (_Gamma * cap)()
        n = ctypes.c_int32(0)
        self._check(self._lib.gpl_calibrate(self._h, arr, len(rows) if rows else 0, out, cap, ctypes.byref(n)))
        return [{k: getattr(out[i], k) for k, _ in _Gamma._fields_} for i in range(n.value)]

    def set_calibration(self, points: list):
        """Load saved Γ points (as calibrate() returned them); [] clears the calibration."""
        arr = (_Gamma * max(1, len(points)))()
        for i, p in enumerate(points):
            for k, _ in _Gamma._fields_:
                setattr(arr[i], k, p[k])
        self._check(self._lib.gpl_set_calibration(self._h, arr, len(points)))

    def run_plan_kbe(self, segment: str):
        self._check(self._lib.gpl_run_plan_kbe(self._h, segment.encode()))

    def check_plan(self, segment: str):
        self._check(self._lib.gpl_check_plan(self._h, segment.encode()))

    def compile_plan(self, segment: str, tile_rows: int = 0):
        """Warm the plan-specialised kernel cache (NVRTC) for this probe segment."""
        self._check(self._lib.gpl_compile_plan(self._h, segment.encode(), int(tile_rows)))

    def sync(self):
        self._check(self._lib.gpl_sync(self._h))

    def _result(self, fn) -> Result:
        # result buffers are reused across calls (grown on GPL_E_CAPACITY)
        if not hasattr(self, "_rbuf"):
            self._rcap = 256
            self._rbuf = self._alloc_result(self._rcap)
        keys, aggs, rat, r = self._rbuf
        st = fn(ctypes.byref(r))
        if st == GPL_E_CAPACITY and r.n_groups > self._rcap:
            self._rcap = r.n_groups
            self._rbuf = self._alloc_result(self._rcap)
            keys, aggs, rat, r = self._rbuf
            st = fn(ctypes.byref(r))
        self._check(st)
        nk, na, ng, nr = r.n_keys, r.n_aggs, r.n_groups, r.n_ratios
        kl = keys[:ng * nk].tolist()
        al = aggs[:ng * na * 2].tolist()
        rl = rat[:ng * nr].tolist()
        out_k = [tuple(kl[i * nk:(i + 1) * nk]) for i in range(ng)]
        out_a = [[_i128(al[(i * na + j) * 2], al[(i * na + j) * 2 + 1]) for j in range(na)] for i in range(ng)]
        nul = [None if x != x else x for x in rl]  # NaN = SQL NULL
        out_r = (nul if nr == 1 else [tuple(nul[i * nr:(i + 1) * nr]) for i in range(ng)]) if nr else []
        return Result(out_k, out_a, _stats_dict(r.stats), out_r)

    @staticmethod
    def _alloc_result(cap):
        keys, aggs, rat = (np.zeros(cap * 4, dtype=np.int32), np.zeros(cap * 8 * 2, dtype=np.int64),
                           np.zeros(cap * 2, dtype=np.float64))
        r = _Result()
        r.cap_groups = cap
        r.keys, r.aggs, r.ratios = keys.ctypes.data, aggs.ctypes.data, rat.ctypes.data
        return keys, aggs, rat, r

    def fetch_groups(self) -> np.ndarray:
        """Rows of the last hash group-by run: int64 [n, 1 + nagg] (packed key, accumulators)."""
        n, w = ctypes.c_int64(0), ctypes.c_int32(0)
        st = self._lib.gpl_fetch_groups(self._h, None, 0, ctypes.byref(n), ctypes.byref(w))  # size query
        if st != 0 and not (st == GPL_E_CAPACITY and n.value > 0):  # CAPACITY is a size answer only with rows
            self._check(st)
        buf = np.zeros((n.value, max(1, w.value)), dtype=np.int64)
        if n.value:
            self._check(self._lib.gpl_fetch_groups(self._h, buf.ctypes.data_as(ctypes.POINTER(ctypes.c_int64)),
                                                   n.value, ctypes.byref(n), ctypes.byref(w)))
        return buf

    def merge_groups(self, segment: str, rows: np.ndarray) -> Result:
        """Exact merge of several ranks' hash group-by rows (int64 [n, 1 + nagg]) with the segment's ORDER BY/LIMIT."""
        rows = np.ascontiguousarray(rows, dtype=np.int64)
        nrows = rows.shape[0] if rows.ndim == 2 else 0
        return self._result(lambda rp: self._lib.gpl_merge_groups(
            self._h, segment.encode(), rows.ctypes.data_as(ctypes.POINTER(ctypes.c_int64)), nrows, rp))

    def fetch_result(self) -> Result:
        return self._result(lambda rp: self._lib.gpl_fetch_result(self._h, rp))

    def fetch_partials(self, out=None):
        """Raw int128 partials of the last run. `out`: a torch CUDA uint8/int64
        tensor (device copy, async) or None (returns a host numpy uint64 array)."""
        nb = ctypes.c_size_t(0)
        if out is None:
            self._lib.gpl_fetch_partials(self._h, None, 0, 0, ctypes.byref(nb))
            buf = np.zeros(nb.value // 8, dtype=np.uint64)
            self._check(self._lib.gpl_fetch_partials(self._h, ctypes.c_void_p(buf.ctypes.data), 0,
                                                     nb.value, ctypes.byref(nb)))
            return buf
        cap = out.numel() * out.element_size()
        self._check(self._lib.gpl_fetch_partials(self._h, ctypes.c_void_p(out.data_ptr()), int(out.is_cuda),
                                                 cap, ctypes.byref(nb)))
        return out

    def partials_nbytes(self) -> int:
        nb = ctypes.c_size_t(0)
        self._lib.gpl_fetch_partials(self._h, None, 0, 0, ctypes.byref(nb))
        return nb.value

    def decode_partials(self, host_partials: np.ndarray) -> Result:
        a = np.ascontiguousarray(host_partials)
        return self._result(lambda rp: self._lib.gpl_decode_partials(
            self._h, ctypes.c_void_p(a.ctypes.data), a.nbytes, rp))

    def choose_tile_rows(self, segment: str, n_rows: int = 0) -> dict:
        m = _Model()
        self._check(self._lib.gpl_choose_tile_rows(self._h, segment.encode(), int(n_rows), ctypes.byref(m)))
        return {k: getattr(m, k) for k, _ in _Model._fields_}


def merge_partials(gathered: np.ndarray, nranks: int) -> np.ndarray:
    """Fixed-order exact int128 sum of `nranks` partial vectors laid end to end."""
    lib = load_library()
    g = np.ascontiguousarray(gathered).view(np.uint64)
    each = g.nbytes // nranks
    out = np.zeros(each // 8, dtype=np.uint64)
    st = lib.gpl_merge_partials(ctypes.c_void_p(g.ctypes.data), nranks, each, ctypes.c_void_p(out.ctypes.data))
    if st:
        raise GplError(st, "gpl_merge_partials")
    return out
