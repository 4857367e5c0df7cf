"""B200-native symbolic LU hot path of Xia et al., "End-to-End LU Factorization of Large Matrices
on GPUs" (PPoPP'23) — Python binding over the C ABI in include/lu_sym.h (liblusym.so).

This module only marshals arguments (device pointers, sizes, the current CUDA stream) into the
C library: every step of the path (validation, fill2 count, prefix sum, fill2 emit, dependency
graph, in-degrees, Kahn levels) runs in the hand-written sm_100a kernels of
paper_conf_ppopp_xia0ar23_b200/csrc.  PyTorch provides device memory, streams and process
groups.  There is no CPU fallback: if the library is missing or no CUDA device is present, the
calls raise.

Public API (names follow the paper / SURVEY §8(b)):
  Symbolic(row_ptr, col_idx, **opts)      handle: .count() .scan() .emit() .run() .stats()
  levelize(row_ptr_lu, col_idx_lu, rule)  Algorithm 5 levels
  partition_rows / assemble_counts / assemble_pattern / symbolic_distributed
                                          row sharding across GPUs
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import numpy as np
import torch

from .parallel import (assemble_counts, assemble_pattern, measured_row_cost,  # noqa: F401
                       partition_rows, row_cost_upper_bound)

__all__ = ["Symbolic", "LuSymError", "levelize", "level_schedule", "load_library", "library_path",
           "partition_rows", "assemble_counts", "assemble_pattern", "symbolic_distributed",
           "row_cost_upper_bound", "measured_row_cost", "DEP_U", "DEP_GLU3", "numeric_scatter", "numeric_factor",
           "factorize"]

_HERE = os.path.dirname(os.path.abspath(__file__))
# LUSYM_LIB selects an alternative build of the same library (kernel-variant experiments)
_LIBPATH = os.environ.get("LUSYM_LIB") or os.path.join(_HERE, "lib", "liblusym.so")

LU_OK, LU_ERR_ARG, LU_ERR_INPUT, LU_ERR_NOMEM, LU_ERR_CAPACITY = 0, 1, 2, 3, 4
LU_ERR_CUDA, LU_ERR_STATE, LU_ERR_INTERNAL = 5, 7, 8
DEP_U, DEP_GLU3 = 0, 1
F_GLOBAL_BITMAP, F_NO_BATCH, F_ASCENDING, F_NO_PRUNE, F_KAHN_WIDE_ONLY = 1, 2, 4, 8, 16
F_NO_CONTRACT, F_TWO_PASS, F_ONE_CLASS, F_FORCE_CLASSES = 32, 64, 128, 256
F_SELF_CONT, F_NO_SELF_CONT, F_PAPER_CHUNKS = 512, 1024, 2048
F_MANAGED, F_MANAGED_PREFETCH, F_NO_DEFER, F_NO_SPARSE = 4096, 8192, 16384, 32768
F_DEFER_GLOBAL, F_COUNT_TE = 65536, 131072
F_ASYNC_BFS, F_NO_ASYNC_BFS = 1 << 18, 1 << 19


class LuSymError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"{msg} [status {status}]")
        self.status = status


class _Opts(ctypes.Structure):
    _fields_ = [("struct_size", ctypes.c_int32), ("flags", ctypes.c_int32),
                ("scratch_budget_bytes", ctypes.c_uint64), ("threads_per_row", ctypes.c_int32),
                ("rows_in_flight", ctypes.c_int32), ("queue_capacity", ctypes.c_int32),
                ("ell_width", ctypes.c_int32), ("pool_bytes", ctypes.c_uint64),
                ("defer_windows", ctypes.c_int32), ("defer_max", ctypes.c_int32),
                ("reserved", ctypes.c_int32 * 4)]


class _Stats(ctypes.Structure):
    _fields_ = [("ms_create", ctypes.c_double), ("ms_count", ctypes.c_double),
                ("ms_scan", ctypes.c_double), ("ms_emit", ctypes.c_double),
                ("ms_levelize", ctypes.c_double), ("nnz_lu", ctypes.c_int64),
                ("edges_read_count", ctypes.c_int64), ("edges_read_emit", ctypes.c_int64),
                ("vertices_scanned_count", ctypes.c_int64),
                ("vertices_scanned_emit", ctypes.c_int64), ("spills", ctypes.c_int64),
                ("scratch_bytes", ctypes.c_int64), ("rows_in_flight", ctypes.c_int32),
                ("threads_per_row", ctypes.c_int32), ("smem_bytes_per_row", ctypes.c_int32),
                ("visited_in_smem", ctypes.c_int32), ("ell_width", ctypes.c_int32),
                ("queue_capacity", ctypes.c_int32), ("num_levels", ctypes.c_int32),
                ("levelize_wide_levels", ctypes.c_int32),
                ("levelize_narrow_levels", ctypes.c_int32),
                ("levelize_rank_rounds", ctypes.c_int32), ("row_classes", ctypes.c_int32),
                ("reserved", ctypes.c_int32 * 1),
                ("pool_bytes", ctypes.c_int64), ("rows_retraversed", ctypes.c_int64),
                ("kernel_launches", ctypes.c_int64), ("rows_deferred", ctypes.c_int64),
                ("rows_merge_failed", ctypes.c_int64), ("merge_entries_read", ctypes.c_int64),
                ("ms_tail", ctypes.c_double), ("merge_rounds", ctypes.c_int64),
                ("merge_waits", ctypes.c_int64), ("sample_mean_sv", ctypes.c_double),
                ("heavy_rows", ctypes.c_int64)]


_lib = None
ABI_VERSION = 2

EXPORTED = ["lu_sym_abi_version", "lu_sym_default_opts", "lu_sym_create", "lu_sym_count",
            "lu_sym_scan", "lu_sym_emit", "lu_sym_run", "lu_levelize", "lu_sym_get_stats",
            "lu_sym_destroy", "lu_status_str", "lu_last_error", "lu_sym_set_row_profile",
            "lu_level_schedule", "lu_sym_run_host", "lu_level_types", "lu_numeric_scatter",
            "lu_numeric_factor", "lu_sym_deferred_flags", "lu_sym_merge_deferred",
            "lu_numeric_factor_ex", "lu_sym_nnz_bound"]


def library_path() -> str:
    return _LIBPATH


def load_library():
    """Load liblusym.so (built by __graft_entry__.build()).  Raises if it is missing."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(_LIBPATH):
        raise ImportError(f"{_LIBPATH} not built: run `python -c 'import __graft_entry__ as g; "
                          f"g.build()'` (no CPU fallback exists)")
    lib = ctypes.CDLL(_LIBPATH)
    P, I32, I64 = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64
    lib.lu_sym_abi_version.restype = I32
    lib.lu_sym_default_opts.argtypes = [P]
    lib.lu_sym_create.argtypes = [P, I32, I64, P, P, P, P]
    lib.lu_sym_count.argtypes = [P, I32, I32, P, P]
    lib.lu_sym_scan.argtypes = [P, P, P, P, P]
    lib.lu_sym_emit.argtypes = [P, I32, I32, P, P, I64, P]
    lib.lu_sym_run.argtypes = [P, P, P, P, I64, P, P]
    lib.lu_sym_run_host.argtypes = [P, I32, P, P, P, I64, P, P, P, P]
    lib.lu_sym_nnz_bound.argtypes = [P, P, P]
    lib.lu_sym_nnz_bound.restype = I32
    lib.lu_levelize.argtypes = [P, I32, P, P, I32, P, P, P]
    lib.lu_sym_get_stats.argtypes = [P, P]
    lib.lu_sym_destroy.argtypes = [P]
    lib.lu_sym_set_row_profile.argtypes = [P, P]
    lib.lu_level_schedule.argtypes = [I32, P, I32, P, P, P]
    lib.lu_level_schedule.restype = I32
    lib.lu_level_types.argtypes = [I32, P, P, P, I32, I32, I32, P, P, P]
    lib.lu_level_types.restype = I32
    lib.lu_numeric_scatter.argtypes = [I32, P, P, P, P, P, I64, P, P]
    lib.lu_numeric_scatter.restype = I32
    lib.lu_numeric_factor.argtypes = [I32, P, P, P, P, I32, P, P]
    lib.lu_numeric_factor.restype = I32
    lib.lu_numeric_factor_ex.argtypes = [I32, P, P, P, P, I32, I32, P, P]
    lib.lu_numeric_factor_ex.restype = I32
    lib.lu_sym_set_row_profile.restype = I32
    lib.lu_sym_deferred_flags.argtypes = [P, P, P]
    lib.lu_sym_deferred_flags.restype = I32
    lib.lu_sym_merge_deferred.argtypes = [P, P, P, P, P, P, P]
    lib.lu_sym_merge_deferred.restype = I32
    lib.lu_status_str.argtypes = [I32]
    lib.lu_status_str.restype = ctypes.c_char_p
    lib.lu_last_error.restype = ctypes.c_char_p
    for f in ("lu_sym_create", "lu_sym_count", "lu_sym_scan", "lu_sym_emit", "lu_sym_run",
              "lu_levelize", "lu_sym_get_stats", "lu_sym_run_host"):
        getattr(lib, f).restype = I32
    if lib.lu_sym_abi_version() != ABI_VERSION:
        raise ImportError("liblusym.so ABI version mismatch")
    _lib = lib
    return lib


def _check(status):
    if status != LU_OK:
        lib = load_library()
        raise LuSymError(status, f"{lib.lu_status_str(status).decode()}: "
                                 f"{lib.lu_last_error().decode()}")


def _stream_ptr(stream=None):
    s = stream if stream is not None else torch.cuda.current_stream()
    return ctypes.c_void_p(s.cuda_stream)


def _dev(t: torch.Tensor, dtype, name):
    if not isinstance(t, torch.Tensor) or not t.is_cuda:
        raise TypeError(f"{name} must be a CUDA tensor")
    if t.dtype != dtype:
        raise TypeError(f"{name} must be {dtype}, got {t.dtype}")
    if not t.is_contiguous():
        raise ValueError(f"{name} must be contiguous")
    return ctypes.c_void_p(t.data_ptr())


@dataclass
class Options:
    flags: int = 0
    scratch_budget_bytes: int = 0
    threads_per_row: int = 0
    rows_in_flight: int = 0
    queue_capacity: int = 0
    ell_width: int = 0
    pool_bytes: int = 0
    defer_windows: int = 0
    defer_max: int = 0

    def to_c(self) -> _Opts:
        o = _Opts()
        load_library().lu_sym_default_opts(ctypes.byref(o))
        o.flags = self.flags
        o.scratch_budget_bytes = self.scratch_budget_bytes
        o.threads_per_row = self.threads_per_row
        o.rows_in_flight = self.rows_in_flight
        o.queue_capacity = self.queue_capacity
        o.ell_width = self.ell_width
        o.pool_bytes = self.pool_bytes
        o.defer_windows = self.defer_windows
        o.defer_max = self.defer_max
        return o


class Symbolic:
    """Handle over lu_sym_create for the pattern A (CSR on the current CUDA device).

    row_ptr: int64[n+1], col_idx: int32[nnz] (rows strictly increasing).  The tensors are
    borrowed: keep them alive and unchanged while the handle lives (the handle keeps a
    reference)."""

    def __init__(self, row_ptr: torch.Tensor, col_idx: torch.Tensor, options: Options | None = None,
                 stream=None, **kw):
        lib = load_library()
        if options is None:
            options = Options(**kw)
        self.row_ptr = row_ptr
        self.col_idx = col_idx
        self.n = int(row_ptr.numel()) - 1
        if self.n < 0:
            raise ValueError("row_ptr must have n+1 >= 1 entries")
        self.device = row_ptr.device
        self._h = ctypes.c_void_p()
        opts = options.to_c()
        _check(lib.lu_sym_create(ctypes.byref(self._h), self.n, int(col_idx.numel()),
                                 _dev(row_ptr, torch.int64, "row_ptr"),
                                 ctypes.c_void_p(col_idx.data_ptr()) if col_idx.numel() else None,
                                 ctypes.byref(opts), _stream_ptr(stream)))
        self.nnz_lu = None

    # -- S3
    def count(self, row_begin: int = 0, row_end: int | None = None, fill_count=None, stream=None):
        row_end = self.n if row_end is None else row_end
        if fill_count is None:
            fill_count = torch.zeros(self.n, dtype=torch.int32, device=self.device)
        _check(load_library().lu_sym_count(self._h, row_begin, row_end,
                                           _dev(fill_count, torch.int32, "fill_count")
                                           if self.n else None, _stream_ptr(stream)))
        return fill_count

    # -- S4
    def scan(self, fill_count, row_ptr_lu=None, stream=None):
        if row_ptr_lu is None:
            row_ptr_lu = torch.empty(self.n + 1, dtype=torch.int64, device=self.device)
        nnz = ctypes.c_int64(0)
        _check(load_library().lu_sym_scan(self._h,
                                          _dev(fill_count, torch.int32, "fill_count")
                                          if self.n else None,
                                          _dev(row_ptr_lu, torch.int64, "row_ptr_lu"),
                                          ctypes.byref(nnz), _stream_ptr(stream)))
        self.nnz_lu = int(nnz.value)
        return row_ptr_lu, self.nnz_lu

    # -- S6
    def emit(self, row_ptr_lu, col_idx_lu=None, row_begin: int = 0, row_end: int | None = None,
             stream=None):
        row_end = self.n if row_end is None else row_end
        if col_idx_lu is None:
            col_idx_lu = torch.empty(max(self.nnz_lu or 0, 1), dtype=torch.int32,
                                     device=self.device)[: self.nnz_lu or 0]
        cap = int(col_idx_lu.numel())
        ptr = ctypes.c_void_p(col_idx_lu.data_ptr()) if cap else ctypes.c_void_p(
            row_ptr_lu.data_ptr())
        _check(load_library().lu_sym_emit(self._h, row_begin, row_end,
                                          _dev(row_ptr_lu, torch.int64, "row_ptr_lu"), ptr, cap,
                                          _stream_ptr(stream)))
        return col_idx_lu

    def run(self, stream=None):
        """S3 + S4 + S5 + S6 on this GPU: (fill_count, row_ptr_lu, col_idx_lu)."""
        fc = self.count(stream=stream)
        rp_lu, nnz = self.scan(fc, stream=stream)
        ci_lu = torch.empty(nnz, dtype=torch.int32, device=self.device)   # Alg. 3 line 8
        self.emit(rp_lu, ci_lu, stream=stream)
        return fc, rp_lu, ci_lu

    def run_host(self, cap: int, host_row_ptr=None, host_col_idx=None, nchunks: int = 0,
                 stream=None):
        """S3-S6 with the pattern streamed to host memory behind the traversal
        (lu_sym_run_host): row chunks in increasing order, each scanned, placed and copied to
        the host while later chunks are traversed.  cap = capacity (>= nnz(L+U)) of the device
        and host column arrays; host_* are CPU tensors (pinned for overlap) or None.
        Returns (fill_count, row_ptr_lu, col_idx_lu[:nnz]) on the device."""
        fc = torch.zeros(self.n, dtype=torch.int32, device=self.device)
        rp_lu = torch.empty(self.n + 1, dtype=torch.int64, device=self.device)
        ci_lu = torch.empty(max(cap, 1), dtype=torch.int32, device=self.device)
        for t, dt, name, size in ((host_row_ptr, torch.int64, "host_row_ptr", self.n + 1),
                                  (host_col_idx, torch.int32, "host_col_idx", cap)):
            if t is not None and (t.is_cuda or t.dtype != dt or not t.is_contiguous()
                                  or t.numel() < size):
                raise ValueError(f"{name} must be a contiguous CPU {dt} tensor of >= {size}")
        nnz = ctypes.c_int64(0)
        _check(load_library().lu_sym_run_host(
            self._h, nchunks, _dev(fc, torch.int32, "fill_count") if self.n else None,
            _dev(rp_lu, torch.int64, "row_ptr_lu"), ctypes.c_void_p(ci_lu.data_ptr()), cap,
            ctypes.c_void_p(host_row_ptr.data_ptr()) if host_row_ptr is not None else None,
            ctypes.c_void_p(host_col_idx.data_ptr()) if host_col_idx is not None else None,
            ctypes.byref(nnz), _stream_ptr(stream)))
        self.nnz_lu = int(nnz.value)
        return fc, rp_lu, ci_lu[: self.nnz_lu]

    def nnz_bound(self, stream=None) -> int:
        """A-priori capacity >= nnz(L+U) from A alone (lu_sym_nnz_bound: the Theorem 1 row
        envelopes), for allocating run_host's outputs before the traversal."""
        b = ctypes.c_int64(0)
        _check(load_library().lu_sym_nnz_bound(self._h, ctypes.byref(b), _stream_ptr(stream)))
        return int(b.value)

    # -- row sharding with deferred rows (F_DEFER_GLOBAL, reading G8 across GPUs)
    def deferred_flags(self, flags=None, stream=None):
        """int32[n] with 1 at the rows the last count deferred (OR-ed into `flags` if given)."""
        if flags is None:
            flags = torch.zeros(self.n, dtype=torch.int32, device=self.device)
        _check(load_library().lu_sym_deferred_flags(
            self._h, _dev(flags, torch.int32, "flags") if self.n else None, _stream_ptr(stream)))
        return flags

    def merge_deferred(self, flags, fill_count, row_ptr_lu, col_idx_lu, stream=None):
        """Finish the flagged rows by row-merge over the assembled pattern of the others
        (lu_sym_merge_deferred); fill_count and row_ptr_lu are updated in place.  Returns the
        final nnz; then emit(row_ptr_lu, new array) writes the final CSR."""
        nnz = ctypes.c_int64(0)
        _check(load_library().lu_sym_merge_deferred(
            self._h, _dev(flags, torch.int32, "flags") if self.n else None,
            _dev(fill_count, torch.int32, "fill_count") if self.n else None,
            _dev(row_ptr_lu, torch.int64, "row_ptr_lu"),
            _dev(col_idx_lu, torch.int32, "col_idx_lu") if col_idx_lu.numel() else None,
            ctypes.byref(nnz), _stream_ptr(stream)))
        self.nnz_lu = int(nnz.value)
        return self.nnz_lu

    def levelize(self, row_ptr_lu, col_idx_lu, rule: str = "u", level=None, stream=None):
        return levelize(row_ptr_lu, col_idx_lu, rule, level=level, handle=self, stream=stream)

    def set_row_profile(self, prof):
        """Record a per-row profile on later count passes into prof (int64[n, 4] on the device:
        cycles, vertices scanned, BFS runs, threshold windows); None switches it off."""
        ptr = None
        if prof is not None:
            if prof.dtype != torch.int64 or prof.numel() < 4 * self.n or not prof.is_cuda:
                raise ValueError("prof must be a CUDA int64 tensor with 4*n elements")
            ptr = ctypes.c_void_p(prof.data_ptr())
        self._prof = prof
        _check(load_library().lu_sym_set_row_profile(self._h, ptr))

    def stats(self) -> dict:
        st = _Stats()
        _check(load_library().lu_sym_get_stats(self._h, ctypes.byref(st)))
        return {k: getattr(st, k) for k, _ in _Stats._fields_ if k != "reserved"}

    def close(self):
        if getattr(self, "_h", None) and self._h.value:
            load_library().lu_sym_destroy(self._h)
            self._h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def levelize(row_ptr_lu: torch.Tensor, col_idx_lu: torch.Tensor, rule: str = "u", level=None,
             handle: Symbolic | None = None, stream=None):
    """S8+S9: Kahn levels of the column-dependency DAG (Alg. 5).

    rule 'u' (U(i,j)!=0 => j depends on i, L167) or 'glu3' (reading R12).
    Returns (level int32[n] on the device, num_levels)."""
    lib = load_library()
    n = int(row_ptr_lu.numel()) - 1
    if level is None:
        level = torch.empty(max(n, 0), dtype=torch.int32, device=row_ptr_lu.device)
    nl = ctypes.c_int32(0)
    rule_id = {"u": DEP_U, "glu3": DEP_GLU3}[rule]
    ci = ctypes.c_void_p(col_idx_lu.data_ptr()) if col_idx_lu.numel() else ctypes.c_void_p(
        row_ptr_lu.data_ptr())
    _check(lib.lu_levelize(handle._h if handle is not None else None, n,
                           _dev(row_ptr_lu, torch.int64, "row_ptr_lu"), ci, rule_id,
                           _dev(level, torch.int32, "level") if n else None, ctypes.byref(nl),
                           _stream_ptr(stream)))
    return level, int(nl.value)


def level_schedule(level: torch.Tensor, num_levels: int, stream=None):
    """Columns grouped by level (Fig. 1(d)): (level_ptr int64[num_levels+1], level_cols int32[n])
    on the device; the columns of level l are level_cols[level_ptr[l]:level_ptr[l+1]], ascending."""
    n = int(level.numel())
    dev = level.device
    level_ptr = torch.empty(num_levels + 1, dtype=torch.int64, device=dev)
    level_cols = torch.empty(max(n, 1), dtype=torch.int32, device=dev)[:n]
    _check(load_library().lu_level_schedule(
        n, _dev(level, torch.int32, "level") if n else None, num_levels,
        _dev(level_ptr, torch.int64, "level_ptr"),
        ctypes.c_void_p(level_cols.data_ptr()) if n else None, _stream_ptr(stream)))
    return level_ptr, level_cols


LEVEL_A, LEVEL_B, LEVEL_C = 0, 1, 2


def level_types(row_ptr_lu: torch.Tensor, col_idx_lu: torch.Tensor, level: torch.Tensor,
                num_levels: int, min_cols: int = 0, max_sub_a: int = 0, stream=None):
    """GLU3.0 level types (L208; lu_level_types): (type int32[num_levels] with LEVEL_A/B/C,
    sub-columns int64[num_levels]) on the device.  min_cols <= 0: the SM count; max_sub_a <= 0:
    32."""
    n = int(row_ptr_lu.numel()) - 1
    dev = row_ptr_lu.device
    typ = torch.empty(max(num_levels, 1), dtype=torch.int32, device=dev)[:num_levels]
    sub = torch.empty(max(num_levels, 1), dtype=torch.int64, device=dev)[:num_levels]
    ci = ctypes.c_void_p(col_idx_lu.data_ptr()) if col_idx_lu.numel() else None
    _check(load_library().lu_level_types(
        n, _dev(row_ptr_lu, torch.int64, "row_ptr_lu"), ci,
        _dev(level, torch.int32, "level") if n else None, num_levels, min_cols, max_sub_a,
        ctypes.c_void_p(typ.data_ptr()) if num_levels else None,
        ctypes.c_void_p(sub.data_ptr()) if num_levels else None, _stream_ptr(stream)))
    return typ, sub


def numeric_scatter(row_ptr: torch.Tensor, col_idx: torch.Tensor, val: torch.Tensor,
                    row_ptr_lu: torch.Tensor, col_idx_lu: torch.Tensor, stream=None):
    """As (Alg. 2's input, L175): A's float values at their positions in the L+U pattern, 0 at
    fill entries (lu_numeric_scatter).  Returns val_lu float32[nnz_lu] on the device."""
    n = int(row_ptr_lu.numel()) - 1
    nnz_lu = int(col_idx_lu.numel())
    nnz_a = int(col_idx.numel())
    if int(row_ptr.numel()) != n + 1:
        raise ValueError("row_ptr and row_ptr_lu must describe the same n")
    if int(val.numel()) != nnz_a:
        raise ValueError(f"val has {val.numel()} entries, A has {nnz_a}")
    val_lu = torch.empty(max(nnz_lu, 1), dtype=torch.float32, device=row_ptr_lu.device)[:nnz_lu]
    opt = lambda t, dt, name: _dev(t, dt, name) if t.numel() else None  # noqa: E731
    _check(load_library().lu_numeric_scatter(
        n, _dev(row_ptr, torch.int64, "row_ptr"), opt(col_idx, torch.int32, "col_idx"),
        opt(val, torch.float32, "val"), _dev(row_ptr_lu, torch.int64, "row_ptr_lu"),
        opt(col_idx_lu, torch.int32, "col_idx_lu"), nnz_lu, opt(val_lu, torch.float32, "val_lu"),
        _stream_ptr(stream)))
    return val_lu


NUMERIC_AUTO, NUMERIC_DENSE, NUMERIC_SPARSE = 0, 1, 2


def numeric_factor(row_ptr_lu: torch.Tensor, col_idx_lu: torch.Tensor, level_ptr: torch.Tensor,
                   level_cols: torch.Tensor, val_lu: torch.Tensor, stream=None,
                   mode: str = "sparse"):
    """Algorithm 2 (L165-204) in place on val_lu (float32, CSR of L+U), level by level over a
    schedule of GLU3-rule levels (lu_numeric_factor): L strictly below, U on and above the
    diagonal.  Returns val_lu."""
    n = int(row_ptr_lu.numel()) - 1
    if val_lu.dtype != torch.float32 or not val_lu.is_cuda or not val_lu.is_contiguous():
        raise TypeError("val_lu must be a contiguous CUDA float32 tensor")
    if int(val_lu.numel()) != int(col_idx_lu.numel()):
        raise ValueError("val_lu and col_idx_lu must have one entry per pattern entry")
    if int(level_cols.numel()) != n:
        raise ValueError("level_cols must list the n columns")
    nl = int(level_ptr.numel()) - 1
    opt = lambda t, dt, name: _dev(t, dt, name) if t.numel() else None  # noqa: E731
    m = {"auto": NUMERIC_AUTO, "dense": NUMERIC_DENSE, "sparse": NUMERIC_SPARSE}[mode]
    _check(load_library().lu_numeric_factor_ex(
        n, _dev(row_ptr_lu, torch.int64, "row_ptr_lu"), opt(col_idx_lu, torch.int32, "col_idx_lu"),
        _dev(level_ptr, torch.int64, "level_ptr"), opt(level_cols, torch.int32, "level_cols"), nl,
        m, opt(val_lu, torch.float32, "val_lu"), _stream_ptr(stream)))
    return val_lu


def factorize(row_ptr: torch.Tensor, col_idx: torch.Tensor, val: torch.Tensor,
              options: Options | None = None, stream=None, mode: str = "sparse"):
    """End to end on this GPU: symbolic (fill2, Alg. 1/3), GLU3-rule levels (Alg. 5), the
    level schedule and the numeric phase (Alg. 2).  Returns (row_ptr_lu, col_idx_lu, val_lu,
    level_ptr, level_cols)."""
    h = Symbolic(row_ptr, col_idx, options, stream=stream)
    try:
        _, rp_lu, ci_lu = h.run(stream=stream)
        level, nl = levelize(rp_lu, ci_lu, rule="glu3", stream=stream)
    finally:
        h.close()
    level_ptr, level_cols = level_schedule(level, max(nl, 1) if level.numel() else 0,
                                           stream=stream)
    val_lu = numeric_scatter(row_ptr, col_idx, val, rp_lu, ci_lu, stream=stream)
    numeric_factor(rp_lu, ci_lu, level_ptr, level_cols, val_lu, stream=stream, mode=mode)
    return rp_lu, ci_lu, val_lu, level_ptr, level_cols


def symbolic_distributed(row_ptr: torch.Tensor, col_idx: torch.Tensor, group=None,
                         options: Options | None = None, rule: str = "u", stream=None,
                         handle: Symbolic | None = None, cost=None, output: str = "replicated"):
    """Row-sharded symbolic factorization + levelization on every rank of `group`.

    A is replicated; rank r runs fill2 count and emit on its contiguous, cost-balanced row block
    (rows are independent); per-row counts are all-reduced (disjoint supports),
    every rank scans them, and the pattern blocks are all-gathered, so all ranks end with the
    identical CSR of L+U; levels are then computed replicated.  Rows whose threshold chain is
    too long are deferred on whichever rank holds them and finished, after the pattern of the
    other rows is assembled, by the row-merge tail on every rank (F_DEFER_GLOBAL, reading G8).
    output="local_rows" (SURVEY 8(b) LU_OUT_LOCAL_ROWS) skips the pattern exchange: col_idx_lu
    holds only this rank's rows [row_ptr_lu[rb], row_ptr_lu[re]) and no levels are computed
    (level = num_levels = None; the DAG is global; rows are not deferred).
    Returns (fill_count, row_ptr_lu, col_idx_lu, level, num_levels)."""
    if output not in ("replicated", "local_rows"):
        raise ValueError(f"output must be 'replicated' or 'local_rows', got {output!r}")
    import torch.distributed as dist
    world = dist.get_world_size(group) if dist.is_initialized() else 1
    rank = dist.get_rank(group) if dist.is_initialized() else 0
    if handle is None:
        options = options or Options()
        if world > 1 and output == "replicated":
            options = Options(**{**options.__dict__, "flags": options.flags | F_DEFER_GLOBAL})
        h = Symbolic(row_ptr, col_idx, options, stream=stream)
    else:
        h = handle
    n = h.n
    if cost is None:
        cost = row_cost_upper_bound(row_ptr)
    bounds = partition_rows(cost, world)
    rb, re = int(bounds[rank]), int(bounds[rank + 1])
    if output == "local_rows":
        fc = torch.zeros(n, dtype=torch.int32, device=h.device)
        h.count(rb, re, fc, stream=stream)
        if world > 1:
            fc = assemble_counts(fc, group)
        rp_lu, nnz = h.scan(fc, stream=stream)
        ci_lu = torch.empty(nnz, dtype=torch.int32, device=h.device)
        h.emit(rp_lu, ci_lu, rb, re, stream=stream)
        return fc, rp_lu, ci_lu, None, None
    fc, rp_lu, ci_lu = sharded_pass(h, rb, re, bounds, group, stream=stream)
    level, nl = levelize(rp_lu, ci_lu, rule, handle=h, stream=stream)
    return fc, rp_lu, ci_lu, level, nl


def sharded_pass(h: Symbolic, rb: int, re: int, bounds, group=None, stream=None):
    """One symbolic pass over this rank's rows [rb, re) and the exchange that gives every rank
    the whole CSR of L+U: count (S3), all-reduce of the counts and of the deferred-row flags
    (S7), scan (S4), allocate (S5), emit of the own rows (S6), all-gather of the pattern (S7);
    then, if any rank deferred rows, the row-merge tail over the assembled pattern (replicated
    on every rank, identical), a rescan and the placement of the final CSR."""
    import torch.distributed as dist
    world = dist.get_world_size(group) if dist.is_initialized() else 1
    n = h.n
    fc = torch.zeros(n, dtype=torch.int32, device=h.device)
    h.count(rb, re, fc, stream=stream)
    flags = h.deferred_flags(stream=stream)
    # device time of the exchange steps (S7), recorded on the current stream: h.ms_assemble
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(4)] if world > 1 else None
    if world > 1:
        ev[0].record()
        assemble_counts(fc, group)
        assemble_counts(flags, group)
        ev[1].record()
    rp_lu, nnz = h.scan(fc, stream=stream)
    ci_lu = torch.empty(nnz, dtype=torch.int32, device=h.device)
    h.emit(rp_lu, ci_lu, rb, re, stream=stream)
    if world > 1:
        ev[2].record()
        assemble_pattern(ci_lu, rp_lu, bounds, group)
        ev[3].record()
        ev[3].synchronize()
        h.ms_assemble = ev[0].elapsed_time(ev[1]) + ev[2].elapsed_time(ev[3])
    else:
        h.ms_assemble = 0.0
    if int(flags.sum()) > 0:
        nnz = h.merge_deferred(flags, fc, rp_lu, ci_lu, stream=stream)
        ci_lu = torch.empty(nnz, dtype=torch.int32, device=h.device)
        h.emit(rp_lu, ci_lu, 0, n, stream=stream)
    return fc, rp_lu, ci_lu
