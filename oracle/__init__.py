"""ORACLE — test infrastructure only (see oracle/fill2_oracle.c for the paper citations).

Plain CPU reference for the symbolic LU hot path of Xia et al. (PPoPP'23):
  * fill2(...)   Algorithm 1 per row + the two-stage count / prefix-sum /
                 emit structure of Algorithm 3 (L253-270), producing CSR of L+U.
  * levels(...)  Kahn levelization, Algorithm 5 (L290-320), level formula L283.

Only tests/, __graft_entry__.smoke() and bench.py (cpu_baseline / --impl reference) may import
this package.  It never imports the CUDA package and the CUDA package never imports it.

Pins (tests/test_oracle_pins.py, run with -m "not gpu"): brute-force boolean Gaussian
elimination, an independent row-merge symbolic, SciPy SuperLU structure, 2D/3D grid closed
forms, special matrices, the Fig. 1 fixture (tests/golden/), the closure+witness certificate,
and an index-order longest-path DP / elimination-tree heights for the levels.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "fill2_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None


def build(force: bool = False) -> str:
    """Compile the C oracle (gcc, OpenMP) next to its source; returns the .so path."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-shared", "-fPIC", _SRC, "-o", tmp])
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    if _lib is None:
        lib = ctypes.CDLL(build())
        P = ctypes.c_void_p
        lib.oracle_fill2.argtypes = [ctypes.c_int32, P, P, P, ctypes.c_int64, P, P, P, P, P,
                                     ctypes.c_int]
        lib.oracle_fill2.restype = ctypes.c_int
        lib.oracle_kahn.argtypes = [ctypes.c_int32, P, P, ctypes.c_int, P]
        lib.oracle_kahn.restype = ctypes.c_int64
        _lib = lib
    return _lib


def _ptr(a):
    return None if a is None else a.ctypes.data_as(ctypes.c_void_p)


def fill2(row_ptr, col_idx, rows=None, emit: bool = True, threads: int = 0):
    """Symbolic factorization by Algorithm 1, rows independent.

    rows=None computes every row; otherwise only the listed rows (sampled parity).
    Returns dict(counts=int32[m], te=int64[m], sv=int64[m], row_ptr=int64[m+1],
    col_idx=int32[nnz] | None); te / sv = traversed edges / scanned vertices per row.
    where m = number of computed rows and row_ptr/col_idx is the CSR of those rows (Alg. 3:
    count, prefix sum, allocate, emit).
    """
    lib = _load()
    rp = np.ascontiguousarray(row_ptr, dtype=np.int64)
    ci = np.ascontiguousarray(col_idx, dtype=np.int32)
    n = rp.size - 1
    if rows is None:
        r = None
        m = n
    else:
        r = np.ascontiguousarray(rows, dtype=np.int32)
        m = r.size
    counts = np.zeros(m, dtype=np.int32)
    te = np.zeros(m, dtype=np.int64)
    sv = np.zeros(m, dtype=np.int64)
    rc = lib.oracle_fill2(n, _ptr(rp), _ptr(ci), _ptr(r), m, _ptr(counts), _ptr(te), _ptr(sv),
                          None, None, threads)
    if rc != 0:
        raise MemoryError("oracle_fill2 allocation failed")
    out_ptr = np.zeros(m + 1, dtype=np.int64)          # Alg. 3 line 7: prefix_sum(fill_count)
    np.cumsum(counts, out=out_ptr[1:])
    cols = None
    if emit:
        cols = np.empty(int(out_ptr[-1]), dtype=np.int32)  # line 8: allocate
        rc = lib.oracle_fill2(n, _ptr(rp), _ptr(ci), _ptr(r), m, None, None, None,
                              _ptr(out_ptr), _ptr(cols), threads)
        if rc != 0:
            raise MemoryError("oracle_fill2 allocation failed")
    return {"counts": counts, "te": te, "sv": sv, "row_ptr": out_ptr, "col_idx": cols}


def levels(row_ptr_lu, col_idx_lu, rule: str = "u"):
    """Kahn levelization of the column-dependency DAG (Algorithm 5).  rule: 'u' | 'glu3'.

    Returns (level int32[n], num_levels)."""
    lib = _load()
    rp = np.ascontiguousarray(row_ptr_lu, dtype=np.int64)
    ci = np.ascontiguousarray(col_idx_lu, dtype=np.int32)
    n = rp.size - 1
    lvl = np.full(n, -1, dtype=np.int32)
    rc = lib.oracle_kahn(n, _ptr(rp), _ptr(ci), 0 if rule == "u" else 1, _ptr(lvl))
    if rc == -1:
        raise MemoryError("oracle_kahn allocation failed")
    if rc == -2:
        raise ValueError("dependency graph has a cycle")
    return lvl, int(rc)


# GLU3.0 level types, reading R28: the sub-columns of column j are
# the columns k > j with As(j,k) != 0 — the columns Alg. 2 lines 7-14 update from column j
# (L165-204), i.e. column j's out-edges in the U-rule dependency graph (L167).
LEVEL_A, LEVEL_B, LEVEL_C = 0, 1, 2


def level_types(row_ptr_lu, col_idx_lu, level, num_levels, min_cols, max_sub_a):
    """Per level l: width[l] = number of columns, sub[l] = total sub-columns of its columns;
    type[l] = C if width < min_cols ("a limited number of columns"), else A if
    sub <= max_sub_a * width ("very few associated sub-columns" per column), else B ("great
    numbers of columns ... also many sub-columns").  Plain loops; returns (type, sub, width)."""
    rp = np.asarray(row_ptr_lu, dtype=np.int64)
    ci = np.asarray(col_idx_lu)
    lv = np.asarray(level)
    n = len(rp) - 1
    width = [0] * num_levels
    sub = [0] * num_levels
    for j in range(n):
        u = 0
        for p in range(rp[j], rp[j + 1]):
            if ci[p] > j:
                u += 1
        width[lv[j]] += 1
        sub[lv[j]] += u
    typ = []
    for l in range(num_levels):
        if width[l] < min_cols:
            typ.append(LEVEL_C)
        elif sub[l] <= max_sub_a * width[l]:
            typ.append(LEVEL_A)
        else:
            typ.append(LEVEL_B)
    return (np.array(typ, dtype=np.int32), np.array(sub, dtype=np.int64),
            np.array(width, dtype=np.int64))
