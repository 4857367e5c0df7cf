"""Seeded synthetic input generators (pattern-only CSR matrices).

This module is shared by the oracle tests, the GPU parity tests and bench.py.
It holds NONE of the method's arithmetic (no fill, no traversal, no levels):
it only builds input sparsity patterns, as SURVEY.md §8(d1) / App. C describe.

Every matrix is returned as a pair of numpy arrays
    row_ptr : int64[n+1]   (CSR offsets, row_ptr[0] = 0)
    col_idx : int32[nnz]   (column ids, strictly increasing inside each row)
0-based everywhere.

Workload shapes mirror the paper's SuiteSparse inputs (Table 2,
L382-403: sparse, nnz/n 3.9-111): 2D/3D grid Laplacians in natural order and
a circuit-like power-law matrix with a zero-free diagonal (north_star).
"""
from __future__ import annotations

import numpy as np

__all__ = [
    "csr_from_edges", "lap2d", "lap3d", "circuit", "random_pattern",
    "tridiag", "arrow_first", "arrow_last", "band", "diag_only",
    "config", "CONFIGS", "dominant_values",
]


def csr_from_edges(n: int, rows, cols):
    """Deduplicate (row, col) pairs and return sorted CSR (row_ptr int64, col_idx int32)."""
    rows = np.asarray(rows, dtype=np.int64)
    cols = np.asarray(cols, dtype=np.int64)
    if rows.size:
        if rows.min() < 0 or rows.max() >= n or cols.min() < 0 or cols.max() >= n:
            raise ValueError("edge endpoint out of range")
    key = np.unique(rows * np.int64(n) + cols)
    r = key // n
    c = (key % n).astype(np.int32)
    counts = np.bincount(r, minlength=n).astype(np.int64)
    row_ptr = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(counts, out=row_ptr[1:])
    return row_ptr, c


def dominant_values(row_ptr, col_idx, seed: int, dtype=np.float64):
    """Seeded values for a pattern (numeric phase): off-diagonal entries uniform
    in [-1, 1), the diagonal 1 + (sum of |off-diagonal| in its row) + (same in its column), so
    A is strictly diagonally dominant by rows and by columns and the pivot-free LU (reading
    R29) is stable.  Rows without a stored diagonal keep only their off-diagonal values."""
    rp = np.asarray(row_ptr, dtype=np.int64)
    ci = np.asarray(col_idx, dtype=np.int64)
    n = rp.size - 1
    rng = np.random.default_rng(seed)
    val = rng.uniform(-1.0, 1.0, size=ci.size)
    row = np.repeat(np.arange(n, dtype=np.int64), np.diff(rp))
    diag = row == ci
    off = np.where(diag, 0.0, np.abs(val))
    val[diag] = 1.0 + np.bincount(row, weights=off, minlength=n)[row[diag]] + \
        np.bincount(ci, weights=off, minlength=n)[ci[diag]]
    return val.astype(dtype)


def _diag(n):
    v = np.arange(n, dtype=np.int64)
    return v, v


def lap2d(k: int):
    """5-point Laplacian pattern on a k x k grid, natural order i = y*k + x."""
    n = k * k
    y, x = np.meshgrid(np.arange(k), np.arange(k), indexing="ij")
    i = (y * k + x).ravel().astype(np.int64)
    y = y.ravel()
    x = x.ravel()
    R = [i]
    C = [i]
    for dy, dx in ((-1, 0), (1, 0), (0, -1), (0, 1)):
        m = (y + dy >= 0) & (y + dy < k) & (x + dx >= 0) & (x + dx < k)
        R.append(i[m])
        C.append(((y[m] + dy) * k + (x[m] + dx)).astype(np.int64))
    return csr_from_edges(n, np.concatenate(R), np.concatenate(C))


def lap3d(k: int):
    """7-point Laplacian pattern on a k^3 grid, natural order i = (z*k + y)*k + x (cfg2/cfg5)."""
    n = k ** 3
    z, y, x = np.meshgrid(np.arange(k), np.arange(k), np.arange(k), indexing="ij")
    z = z.ravel(); y = y.ravel(); x = x.ravel()
    i = ((z * k + y) * k + x).astype(np.int64)
    R = [i]
    C = [i]
    for dz, dy, dx in ((-1, 0, 0), (1, 0, 0), (0, -1, 0), (0, 1, 0), (0, 0, -1), (0, 0, 1)):
        m = ((z + dz >= 0) & (z + dz < k) & (y + dy >= 0) & (y + dy < k)
             & (x + dx >= 0) & (x + dx < k))
        R.append(i[m])
        C.append((((z[m] + dz) * k + (y[m] + dy)) * k + (x[m] + dx)).astype(np.int64))
    return csr_from_edges(n, np.concatenate(R), np.concatenate(C))


def _nd_order(s: int, leaf: int = 64):
    """Nested-dissection order of an s x s mesh by recursive coordinate bisection."""
    out = []

    def rec(r0, r1, c0, c1):
        h = r1 - r0
        w = c1 - c0
        if h <= 0 or w <= 0:
            return
        if h * w <= leaf or (h < 3 and w < 3):
            rr, cc = np.meshgrid(np.arange(r0, r1), np.arange(c0, c1), indexing="ij")
            out.append((rr * s + cc).ravel())
            return
        if w >= h:
            m = (c0 + c1) // 2
            rec(r0, r1, c0, m)
            rec(r0, r1, m + 1, c1)
            out.append(np.arange(r0, r1) * s + m)
        else:
            m = (r0 + r1) // 2
            rec(r0, m, c0, c1)
            rec(m + 1, r1, c0, c1)
            out.append(m * s + np.arange(c0, c1))

    rec(0, s, 0, s)
    return np.concatenate(out).astype(np.int64)


def circuit(s: int, seed: int = 1):
    """Circuit-like power-law pattern, n = s*s, zero-free diagonal, unsymmetric.

    Mesh with 85% of edges kept (10% one-directional), 32 Zipf hubs covering 0.45 n
    incidences, nested-dissection order with hubs last.
    """
    rng = np.random.default_rng(seed)
    n = s * s
    r, c = np.meshgrid(np.arange(s), np.arange(s), indexing="ij")
    r = r.ravel(); c = c.ravel()
    v = (r * s + c).astype(np.int64)
    hm = c < s - 1
    vm = r < s - 1
    a = np.concatenate([v[hm], v[vm]])
    b = np.concatenate([v[hm] + 1, v[vm] + s])
    m = a.size
    keep = rng.random(m) < 0.85
    a = a[keep]; b = b[keep]
    m = a.size
    sym = rng.random(m) < 0.9
    fwd = rng.random(m) < 0.5
    R = [a[sym], b[sym], a[~sym & fwd], b[~sym & ~fwd]]
    C = [b[sym], a[sym], b[~sym & fwd], a[~sym & ~fwd]]
    hubs = rng.choice(n, 32, replace=False)
    H = sum(1.0 / kk for kk in range(1, 33))
    for kk in range(1, 33):
        h = np.int64(hubs[kk - 1])
        deg = max(1, int(np.round(0.45 * n * (1.0 / kk) / H)))
        nb = rng.choice(n, deg, replace=False).astype(np.int64)
        nb = nb[nb != h]
        sym = rng.random(nb.size) < 0.9
        fwd = rng.random(nb.size) < 0.5
        hh = np.full(nb.size, h, dtype=np.int64)
        R += [hh[sym], nb[sym], hh[~sym & fwd], nb[~sym & ~fwd]]
        C += [nb[sym], hh[sym], nb[~sym & fwd], hh[~sym & ~fwd]]
    d, _ = _diag(n)
    R.append(d); C.append(d)
    rows = np.concatenate(R); cols = np.concatenate(C)
    # ordering: nested dissection, hubs dropped and appended last in rng.choice order
    nd = _nd_order(s)
    is_hub = np.zeros(n, dtype=bool)
    is_hub[hubs] = True
    order = np.concatenate([nd[~is_hub[nd]], hubs.astype(np.int64)])
    perm = np.empty(n, dtype=np.int64)       # old label -> new label
    perm[order] = np.arange(n, dtype=np.int64)
    return csr_from_edges(n, perm[rows], perm[cols])


def random_pattern(n: int, per_row: float, seed: int, zero_free_diag: bool = True,
                   sym_frac: float = 0.0):
    """Uniform random pattern with ~per_row off-diagonal entries per row (tiny-matrix tests)."""
    rng = np.random.default_rng(seed)
    m = int(round(per_row * n))
    rows = rng.integers(0, n, m)
    cols = rng.integers(0, n, m)
    if sym_frac > 0:
        s = rng.random(m) < sym_frac
        rows, cols = np.concatenate([rows, cols[s]]), np.concatenate([cols, rows[s]])
    if zero_free_diag:
        d = np.arange(n)
        rows = np.concatenate([rows, d]); cols = np.concatenate([cols, d])
    else:
        keep = rows != cols
        rows = rows[keep]; cols = cols[keep]
        dmask = rng.random(n) < 0.5
        d = np.arange(n)[dmask]
        rows = np.concatenate([rows, d]); cols = np.concatenate([cols, d])
    return csr_from_edges(n, rows, cols)


def tridiag(n: int):
    i = np.arange(n)
    R = [i, i[1:], i[:-1]]
    C = [i, i[:-1], i[1:]]
    return csr_from_edges(n, np.concatenate(R), np.concatenate(C))


def arrow_first(n: int):
    """Dense first row and first column plus the diagonal ("down-pointing arrow": full fill)."""
    i = np.arange(n)
    R = [i, np.zeros(n, np.int64), i]
    C = [i, i, np.zeros(n, np.int64)]
    return csr_from_edges(n, np.concatenate(R), np.concatenate(C))


def arrow_last(n: int):
    """Dense last row and last column plus the diagonal (no fill)."""
    i = np.arange(n)
    last = np.full(n, n - 1)
    R = [i, last, i]
    C = [i, i, last]
    return csr_from_edges(n, np.concatenate(R), np.concatenate(C))


def band(n: int, b: int):
    """Full band of half-width b (|i-j| <= b)."""
    R = []
    C = []
    i = np.arange(n)
    for d in range(-b, b + 1):
        m = (i + d >= 0) & (i + d < n)
        R.append(i[m]); C.append(i[m] + d)
    return csr_from_edges(n, np.concatenate(R), np.concatenate(C))


def diag_only(n: int):
    i = np.arange(n)
    return csr_from_edges(n, i, i)


# --- the five BASELINE.json configs ---------------------------------------
CONFIGS = {
    1: ("lap2d_k64", lambda: lap2d(64)),
    2: ("lap3d_k40", lambda: lap3d(40)),
    3: ("circuit_s1024_seed1", lambda: circuit(1024, 1)),
    4: ("lap2d_k1024", lambda: lap2d(1024)),
    5: ("lap3d_k64", lambda: lap3d(64)),
}


def config(i: int):
    """Return (name, row_ptr, col_idx) for BASELINE.json configs[i-1]."""
    name, fn = CONFIGS[i]
    rp, ci = fn()
    return name, rp, ci
