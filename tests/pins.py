"""Independent checks that pin the oracle to something other than itself (no shared code with
oracle/ or with the CUDA path).  Each function states the fact it encodes.

  bge(...)              Theorem 1 as dense boolean Gaussian elimination: row i
                        receives row k's entries right of k whenever M[i,k] is set, k < i.
  rowmerge(...)         An independent symbolic algorithm: split every fill path at its largest
                        intermediate t, P_i = A_i U  U_{t in L_i} (U_t \\ {t, i}).
  closed_form_2d/3d     Exact L+U rows of natural-ordered 5-/7-point grids (derivation in
                        DESIGN.md "Pins").
  certificate(...)      pattern(A) subset P, closure and witness of Theorem 1 over t < min(i,j).
  levels_dp(...)        level(k) = max(-1, level(preds)) + 1 evaluated in index
                        order (every edge goes low -> high), i.e. a longest-path DP, not Kahn.
  etree_heights(...)    On structurally symmetric P the U-rule levels equal the subtree heights of
                        the elimination tree parent(i) = min(U_i \\ {i}).
"""
from __future__ import annotations

import heapq

import numpy as np


def to_dense(row_ptr, col_idx, n=None):
    n = len(row_ptr) - 1 if n is None else n
    M = np.zeros((n, n), dtype=bool)
    for i in range(n):
        M[i, col_idx[row_ptr[i]:row_ptr[i + 1]]] = True
    return M


def bge(A: np.ndarray) -> np.ndarray:
    """Boolean Gaussian elimination (no pivoting) on a dense bool matrix; returns the filled M."""
    M = A.copy()
    n = M.shape[0]
    for k in range(n):
        rows = np.nonzero(M[k + 1:, k])[0] + k + 1
        if rows.size:
            M[np.ix_(rows, np.arange(k + 1, n))] |= M[k, k + 1:]
    return M


def rowmerge(row_ptr, col_idx):
    """Row-merge symbolic factorization; returns list of sorted int lists (rows of L+U)."""
    n = len(row_ptr) - 1
    U = [None] * n
    rows = []
    for i in range(n):
        Ai = [int(c) for c in col_idx[row_ptr[i]:row_ptr[i + 1]]]
        S = set(Ai)
        heap = [v for v in Ai if v < i]
        heapq.heapify(heap)
        while heap:
            t = heapq.heappop(heap)
            for x in U[t]:
                if x != t and x != i and x not in S:
                    S.add(x)
                    if x < i:
                        heapq.heappush(heap, x)
        r = sorted(S)
        rows.append(r)
        U[i] = [x for x in r if x >= i]
    return rows


def closed_form_2d(k: int):
    """Rows of L+U for the natural-ordered k x k 5-point Laplacian, i = y*k + x (k >= 2)."""
    n = k * k
    rows = []
    for i in range(n):
        y, x = divmod(i, k)
        if y >= 1:
            L = list(range(i - k, i))
        else:
            L = [i - 1] if x >= 1 else []
        if y == k - 1:
            U = list(range(i, n))
        elif y >= 1:
            U = list(range(i, i + k + 1))
        else:
            U = [i] + ([i + 1] if x < k - 1 else []) + list(range(k, k + x + 1))
        rows.append(sorted(set(L + U)))
    return rows


def closed_form_3d(k: int):
    """Rows of L+U for the natural-ordered k^3 7-point Laplacian, i = z*k^2 + p (k >= 2)."""
    n = k ** 3
    k2 = k * k
    plane0 = closed_form_2d(k)
    rows = []
    for i in range(n):
        z, p = divmod(i, k2)
        if z == 0:
            r = set(plane0[p]) | set(range(k2, k2 + p + 1))
        else:
            L = range(i - k2, i)
            U = range(i, n) if z == k - 1 else range(i, i + k2 + 1)
            r = set(L) | set(U)
        rows.append(sorted(r))
    return rows


def nnz_2d(k):
    return 2 * k ** 3 - k ** 2 + 2 * k - 2


def nnz_3d(k):
    return 2 * k ** 5 - 2 * k ** 4 + 3 * k ** 3 - 2 * k ** 2 + 2 * k - 2


def certificate(A: np.ndarray, P: np.ndarray) -> bool:
    """True iff P is exactly the Theorem-1 pattern of A (dense bool, zero-free diagonal or not).

    (a) A subset P; (b) closure: (i,t),(t,j) in P with t < min(i,j), i != j  =>  (i,j) in P;
    (c) witness: every off-diagonal (i,j) in P \\ A has such a t; (d) diag(P) == diag(A).
    Induction on min(i,j) shows (a)-(d) determine P uniquely.
    """
    n = A.shape[0]
    if np.any(A & ~P):
        return False
    if np.any(np.diag(P) != np.diag(A)):
        return False
    Lo = np.tril(P, -1).astype(np.int64)   # (i,t), t < i
    Up = np.triu(P, 1).astype(np.int64)    # (t,j), t < j
    M = (Lo @ Up) > 0                      # exists t < min(i,j) with (i,t),(t,j) in P
    off = ~np.eye(n, dtype=bool)
    if np.any(M & off & ~P):
        return False
    if np.any(P & ~A & off & ~M):
        return False
    return True


def dep_edges(row_ptr, col_idx, rule="u"):
    """Edges (i, j), i < j, of the column-dependency graph (GLU3 reading R12)."""
    n = len(row_ptr) - 1
    E = []
    for r in range(n):
        for c in col_idx[row_ptr[r]:row_ptr[r + 1]]:
            c = int(c)
            if c > r:
                E.append((r, c))
            elif c < r and rule == "glu3":
                E.append((c, r))
    return E


def levels_dp(n, edges):
    preds = [[] for _ in range(n)]
    for i, j in edges:
        assert i < j
        preds[j].append(i)
    lvl = [0] * n
    for j in range(n):
        lvl[j] = max([-1] + [lvl[i] for i in preds[j]]) + 1
    return np.array(lvl, dtype=np.int32)


def etree_heights(rows):
    n = len(rows)
    parent = [-1] * n
    for i, r in enumerate(rows):
        ups = [c for c in r if c > i]
        parent[i] = min(ups) if ups else -1
    h = [0] * n
    for i in range(n):          # children have smaller index than parents
        p = parent[i]
        if p >= 0:
            h[p] = max(h[p], h[i] + 1)
    return np.array(h, dtype=np.int32)


def csr_rows(row_ptr, col_idx):
    return [list(map(int, col_idx[row_ptr[i]:row_ptr[i + 1]])) for i in range(len(row_ptr) - 1)]


def read_fig1_golden(path):
    """Parse tests/golden/fig1_fixture.txt -> (A rows 0-based dict, fills 0-based, levels dict)."""
    A = {}
    fills = []
    levels = {}
    with open(path) as f:
        for line in f:
            line = line.strip()
            if not line or line.startswith("#"):
                continue
            tag, rest = line.split(" ", 1)
            if tag == "A":
                r, cs = rest.split(":")
                A[int(r) - 1] = [int(c) - 1 for c in cs.split()]
            elif tag == "FILL":
                a, b = rest.split()
                fills.append((int(a) - 1, int(b) - 1))
            elif tag == "LEVEL":
                lv, cs = rest.split(":")
                for c in cs.split():
                    levels[int(c) - 1] = int(lv)
    return A, fills, levels
