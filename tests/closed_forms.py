"""Vectorised closed forms of the L+U pattern of natural-ordered grid Laplacians (cfg1/2/4/5), as
unions of at most three index intervals per row, for an O(nnz) check of EVERY row of a GPU
result at full size (2.1e9 entries on cfg4/cfg5) — on the device, chunk by chunk.

The row sets are those of tests/pins.py closed_form_2d / closed_form_3d (SURVEY §8(c4),
verified there against brute-force elimination and the oracle); test_oracle_pins.py checks
that the interval form below expands to exactly those rows.

2D k x k, i = y*k + x (5-point):        row i = [i-k, i+k]                        1 <= y <= k-2
                                                [i-k, n-1]                        y = k-1
                                                [i-(x>=1), i+(x<k-1)] U [k, k+x]   y = 0
3D k^3, i = z*k^2 + p (7-point):        row i = [i-k^2, i+k^2]                    1 <= z <= k-2
                                                [i-k^2, n-1]                      z = k-1
                                                (2D row p of plane 0) U [k^2, k^2+p]  z = 0
(for k = 1 the only row is [0, 0]).
"""
from __future__ import annotations

import numpy as np


def _int(cond, like):
    """bool array -> the integer dtype of `like` (numpy or torch)."""
    return cond.astype(like.dtype) if isinstance(cond, np.ndarray) else cond.to(like.dtype)


def _intervals_2d(i, k, n, xp):
    y, x = i // k, i % k
    top = y == k - 1
    mid = (y >= 1) & ~top
    first = y == 0
    a1 = xp.where(first, i - _int(x >= 1, i), i - k)
    b1 = xp.where(top, n - 1 + 0 * i, xp.where(mid, i + k, i + _int(x < k - 1, i)))
    # second interval only on the first grid row: [k, k + x]
    a2 = xp.where(first, k + 0 * i, 0 * i)
    b2 = xp.where(first, k + x, -1 + 0 * i)
    if k == 1:
        a1, b1 = 0 * i, 0 * i
        a2, b2 = 0 * i, -1 + 0 * i
    return a1, b1, a2, b2


def intervals(kind: str, k: int, i, xp=np):
    """Per row i (int64 array, numpy or torch): three inclusive intervals (a1,b1),(a2,b2),(a3,b3),
    sorted and disjoint (an empty one has b < a)."""
    if kind == "2d":
        n = k * k
        a1, b1, a2, b2 = _intervals_2d(i, k, n, xp)
        return a1, b1, a2, b2, 0 * i, -1 + 0 * i
    n, k2 = k ** 3, k * k
    z, p = i // k2, i % k2
    top = z == k - 1
    pa1, pb1, pa2, pb2 = _intervals_2d(p, k, k2, xp)
    zero = z == 0
    a1 = xp.where(zero, pa1, i - k2)
    b1 = xp.where(zero, pb1, xp.where(top, n - 1, i + k2))
    a2 = xp.where(zero, pa2, 0 * i)
    b2 = xp.where(zero, pb2, -1 + 0 * i)
    a3 = xp.where(zero, k2 + 0 * i, 0 * i)
    b3 = xp.where(zero, k2 + p, -1 + 0 * i)
    if k == 1:
        a1, b1 = 0 * i, 0 * i
        a2, b2, a3, b3 = 0 * i, -1 + 0 * i, 0 * i, -1 + 0 * i
    return a1, b1, a2, b2, a3, b3


def counts(kind: str, k: int, xp=np, device=None):
    n = k * k if kind == "2d" else k ** 3
    i = np.arange(n, dtype=np.int64) if xp is np else xp.arange(n, dtype=xp.int64, device=device)
    a1, b1, a2, b2, a3, b3 = intervals(kind, k, i, xp)
    return (b1 - a1 + 1) + xp.clip(b2 - a2 + 1, 0, None) + xp.clip(b3 - a3 + 1, 0, None) \
        if xp is np else (b1 - a1 + 1) + (b2 - a2 + 1).clamp(min=0) + (b3 - a3 + 1).clamp(min=0)


def expand_rows(kind: str, k: int, r0: int, r1: int, xp=np, device=None):
    """Expected col_idx of rows [r0, r1) (concatenated, sorted per row)."""
    if xp is np:
        i = np.arange(r0, r1, dtype=np.int64)
    else:
        i = xp.arange(r0, r1, dtype=xp.int64, device=device)
    a1, b1, a2, b2, a3, b3 = intervals(kind, k, i, xp)
    if xp is np:
        l1 = b1 - a1 + 1
        l2 = np.clip(b2 - a2 + 1, 0, None)
        l3 = np.clip(b3 - a3 + 1, 0, None)
        lens = l1 + l2 + l3
        row = np.repeat(np.arange(r1 - r0), lens)
        start = np.concatenate([[0], np.cumsum(lens)[:-1]])
    else:
        l1 = b1 - a1 + 1
        l2 = (b2 - a2 + 1).clamp(min=0)
        l3 = (b3 - a3 + 1).clamp(min=0)
        lens = l1 + l2 + l3
        row = xp.repeat_interleave(xp.arange(r1 - r0, device=device), lens)
        start = xp.cumsum(lens, 0) - lens
    off = (xp.arange(int(lens.sum()), dtype=xp.int64) if xp is np
           else xp.arange(int(lens.sum()), dtype=xp.int64, device=device)) - start[row]
    o1, o2 = l1[row], l2[row]
    v = xp.where(off < o1, a1[row] + off,
                 xp.where(off < o1 + o2, a2[row] + off - o1, a3[row] + off - o1 - o2))
    return v


def check_device(kind: str, k: int, row_ptr_lu, col_idx_lu, chunk_entries: int = 1 << 27):
    """Every row of a device CSR (torch int64 row_ptr_lu, int32 col_idx_lu) equals the closed
    form; returns the number of entries compared.  Raises AssertionError on the first bad chunk."""
    import torch
    dev = col_idx_lu.device
    n = row_ptr_lu.numel() - 1
    rp = row_ptr_lu
    exp_counts = counts(kind, k, torch, dev)
    assert torch.equal(rp[1:] - rp[:-1], exp_counts), "row lengths differ from the closed form"
    rph = rp.cpu().numpy()
    r0 = 0
    done = 0
    while r0 < n:
        r1 = int(np.searchsorted(rph, rph[r0] + chunk_entries, side="right")) - 1
        r1 = min(max(r1, r0 + 1), n)
        exp = expand_rows(kind, k, r0, r1, torch, dev)
        got = col_idx_lu[int(rph[r0]):int(rph[r1])].to(torch.int64)
        if not torch.equal(got, exp):
            bad = int(torch.nonzero(got != exp)[0])
            row = int(np.searchsorted(rph, rph[r0] + bad, side="right")) - 1
            raise AssertionError(f"{kind} k={k}: row {row} differs from the closed form")
        done += exp.numel()
        r0 = r1
    return done
