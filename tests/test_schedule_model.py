"""A sequential model of the fill2 kernel's per-row SCHEDULE (fill2_impl.cuh), checked against
the oracle on CPU.

The kernel does not follow Algorithm 1's one-threshold-at-a-time order literally: it takes a
sorted window of pending thresholds, processes the "simple" ones (all below-neighbours
visited, reading R5b) together, runs a BFS only for the smallest non-simple one, marks simple
thresholds finished ahead of the pointer in a "done" bitmap so they are never re-scanned,
shrinks the window after it was cut short, and emits L(src,:) from the visited bitmap as the
pointer passes.  This model executes exactly that schedule (one valid interleaving
of the parallel window: candidates in increasing order) with Python sets, so a flaw in the
schedule's reasoning shows up here on CPU, independently of the CUDA code and of the oracle's
implementation.  It shares no code with either.
"""
import numpy as np
import pytest

import oracle
from inputs import gen


def model_row(rp, ci, i, wcap, small=32):
    def adj(v):
        return [int(w) for w in ci[rp[v]:rp[v + 1]] if w != v]

    seeds = [int(v) for v in ci[rp[i]:rp[i + 1]]]
    V = set(seeds) | {i}   # visited bitmap
    D = set()              # "done": simple thresholds processed ahead of the pointer
    U = set(v for v in seeds if v > i)
    below = [v for v in seeds if v < i]
    ptr = (min(below) if below else i) - 1
    L = []
    cap = wcap
    while True:
        win = sorted(v for v in V if ptr < v < i and v not in D)[:cap]
        if not win:
            break
        tns = newmin = None
        simple = set()
        for t in win:
            nb = adj(t)
            if not all(w in V for w in nb if w < t):
                tns = t if tns is None else min(tns, t)
                continue
            simple.add(t)
            for w in nb:
                if w > t and w not in V:
                    V.add(w)
                    if w < i:
                        newmin = w if newmin is None else min(newmin, w)
                    else:
                        U.add(w)
        inf = 1 << 62
        m = min(inf if tns is None else tns, inf if newmin is None else newmin)
        last = win[-1]
        nptr = last if m > last else (m if m == tns else m - 1)
        L += sorted(v for v in V if ptr < v <= nptr)   # the pointer passes only L entries
        D |= {t for t in simple if t > nptr}
        if m <= last and m == tns:                      # BFS below the smallest non-simple one
            F = [m]
            while F:
                NF = []
                for f in F:
                    for w in adj(f):
                        if w not in V:
                            V.add(w)
                            if w < m:
                                NF.append(w)
                            elif w > i:
                                U.add(w)
                F = NF
        cap = min(cap, small) if m <= last else min(2 * cap, wcap)
        ptr = nptr
    L += sorted(v for v in V if ptr < v < i)
    return L + ([i] if i in seeds else []) + sorted(U)


@pytest.mark.parametrize("wcap", [1, 2, 3, 7, 2048])
def test_schedule_model_matches_oracle(wcap):
    rng = np.random.default_rng(wcap)
    for case in range(120):
        n = int(rng.integers(2, 60))
        rp, ci = gen.random_pattern(n, float(rng.uniform(0.5, 3)), seed=80_000 + case,
                                    sym_frac=float(rng.uniform(0, 1)),
                                    zero_free_diag=bool(case % 3))
        ref = oracle.fill2(rp, ci)
        for i in range(n):
            exp = ref["col_idx"][ref["row_ptr"][i]:ref["row_ptr"][i + 1]].tolist()
            assert model_row(rp, ci, i, wcap) == exp, (case, i)


def test_schedule_model_structured():
    for rp, ci in (gen.circuit(24, 3), gen.lap3d(5), gen.lap2d(9)):
        ref = oracle.fill2(rp, ci)
        n = len(rp) - 1
        for i in range(n):
            exp = ref["col_idx"][ref["row_ptr"][i]:ref["row_ptr"][i + 1]].tolist()
            assert model_row(rp, ci, i, 16) == exp
