"""Pins of the CPU oracle (oracle/) against facts fixed by the paper and by mathematics.

None of these compare the oracle with itself: each check is an independent algorithm, a
closed form, a library routine, an invariant, or a value printed in PAPER.md.
"""
import os

import numpy as np
import pytest

import oracle
from inputs import gen
from tests import pins

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "fig1_fixture.txt")


def _oracle_dense(rp, ci):
    r = oracle.fill2(rp, ci)
    return pins.to_dense(r["row_ptr"], r["col_idx"], len(rp) - 1), r


# ---------------------------------------------------------------- Theorem 1 by brute force
def test_bge_random_zero_free_diagonal():
    """Theorem 1 (L96) == Algorithm 1 on 1,000 random tiny matrices (SURVEY §8(c4) BGE)."""
    rng = np.random.default_rng(12345)
    for case in range(1000):
        n = int(rng.integers(1, 41))
        per_row = float(rng.uniform(0.3, 3.5))
        rp, ci = gen.random_pattern(n, per_row, seed=case, zero_free_diag=True,
                                    sym_frac=float(rng.uniform(0, 1)))
        A = pins.to_dense(rp, ci)
        P, r = _oracle_dense(rp, ci)
        assert np.array_equal(P, pins.bge(A)), f"case {case}"
        # sorted, unique rows (R9) and counts == row lengths (R10)
        for i in range(n):
            row = r["col_idx"][r["row_ptr"][i]:r["row_ptr"][i + 1]]
            assert np.all(np.diff(row) > 0)
        assert np.array_equal(np.diff(r["row_ptr"]), r["counts"])


def test_bge_random_with_zero_diagonals():
    """Off-diagonal pattern == BGE; the diagonal is A's own diagonal (R7, L116-129)."""
    for case in range(300):
        n = 3 + case % 30
        rp, ci = gen.random_pattern(n, 2.0, seed=10_000 + case, zero_free_diag=False)
        A = pins.to_dense(rp, ci)
        P, _ = _oracle_dense(rp, ci)
        B = pins.bge(A)
        off = ~np.eye(n, dtype=bool)
        assert np.array_equal(P & off, B & off), f"case {case}"
        assert np.array_equal(np.diag(P), np.diag(A))


def test_certificate_random_and_rejects_corruption():
    """Closure + witness + pattern(A) subset P certify P exactly; corrupted P is rejected."""
    rng = np.random.default_rng(7)
    for case in range(200):
        n = int(rng.integers(2, 60))
        rp, ci = gen.random_pattern(n, float(rng.uniform(0.5, 3)), seed=20_000 + case,
                                    zero_free_diag=bool(case % 2))
        A = pins.to_dense(rp, ci)
        P, _ = _oracle_dense(rp, ci)
        assert pins.certificate(A, P), f"case {case}"
        # flip one off-diagonal bit: must be rejected
        i, j = rng.integers(0, n, 2)
        if i != j:
            Q = P.copy()
            Q[i, j] = ~Q[i, j]
            assert not pins.certificate(A, Q)


# ---------------------------------------------------------------- independent algorithm
@pytest.mark.parametrize("maker", [
    lambda: gen.lap2d(64),                       # cfg1, full
    lambda: gen.lap3d(9),
    lambda: gen.random_pattern(3000, 1.6, seed=3),
    lambda: gen.random_pattern(1500, 2.5, seed=4, sym_frac=0.5),
    lambda: gen.circuit(32, 1),
    lambda: gen.circuit(48, 5),
])
def test_rowmerge_equals_oracle(maker):
    rp, ci = maker()
    r = oracle.fill2(rp, ci)
    rows = pins.rowmerge(rp, ci)
    got = pins.csr_rows(r["row_ptr"], r["col_idx"])
    assert got == rows


def test_superlu_structure():
    """SciPy SuperLU stored L+U structure (natural order, no pivoting) == oracle, small n."""
    sla = pytest.importorskip("scipy.sparse.linalg")
    sp = pytest.importorskip("scipy.sparse")
    mats = [gen.lap2d(12), gen.lap3d(5), gen.circuit(24, 2)]
    mats += [gen.random_pattern(n, 1.8, seed=100 + n, sym_frac=0.3) for n in (50, 200, 400)]
    for rp, ci in mats:
        n = len(rp) - 1
        rng = np.random.default_rng(n)
        vals = rng.uniform(0.1, 1.0, ci.size)
        rows = np.repeat(np.arange(n), np.diff(rp))
        vals[rows == ci] = 10.0 * n                 # diagonally dominant: no pivoting needed
        A = sp.csc_matrix((vals, (rows, ci)), shape=(n, n))
        lu = sla.splu(A, permc_spec="NATURAL", diag_pivot_thresh=0.0, relax=1, panel_size=1,
                      options=dict(Equil=False))
        assert np.array_equal(lu.perm_r, np.arange(n))
        assert np.array_equal(lu.perm_c, np.arange(n))
        S = (lu.L.toarray() != 0) | (lu.U.toarray() != 0)
        S[np.arange(n), np.arange(n)] = True
        P, _ = _oracle_dense(rp, ci)
        assert np.array_equal(P, S)


# ---------------------------------------------------------------- closed forms
@pytest.mark.parametrize("k", list(range(2, 13)) + [64])
def test_closed_form_2d(k):
    rp, ci = gen.lap2d(k)
    r = oracle.fill2(rp, ci)
    assert int(r["row_ptr"][-1]) == pins.nnz_2d(k)
    assert pins.csr_rows(r["row_ptr"], r["col_idx"]) == pins.closed_form_2d(k)
    # TE (R24): every vertex below row i is scanned once -> TE(i) = row_ptr_A[i+1], SV(i) = i
    assert np.array_equal(r["te"], rp[1:])
    assert np.array_equal(r["sv"], np.arange(len(rp) - 1))


@pytest.mark.parametrize("k", [2, 3, 4, 5, 6, 7, 8])
def test_closed_form_3d(k):
    rp, ci = gen.lap3d(k)
    r = oracle.fill2(rp, ci)
    assert int(r["row_ptr"][-1]) == pins.nnz_3d(k)
    assert pins.csr_rows(r["row_ptr"], r["col_idx"]) == pins.closed_form_3d(k)
    assert np.array_equal(r["te"], rp[1:])
    assert np.array_equal(r["sv"], np.arange(len(rp) - 1))


@pytest.mark.parametrize("kind,k", [("2d", k) for k in (1, 2, 3, 5, 8, 17, 40)] +
                         [("3d", k) for k in (1, 2, 3, 4, 7, 9)])
def test_interval_closed_forms_expand_to_pinned_rows(kind, k):
    """tests/closed_forms.py (the O(nnz) checker used on cfg4/cfg5 at full size, on the device)
    expands to exactly the pinned closed-form rows and to the oracle's CSR, whole and in row
    blocks, with numpy and with torch."""
    import torch
    from tests import closed_forms
    rows = [[0]] if k == 1 else (pins.closed_form_2d(k) if kind == "2d" else pins.closed_form_3d(k))
    flat = np.concatenate([np.array(r, dtype=np.int64) for r in rows])
    n = len(rows)
    assert np.array_equal(closed_forms.expand_rows(kind, k, 0, n), flat)
    assert np.array_equal(closed_forms.counts(kind, k), [len(r) for r in rows])
    rp, ci = gen.lap2d(k) if kind == "2d" else gen.lap3d(k)
    ref = oracle.fill2(rp, ci)
    assert np.array_equal(ref["col_idx"], flat)
    for a, b in ((0, n // 2), (n // 3, n), (n - 1, n)):
        if a < b:
            got = closed_forms.expand_rows(kind, k, a, b, torch, "cpu").numpy()
            assert np.array_equal(got, ref["col_idx"][ref["row_ptr"][a]:ref["row_ptr"][b]])
    # the device checker itself, run here on CPU tensors: accepts the truth, rejects a flip
    trp, tci = torch.from_numpy(ref["row_ptr"]), torch.from_numpy(ref["col_idx"].copy())
    assert closed_forms.check_device(kind, k, trp, tci, chunk_entries=97) == flat.size
    if flat.size > 3:
        tci[flat.size // 2] += 1
        with pytest.raises(AssertionError):
            closed_forms.check_device(kind, k, trp, tci, chunk_entries=97)


def test_closed_form_counts_cfg2():
    """cfg2 (3D 40^3): nnz(L+U) = 2k^5-2k^4+3k^3-2k^2+2k-2 = 199,868,878 (counts only)."""
    rp, ci = gen.lap3d(40)
    r = oracle.fill2(rp, ci, emit=False)
    assert int(r["counts"].sum()) == pins.nnz_3d(40) == 199_868_878
    assert int(r["te"].sum()) == int(rp[1:].sum()) == 14_029_019_200


# ---------------------------------------------------------------- special matrices
def test_special_matrices():
    n = 12
    # tridiagonal: no fill, chain levels, TE(i) = row_ptr[i+1]
    rp, ci = gen.tridiag(n)
    r = oracle.fill2(rp, ci)
    assert np.array_equal(r["col_idx"], ci) and np.array_equal(r["row_ptr"], rp)
    assert int(r["te"].sum()) == int(rp[1:].sum()) == 221
    lv, nl = oracle.levels(r["row_ptr"], r["col_idx"])
    assert np.array_equal(lv, np.arange(n)) and nl == n
    # arrow with dense first row/column ("down-pointing arrow"): full fill
    rp, ci = gen.arrow_first(n)
    r = oracle.fill2(rp, ci)
    assert int(r["row_ptr"][-1]) == n * n
    lv, nl = oracle.levels(r["row_ptr"], r["col_idx"])
    assert np.array_equal(lv, np.arange(n))
    # arrow with dense last row/column: no fill; levels 0 except the last column (=1)
    rp, ci = gen.arrow_last(n)
    r = oracle.fill2(rp, ci)
    assert np.array_equal(r["col_idx"], ci)
    assert int(r["te"].sum()) == 2 * (n - 1) + (n + 2 * (n - 1))
    lv, nl = oracle.levels(r["row_ptr"], r["col_idx"])
    assert np.array_equal(lv, np.r_[np.zeros(n - 1, np.int32), 1]) and nl == 2
    # full band: fills exactly its band
    for b in (1, 2, 3, 5):
        rp, ci = gen.band(n, b)
        r = oracle.fill2(rp, ci)
        assert np.array_equal(r["col_idx"], ci)
        lv, _ = oracle.levels(r["row_ptr"], r["col_idx"])
        assert np.array_equal(lv, np.arange(n))
    # diagonal only: nothing to do, all level 0
    rp, ci = gen.diag_only(9)
    r = oracle.fill2(rp, ci)
    assert np.array_equal(r["col_idx"], ci)
    assert np.array_equal(r["te"], np.ones(9))
    lv, nl = oracle.levels(r["row_ptr"], r["col_idx"])
    assert np.all(lv == 0) and nl == 1
    # n = 1 and empty rows
    rp, ci = gen.diag_only(1)
    r = oracle.fill2(rp, ci)
    assert r["counts"].tolist() == [1]
    rp = np.zeros(5, np.int64)
    ci = np.zeros(0, np.int32)
    r = oracle.fill2(rp, ci)
    assert r["counts"].tolist() == [0, 0, 0, 0]
    lv, nl = oracle.levels(r["row_ptr"], r["col_idx"])
    assert np.all(lv == 0) and nl == 1


# ---------------------------------------------------------------- the paper's Fig. 1
def test_fig1_fixture():
    A, fills, table = pins.read_fig1_golden(GOLDEN)
    R = [r for r, cs in A.items() for _ in cs]
    C = [c for r, cs in A.items() for c in cs]
    rp, ci = gen.csr_from_edges(10, R, C)
    r = oracle.fill2(rp, ci)
    P = pins.to_dense(r["row_ptr"], r["col_idx"])
    Adense = pins.to_dense(rp, ci)
    for (i, j) in fills:                 # (9,8) of L92 (1-based)
        assert P[i, j] and not Adense[i, j]
    # the L92 mechanism: row 9 has a non-zero at column 5 and row 5 reaches column 8
    assert Adense[8, 4] and Adense[4, 7]
    lv, nl = oracle.levels(r["row_ptr"], r["col_idx"], "u")
    assert nl == 5
    assert {j: int(lv[j]) for j in range(10)} == table      # Fig. 1(d), L72-78


# ---------------------------------------------------------------- levels
def _check_levels(rp_lu, ci_lu, rule):
    n = len(rp_lu) - 1
    E = pins.dep_edges(rp_lu, ci_lu, rule)
    lv, nl = oracle.levels(rp_lu, ci_lu, rule)
    dp = pins.levels_dp(n, E)
    assert np.array_equal(lv, dp)
    assert nl == (int(dp.max()) + 1 if n else 0)
    for i, j in E:                       # every dependency respected
        assert lv[j] > lv[i]
    has_pred_at = set((j, int(lv[i])) for i, j in E)
    for j in range(n):                   # tightness
        if lv[j] > 0:
            assert (j, int(lv[j]) - 1) in has_pred_at
    return lv


def test_levels_dp_random_both_rules():
    differ = 0
    for case in range(300):
        n = 2 + case % 50
        rp, ci = gen.random_pattern(n, 1.5, seed=30_000 + case, sym_frac=0.2)
        r = oracle.fill2(rp, ci)
        a = _check_levels(r["row_ptr"], r["col_idx"], "u")
        b = _check_levels(r["row_ptr"], r["col_idx"], "glu3")
        differ += int(not np.array_equal(a, b))
    assert differ > 0                    # the two rules are distinguishable (R12)


def test_levels_medium_and_etree():
    for rp, ci in (gen.lap2d(20), gen.lap3d(6), gen.circuit(32, 1)):
        r = oracle.fill2(rp, ci)
        _check_levels(r["row_ptr"], r["col_idx"], "u")
        _check_levels(r["row_ptr"], r["col_idx"], "glu3")
    # structurally symmetric P: U-rule levels == elimination-tree subtree heights
    for case in range(100):
        n = 5 + case % 60
        rp, ci = gen.random_pattern(n, 1.2, seed=40_000 + case, sym_frac=1.0)
        r = oracle.fill2(rp, ci)
        P = pins.to_dense(r["row_ptr"], r["col_idx"])
        assert np.array_equal(P, P.T)
        lv, _ = oracle.levels(r["row_ptr"], r["col_idx"], "u")
        assert np.array_equal(lv, pins.etree_heights(pins.csr_rows(r["row_ptr"], r["col_idx"])))


def test_laplacian_levels_are_chains():
    for rp, ci in (gen.lap2d(30), gen.lap3d(7)):
        r = oracle.fill2(rp, ci)
        n = len(rp) - 1
        lv, nl = oracle.levels(r["row_ptr"], r["col_idx"], "u")
        assert np.array_equal(lv, np.arange(n)) and nl == n


# ---------------------------------------------------------------- sampled rows
def test_row_subset_matches_full():
    rp, ci = gen.circuit(40, 3)
    full = oracle.fill2(rp, ci)
    rows = np.array([0, 5, 17, 1599, 800, 3], dtype=np.int32)
    sub = oracle.fill2(rp, ci, rows=rows)
    fr = pins.csr_rows(full["row_ptr"], full["col_idx"])
    sr = pins.csr_rows(sub["row_ptr"], sub["col_idx"])
    assert sr == [fr[i] for i in rows]
    assert np.array_equal(sub["te"], full["te"][rows])


# ---------------------------------------------------------------- GLU3.0 level types (f3)
def test_level_types_against_bge_dense_rows():
    """Sub-columns per level (Alg. 2 lines 7-14: column j updates every k > j with As(j,k) != 0,
    reading R28) from BGE's dense pattern and the index-order level DP, vs the oracle."""
    rng = np.random.default_rng(99)
    for case in range(150):
        n = int(rng.integers(1, 40))
        rp, ci = gen.random_pattern(n, float(rng.uniform(0.3, 3)), seed=77_000 + case,
                                    sym_frac=float(rng.uniform(0, 1)))
        P = pins.bge(pins.to_dense(rp, ci))
        sub_col = np.triu(P, 1).sum(axis=1)                     # strict-U row counts
        E = [(i, j) for i in range(n) for j in range(i + 1, n) if P[i, j]]
        lv = pins.levels_dp(n, E)
        nl = int(lv.max()) + 1 if n else 0
        r = oracle.fill2(rp, ci)
        lvo, nlo = oracle.levels(r["row_ptr"], r["col_idx"], "u")
        assert nlo == nl and np.array_equal(lvo, lv)
        mc, ms = int(rng.integers(0, 6)), int(rng.integers(0, 5))
        typ, sub, width = oracle.level_types(r["row_ptr"], r["col_idx"], lvo, nl, mc, ms)
        assert np.array_equal(width, np.bincount(lv, minlength=nl))
        assert np.array_equal(sub, np.bincount(lv, weights=sub_col, minlength=nl).astype(np.int64))
        # the three regimes of L208, at the extremes of the two thresholds
        assert np.all(oracle.level_types(r["row_ptr"], r["col_idx"], lvo, nl, n + 1, 0)[0] == 2)
        assert np.all(oracle.level_types(r["row_ptr"], r["col_idx"], lvo, nl, 0, n)[0] == 0)
        tb = oracle.level_types(r["row_ptr"], r["col_idx"], lvo, nl, 0, -1)[0]
        assert np.all(tb == 1)


def test_level_types_2d_grid_closed_form():
    """Natural-order 2D grid: rows of L+U in closed form (pins.closed_form_2d), levels are the
    chain 0..n-1, so level l holds column l with its strict-U count as sub-columns (k in the
    interior, i+2 in the first grid row, n-1-l in the last): every level is type C for
    min_cols >= 2, and the A/B split follows max_sub_a exactly."""
    k = 9
    rp, ci = gen.lap2d(k)
    n = k * k
    r = oracle.fill2(rp, ci)
    lv, nl = oracle.levels(r["row_ptr"], r["col_idx"], "u")
    assert nl == n and np.array_equal(lv, np.arange(n))
    expect_sub = np.array([sum(1 for c in row if c > l)
                           for l, row in enumerate(pins.closed_form_2d(k))], dtype=np.int64)
    assert expect_sub.max() == k and expect_sub[0] == 2 and expect_sub[-1] == 0
    typ, sub, width = oracle.level_types(r["row_ptr"], r["col_idx"], lv, nl, 2, 4)
    assert np.array_equal(sub, expect_sub) and np.all(width == 1) and np.all(typ == 2)
    typ, _, _ = oracle.level_types(r["row_ptr"], r["col_idx"], lv, nl, 1, k - 1)
    assert np.array_equal(typ, np.where(expect_sub <= k - 1, 0, 1))


def test_level_types_fig1():
    """Fig. 1 fixture: level widths are the printed table's (Fig. 1(d), L72-78: {1,2,3,6,7},
    {4,5}, {8}, {9}, {10}); sub-columns are the dependency graph's out-degrees (Fig. 1(b))."""
    A, fills, table = pins.read_fig1_golden(GOLDEN)
    R = [r for r, cs in A.items() for _ in cs]
    C = [c for r, cs in A.items() for c in cs]
    rp, ci = gen.csr_from_edges(10, R, C)
    r = oracle.fill2(rp, ci)
    lv, nl = oracle.levels(r["row_ptr"], r["col_idx"], "u")
    typ, sub, width = oracle.level_types(r["row_ptr"], r["col_idx"], lv, nl, 2, 1)
    assert list(width) == [5, 2, 1, 1, 1]
    outdeg = np.zeros(10, dtype=np.int64)
    for i, j in pins.dep_edges(r["row_ptr"], r["col_idx"], "u"):
        outdeg[i] += 1
    assert list(sub) == [int(outdeg[[c for c in range(10) if table[c] == l]].sum())
                         for l in range(5)]
    assert list(typ[2:]) == [2, 2, 2]
