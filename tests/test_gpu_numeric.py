"""GPU parity of the numeric phase (Alg. 2) through the C ABI.

The kernels compute in float (the paper's precision) with atomic updates (rounding order free);
the oracle computes Alg. 2 in float64 on the same float32-rounded A.  Bars:
  * backward error (Higham, Thm 9.3): |A - L^ U^| <= 4 k u (|L^| |U^|) elementwise, k = the
    longest row of L+U, u = 2^-24 — holds at any size, so it also covers cases the oracle is
    too slow for;
  * forward: |F^ - F| <= 16 k u max((|L| |U|)_ij, 2^-12 max_j' (|L| |U|)_ij') + 1e-6 |F|
    + 4 k FLT_MIN (subnormals flush to zero in the float atomic add) on every factor entry
    against the
    oracle (diagonally dominant A: the factors are well conditioned, so the forward error
    stays within a small multiple of the backward bound).
"""
import numpy as np
import pytest
import scipy.sparse as sp
import torch

import oracle
from oracle import numeric
from inputs import gen

pytestmark = pytest.mark.gpu

lu = pytest.importorskip("paper_conf_ppopp_xia0ar23_b200")

U32 = 2.0 ** -24
FLT_MIN = 2.0 ** -126


def dev():
    return torch.device("cuda", torch.cuda.current_device())


def t(a):
    return torch.from_numpy(np.ascontiguousarray(a)).to(dev())


def csr(rp, ci, v, n):
    return sp.csr_matrix((np.asarray(v, dtype=np.float64), np.asarray(ci), np.asarray(rp)),
                         shape=(n, n))


def split_lu(rp, ci, v, n):
    M = csr(rp, ci, v, n)
    L = sp.tril(M, -1, format="csr") + sp.eye(n, format="csr")
    U = sp.triu(M, 0, format="csr")
    return L, U


def gpu_factor(rp, ci, val32, mode="sparse"):
    rp_lu, ci_lu, val_lu, lptr, lcols = lu.factorize(t(rp), t(ci), t(val32), mode=mode)
    torch.cuda.synchronize()
    return rp_lu.cpu().numpy(), ci_lu.cpu().numpy(), val_lu.cpu().numpy().astype(np.float64)


def check_backward(rp, ci, val32, rp_lu, ci_lu, g):
    n = len(rp) - 1
    A = csr(rp, ci, val32.astype(np.float64), n)
    L, U = split_lu(rp_lu, ci_lu, g, n)
    k = int(np.diff(rp_lu).max()) if n else 0
    R = abs(A - L @ U)
    B = abs(L) @ abs(U)
    bound = (4 * k * U32) * B
    viol = (R - bound).tocsr()
    assert viol.nnz == 0 or viol.data.max() <= 4 * max(k, 1) * FLT_MIN, \
        f"backward error above 4ku|L||U| (max excess {viol.data.max():.3e})"


def check_case(rp, ci, seed, tag="", with_oracle=True, mode="sparse"):
    n = len(rp) - 1
    val32 = gen.dominant_values(rp, ci, seed, dtype=np.float32)
    rp_lu, ci_lu, g = gpu_factor(rp, ci, val32, mode)
    check_backward(rp, ci, val32, rp_lu, ci_lu, g)
    if not with_oracle:
        return
    ref = oracle.fill2(rp, ci)
    assert np.array_equal(rp_lu, ref["row_ptr"]) and np.array_equal(ci_lu, ref["col_idx"])
    As = numeric.scatter(rp, ci, val32.astype(np.float64), ref["row_ptr"], ref["col_idx"])
    f = numeric.factor(ref["row_ptr"], ref["col_idx"], As)
    L, U = split_lu(rp_lu, ci_lu, f, n)
    B = (abs(L) @ abs(U)).tocsr()
    B.sort_indices()
    Bv = np.zeros(len(f))
    for i in range(n):   # (|L||U|)_ij at every pattern entry (i, j)
        cols = B.indices[B.indptr[i]:B.indptr[i + 1]]
        vals = B.data[B.indptr[i]:B.indptr[i + 1]]
        want = ci_lu[rp_lu[i]:rp_lu[i + 1]]
        at = np.searchsorted(cols, want)
        hit = (at < len(cols)) & (cols[np.minimum(at, len(cols) - 1)] == want) if len(cols) else \
            np.zeros(len(want), bool)
        Bv[rp_lu[i]:rp_lu[i + 1]][hit] = vals[at[hit]]
    k = max(1, int(np.diff(rp_lu).max()) if n else 1)
    # + an absolute floor at float's normal range: the float atomic add flushes subnormal
    # results to zero (FTZ), so each of up to k updates of an entry may lose up to 2^-126
    # entries far below their row's scale (decaying fill chains) carry forward error relative
    # to that scale: componentwise forward error is not bounded by the backward error, so
    # the scale used is max(B_ij, 2^-12 max_row B) (the backward check above is elementwise)
    rowmax = (np.maximum.reduceat(np.append(Bv, 0.0), np.minimum(rp_lu[:-1], len(Bv)))
              if n else np.zeros(0))
    scale = np.maximum(Bv, 2.0 ** -12 * np.repeat(rowmax, np.diff(rp_lu)))
    tol = 16 * k * U32 * scale + 1e-6 * np.abs(f) + 4 * k * FLT_MIN
    err = np.abs(g - f)
    bad = np.nonzero(err > tol)[0]
    assert bad.size == 0, (f"{tag}: {bad.size} entries off, first at {bad[0]}: gpu {g[bad[0]]} "
                           f"oracle {f[bad[0]]} tol {tol[bad[0]]}")


def test_random_small():
    rng = np.random.default_rng(77)
    for case in range(40):
        n = int(rng.integers(1, 160))
        rp, ci = gen.random_pattern(n, float(rng.uniform(0.5, 4)), seed=9000 + case,
                                    zero_free_diag=True, sym_frac=float(rng.uniform(0, 1)))
        check_case(rp, ci, case, tag=f"random {case}")


@pytest.mark.parametrize("name", ["lap2d24", "lap3d8", "tridiag", "arrow_first", "arrow_last",
                                  "band", "diag", "circuit", "one"])
def test_structured(name):
    rp, ci = {"lap2d24": lambda: gen.lap2d(24), "lap3d8": lambda: gen.lap3d(8),
              "tridiag": lambda: gen.tridiag(500), "arrow_first": lambda: gen.arrow_first(300),
              "arrow_last": lambda: gen.arrow_last(300), "band": lambda: gen.band(400, 5),
              "diag": lambda: gen.diag_only(1000), "circuit": lambda: gen.circuit(32, 3),
              "one": lambda: gen.diag_only(1)}[name]()
    check_case(rp, ci, 5, tag=name)


@pytest.mark.parametrize("name", ["lap2d64", "lap3d16", "circuit128"])
def test_larger_backward_error(name):
    """Sizes the pure-Python oracle is too slow for: the backward-error bound (any size)."""
    rp, ci = {"lap2d64": lambda: gen.lap2d(64), "lap3d16": lambda: gen.lap3d(16),
              "circuit128": lambda: gen.circuit(128, 1)}[name]()
    check_case(rp, ci, 11, tag=name, with_oracle=False)


def test_zero_pivot_is_an_error():
    rp = np.array([0, 2, 4], dtype=np.int64)
    ci = np.array([0, 1, 0, 1], dtype=np.int32)
    with pytest.raises(lu.LuSymError):
        gpu_factor(rp, ci, np.array([0.0, 1.0, 1.0, 1.0], dtype=np.float32))


def test_missing_diagonal_is_an_error():
    rp = np.array([0, 2, 3], dtype=np.int64)
    ci = np.array([0, 1, 0], dtype=np.int32)
    with pytest.raises(lu.LuSymError):
        gpu_factor(rp, ci, np.array([2.0, 1.0, 1.0], dtype=np.float32))


def test_scatter_rejects_foreign_pattern():
    rp, ci = gen.tridiag(8)
    rp2, ci2 = gen.diag_only(8)
    with pytest.raises(lu.LuSymError):
        lu.numeric_scatter(t(rp), t(ci), t(np.ones(len(ci), np.float32)), t(rp2), t(ci2))


def test_empty():
    rp = np.zeros(1, dtype=np.int64)
    ci = np.zeros(0, dtype=np.int32)
    out = gpu_factor(rp, ci, np.zeros(0, dtype=np.float32))
    assert out[2].size == 0


def test_per_level_launches(monkeypatch):
    """The per-level launch path (LUSYM_NUMERIC_LAUNCH_PER_LEVEL=1) against the same bars."""
    monkeypatch.setenv("LUSYM_NUMERIC_LAUNCH_PER_LEVEL", "1")
    for k, (rp, ci) in enumerate([gen.lap2d(20), gen.circuit(32, 2),
                                  gen.random_pattern(150, 3.0, seed=4, zero_free_diag=True)]):
        check_case(rp, ci, 20 + k, tag=f"per-level {k}")


def test_coop_without_pair_table(monkeypatch):
    """The cooperative kernel resolving positions inline (LUSYM_NUMERIC_TABLE=0)."""
    monkeypatch.setenv("LUSYM_NUMERIC_TABLE", "0")
    for k, (rp, ci) in enumerate([gen.lap2d(20), gen.circuit(32, 2),
                                  gen.random_pattern(150, 3.0, seed=5, zero_free_diag=True)]):
        check_case(rp, ci, 30 + k, tag=f"no-table {k}")


def test_argument_checks():
    """Bad arguments fail loudly instead of computing garbage or faulting: float64 values, host
    tensors, wrong lengths, a level schedule that is not a GLU3-rule schedule of the pattern
    (here the U-rule schedule of an unsymmetric pattern), a repeated column, a level outside
    [0, num_levels)."""
    rp, ci = gen.random_pattern(300, 2.5, seed=21, sym_frac=0.2)
    val = gen.dominant_values(rp, ci, 5, dtype=np.float32)
    h = lu.Symbolic(t(rp), t(ci))
    _, rp_lu, ci_lu = h.run()
    lv_u, nl_u = h.levelize(rp_lu, ci_lu, "u")
    lv_g, nl_g = h.levelize(rp_lu, ci_lu, "glu3")
    h.close()
    with pytest.raises(TypeError):
        lu.numeric_scatter(t(rp), t(ci), t(val.astype(np.float64)), rp_lu, ci_lu)
    with pytest.raises(TypeError):
        lu.numeric_scatter(t(rp), t(ci), torch.from_numpy(val), rp_lu, ci_lu)
    with pytest.raises(ValueError):
        lu.numeric_scatter(t(rp), t(ci), t(val[:-1]), rp_lu, ci_lu)
    v = lu.numeric_scatter(t(rp), t(ci), t(val), rp_lu, ci_lu)
    ptr_u, cols_u = lu.level_schedule(lv_u, nl_u)
    ref_u = oracle.levels(rp_lu.cpu().numpy(), ci_lu.cpu().numpy(), "u")
    ref_g = oracle.levels(rp_lu.cpu().numpy(), ci_lu.cpu().numpy(), "glu3")
    assert ref_u[1] != ref_g[1] or not np.array_equal(ref_u[0], ref_g[0])
    with pytest.raises(lu.LuSymError) as e:
        lu.numeric_factor(rp_lu, ci_lu, ptr_u, cols_u, v.clone())
    assert e.value.status == lu.LU_ERR_ARG
    ptr_g, cols_g = lu.level_schedule(lv_g, nl_g)
    bad = cols_g.clone()
    bad[1] = bad[0]
    with pytest.raises(lu.LuSymError) as e:
        lu.numeric_factor(rp_lu, ci_lu, ptr_g, bad, v.clone())
    assert e.value.status == lu.LU_ERR_ARG
    lu.numeric_factor(rp_lu, ci_lu, ptr_g, cols_g, v)    # the GLU3 schedule is accepted
    lvb = lv_g.clone()
    lvb[3] = nl_g
    with pytest.raises(lu.LuSymError) as e:
        lu.level_schedule(lvb, nl_g)
    assert e.value.status == lu.LU_ERR_ARG


@pytest.mark.parametrize("mode", ["dense", "auto"])
def test_dense_column_mode(mode):
    """GLU3.0's dense column format and the paper's dense/sparse switch
    (L372, "auto": on one B200 every size here is dense) against the same forward / backward
    bars as the sparse (Alg. 6) mode."""
    rng = np.random.default_rng(88)
    for case in range(12):
        n = int(rng.integers(1, 160))
        rp, ci = gen.random_pattern(n, float(rng.uniform(0.5, 4)), seed=9100 + case,
                                    zero_free_diag=True, sym_frac=float(rng.uniform(0, 1)))
        check_case(rp, ci, case, tag=f"{mode} random {case}", mode=mode)
    for name, (rp, ci) in (("lap2d24", gen.lap2d(24)), ("lap3d8", gen.lap3d(8)),
                           ("circuit", gen.circuit(32, 3)), ("arrow_first", gen.arrow_first(300)),
                           ("band", gen.band(400, 5)), ("one", gen.diag_only(1))):
        check_case(rp, ci, 5, tag=f"{mode} {name}", mode=mode)
    check_case(*gen.lap3d(16), 11, tag=f"{mode} lap3d16", with_oracle=False, mode=mode)
    with pytest.raises(lu.LuSymError):     # zero pivot
        gpu_factor(np.array([0, 2, 4], dtype=np.int64), np.array([0, 1, 0, 1], dtype=np.int32),
                   np.array([0.0, 1.0, 1.0, 1.0], dtype=np.float32), mode)
