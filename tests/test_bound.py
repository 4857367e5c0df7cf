"""A-priori capacity of L+U (lu_sym_nnz_bound, include/lu_sym.h): the Theorem 1 row envelopes.

Row i of L+U lies in [min(i, min A(i,:)), max(i, max_{u<=i} max A(u,:))] (a fill
path's first vertex is in A(i,:) and its intermediates are below min(i,j)).  The CPU tests pin
that reasoning against the oracle (every row of the pattern inside its envelope, so the sum of
envelope lengths bounds nnz, and is tight on the natural-ordered grids, whose band fills in every
row past the first k (2D) or k^2 (3D)); the GPU test checks the library's value against the same
sums."""
import numpy as np
import pytest

import oracle
from inputs import gen
from tests import closed_forms, pins


def envelope(rp, ci):
    """Per-row [lo, hi] of the Theorem 1 envelope (plain numpy, test-side)."""
    n = len(rp) - 1
    i = np.arange(n)
    nz = np.diff(rp) > 0
    first = np.where(nz, ci[np.minimum(rp[:-1], max(len(ci) - 1, 0))] if len(ci) else i, i)
    last = np.where(nz, ci[np.maximum(rp[1:] - 1, 0)] if len(ci) else i, i)
    lo = np.minimum(i, first)
    hi = np.maximum.accumulate(np.maximum(i, last)) if n else last
    return lo, hi


def bound(rp, ci):
    lo, hi = envelope(rp, ci)
    return int((hi - lo + 1).sum())


CASES = [gen.lap2d(9), gen.lap3d(5), gen.circuit(20, 1), gen.circuit(24, 3),
         gen.random_pattern(300, 2.5, seed=4), gen.random_pattern(200, 1.5, seed=8, sym_frac=0.3),
         gen.random_pattern(150, 2.0, seed=2, zero_free_diag=False)]


@pytest.mark.parametrize("k", range(len(CASES)))
def test_every_row_lies_in_its_envelope(k):
    rp, ci = CASES[k]
    ref = oracle.fill2(rp, ci)
    lo, hi = envelope(rp, ci)
    r, c = ref["row_ptr"], ref["col_idx"]
    for i in range(len(rp) - 1):
        row = c[r[i]:r[i + 1]]
        if len(row):
            assert row[0] >= lo[i] and row[-1] <= hi[i], i
    assert bound(rp, ci) >= int(r[-1])


@pytest.mark.parametrize("kind,k", [("2d", 6), ("2d", 17), ("2d", 64), ("3d", 4), ("3d", 7),
                                    ("3d", 20)])
def test_grid_band_fills_its_envelope(kind, k):
    """Rows past the first b = k (2D) or k^2 (3D) fill their whole envelope [i - b, i + b]
    (per-row counts from tests/closed_forms.py, pinned to the oracle elsewhere), so the bound
    exceeds nnz only by the first rows' missing fill."""
    rp, ci = gen.lap2d(k) if kind == "2d" else gen.lap3d(k)
    nnz = pins.nnz_2d(k) if kind == "2d" else pins.nnz_3d(k)
    b = k if kind == "2d" else k * k
    lo, hi = envelope(rp, ci)
    n = len(rp) - 1
    cnt = np.asarray(closed_forms.counts(kind, k))
    assert int(cnt.sum()) == nnz
    assert np.array_equal((hi - lo + 1)[b:], cnt[b:])
    assert nnz <= bound(rp, ci) <= nnz * (1 + 2.0 / k)


def test_hub_last_loosens_the_bound():
    rp, ci = gen.circuit(24, 1)   # hubs ordered last widen every later row's U envelope
    assert bound(rp, ci) > 2 * int(oracle.fill2(rp, ci, emit=False)["counts"].sum())


@pytest.mark.gpu
def test_library_bound_matches():
    import torch
    lu = pytest.importorskip("paper_conf_ppopp_xia0ar23_b200")
    d = torch.device("cuda", torch.cuda.current_device())
    for rp, ci in CASES + [gen.config(2)[1:], gen.config(3)[1:], gen.lap2d(1024)]:
        h = lu.Symbolic(torch.from_numpy(rp).to(d), torch.from_numpy(ci).to(d))
        assert h.nnz_bound() == bound(rp, ci)
        h.close()


@pytest.mark.gpu
def test_run_host_with_bound_capacity():
    """The e2e protocol of bench.py: outputs allocated from the bound, one lu_sym_run_host call
    streaming the pattern to pinned host memory; bit-exact against the oracle."""
    import torch
    lu = pytest.importorskip("paper_conf_ppopp_xia0ar23_b200")
    d = torch.device("cuda", torch.cuda.current_device())
    for rp, ci in [gen.lap2d(40), gen.lap3d(9), gen.circuit(32, 2),
                   gen.random_pattern(900, 2.5, seed=5)]:
        ref = oracle.fill2(rp, ci)
        n = len(rp) - 1
        h = lu.Symbolic(torch.from_numpy(rp).to(d), torch.from_numpy(ci).to(d))
        cap = h.nnz_bound()
        assert cap >= int(ref["row_ptr"][-1])
        hrp = torch.empty(n + 1, dtype=torch.int64, pin_memory=True)
        hci = torch.empty(cap, dtype=torch.int32, pin_memory=True)
        fc, rp_lu, ci_lu = h.run_host(cap, hrp, hci)
        nz = int(ci_lu.numel())
        assert np.array_equal(hrp.numpy(), ref["row_ptr"])
        assert np.array_equal(hci.numpy()[:nz], ref["col_idx"])
        assert np.array_equal(fc.cpu().numpy(), ref["counts"])
        h.close()


@pytest.mark.gpu
def test_bound_degenerate():
    import torch
    lu = pytest.importorskip("paper_conf_ppopp_xia0ar23_b200")
    d = torch.device("cuda", torch.cuda.current_device())
    # n = 0, and rows with no entries at all (no diagonal)
    for rp, ci in [(np.zeros(1, np.int64), np.zeros(0, np.int32)),
                   (np.array([0, 0, 1, 1], np.int64), np.array([0], np.int32))]:
        h = lu.Symbolic(torch.from_numpy(rp).to(d), torch.from_numpy(ci).to(d))
        assert h.nnz_bound() == bound(rp, ci)
        h.close()
