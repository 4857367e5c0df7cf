"""GPU parity: the CUDA path (through the C ABI) vs the CPU oracle, element by element.

Bar: the pattern is a set emitted sorted and levels are unique, so counts,
row_ptr, col_idx and level must be bit-exact.
"""
import numpy as np
import pytest
import torch

import oracle
from inputs import gen
from tests import pins

pytestmark = pytest.mark.gpu

lu = pytest.importorskip("paper_conf_ppopp_xia0ar23_b200")


def dev():
    return torch.device("cuda", torch.cuda.current_device())


def gpu_run(rp, ci, rules=("u", "glu3"), **opts):
    d = dev()
    h = lu.Symbolic(torch.from_numpy(rp).to(d), torch.from_numpy(ci).to(d), **opts)
    fc, rp_lu, ci_lu = h.run()
    levels = {}
    for r in rules:
        lv, nl = h.levelize(rp_lu, ci_lu, r)
        levels[r] = (lv.cpu().numpy(), nl)
    out = dict(counts=fc.cpu().numpy(), row_ptr=rp_lu.cpu().numpy(), col_idx=ci_lu.cpu().numpy(),
               levels=levels, stats=h.stats())
    h.close()
    return out


def assert_same(g, ref, rules=("u", "glu3"), tag=""):
    assert np.array_equal(g["counts"], ref["counts"]), f"{tag}: counts differ"
    assert np.array_equal(g["row_ptr"], ref["row_ptr"]), f"{tag}: row_ptr differs"
    assert np.array_equal(g["col_idx"], ref["col_idx"]), f"{tag}: col_idx differs"
    for r in rules:
        lv, nl = oracle.levels(ref["row_ptr"], ref["col_idx"], r)
        assert np.array_equal(g["levels"][r][0], lv), f"{tag}: levels ({r}) differ"
        assert g["levels"][r][1] == nl, f"{tag}: num_levels ({r})"


def check(rp, ci, tag="", rules=("u", "glu3"), **opts):
    ref = oracle.fill2(rp, ci)
    g = gpu_run(rp, ci, rules=rules, **opts)
    assert_same(g, ref, rules, tag)
    return g


# ---------------------------------------------------------------- many small random cases
def test_random_tiny_zero_free_diag():
    rng = np.random.default_rng(2024)
    for case in range(150):
        n = int(rng.integers(1, 200))
        rp, ci = gen.random_pattern(n, float(rng.uniform(0.3, 4)), seed=50_000 + case,
                                    sym_frac=float(rng.uniform(0, 1)))
        check(rp, ci, f"case {case}")


def test_random_with_zero_diagonals():
    for case in range(60):
        n = 5 + 13 * case % 300
        rp, ci = gen.random_pattern(n, 2.2, seed=60_000 + case, zero_free_diag=False)
        check(rp, ci, f"zd case {case}")


def test_random_medium_heavy_rows():
    # a few dense rows/columns exercise the warp-cooperative heavy-vertex path (degree > W)
    for case in range(8):
        n = 3000
        rng = np.random.default_rng(case)
        rp, ci = gen.random_pattern(n, 1.5, seed=70_000 + case)
        R = [np.repeat(np.arange(n), np.diff(rp))]
        C = [ci.astype(np.int64)]
        for hub in rng.choice(n, 6, replace=False):
            nb = rng.choice(n, 400, replace=False)
            R += [np.full(nb.size, hub), nb]
            C += [nb, np.full(nb.size, hub)]
        rp2, ci2 = gen.csr_from_edges(n, np.concatenate(R), np.concatenate(C))
        check(rp2, ci2, f"hub case {case}")


# ---------------------------------------------------------------- structured inputs
@pytest.mark.parametrize("k", [2, 3, 5, 8, 16, 64])
def test_lap2d(k):
    g = check(*gen.lap2d(k), tag=f"lap2d {k}")
    assert int(g["row_ptr"][-1]) == pins.nnz_2d(k)


@pytest.mark.parametrize("k", [2, 3, 4, 7, 12])
def test_lap3d(k):
    g = check(*gen.lap3d(k), tag=f"lap3d {k}")
    assert int(g["row_ptr"][-1]) == pins.nnz_3d(k)


@pytest.mark.parametrize("s", [16, 32, 64, 128])
def test_circuit(s):
    check(*gen.circuit(s, 1), tag=f"circuit {s}")


def test_special_matrices():
    for n in (1, 2, 3, 12, 100, 1000):
        for name, fn in (("tridiag", gen.tridiag), ("arrow_first", gen.arrow_first),
                         ("arrow_last", gen.arrow_last), ("diag", gen.diag_only)):
            check(*fn(n), tag=f"{name} {n}")
        for b in (1, 3, 9):
            check(*gen.band(n, b), tag=f"band {n} {b}")
    # empty rows / no diagonal at all
    rp = np.zeros(6, np.int64)
    ci = np.zeros(0, np.int32)
    check(rp, ci, tag="empty")
    rp, ci = gen.csr_from_edges(5, [4, 3, 1], [0, 2, 3])
    check(rp, ci, tag="no-diagonal")


def test_fig1_fixture():
    import os
    A, fills, table = pins.read_fig1_golden(
        os.path.join(os.path.dirname(__file__), "golden", "fig1_fixture.txt"))
    R = [r for r, cs in A.items() for _ in cs]
    C = [c for r, cs in A.items() for c in cs]
    rp, ci = gen.csr_from_edges(10, R, C)
    g = check(rp, ci, tag="fig1")
    lv, nl = g["levels"]["u"]
    assert nl == 5 and {j: int(lv[j]) for j in range(10)} == table


# ---------------------------------------------------------------- planner / schedule knobs
KNOBS = [
    dict(flags=lu.F_NO_BATCH),                       # one threshold at a time (Alg. 1 order)
    dict(flags=lu.F_GLOBAL_BITMAP),                  # visited bitmaps in HBM slots
    dict(flags=lu.F_ASCENDING),
    dict(queue_capacity=32),                         # forces frontier spills to HBM
    dict(rows_in_flight=1), dict(rows_in_flight=3), dict(rows_in_flight=17),
    dict(threads_per_row=128), dict(threads_per_row=512), dict(threads_per_row=1024),
    dict(threads_per_row=1025),                      # 1024 threads, one-CTA-per-SM registers
    dict(threads_per_row=1025, queue_capacity=32, flags=lu.F_FORCE_CLASSES),
    # bfs_async (warp rings + CTA pool, no level barriers) and the level-synchronous BFS on
    # the one-CTA-per-SM kernel; 2048-entry queues give 64-entry rings: constant donations
    dict(threads_per_row=1025, flags=lu.F_NO_ASYNC_BFS),
    dict(threads_per_row=1025, flags=lu.F_ASYNC_BFS, queue_capacity=2048),
    dict(threads_per_row=1025, flags=lu.F_ASYNC_BFS | lu.F_GLOBAL_BITMAP),
    dict(threads_per_row=1025, flags=lu.F_ASYNC_BFS | lu.F_FORCE_CLASSES, queue_capacity=2048),
    dict(threads_per_row=1025, flags=lu.F_ASYNC_BFS | lu.F_TWO_PASS, ell_width=4),
    dict(threads_per_row=1025, flags=lu.F_ASYNC_BFS | lu.F_NO_BATCH),
    dict(ell_width=4), dict(ell_width=6), dict(ell_width=8),
    dict(flags=lu.F_GLOBAL_BITMAP, queue_capacity=32, rows_in_flight=5),
    dict(flags=lu.F_NO_PRUNE), dict(flags=lu.F_KAHN_WIDE_ONLY), dict(flags=lu.F_NO_CONTRACT),
    dict(flags=lu.F_NO_CONTRACT | lu.F_NO_PRUNE | lu.F_KAHN_WIDE_ONLY),
    dict(flags=lu.F_TWO_PASS),                       # Alg. 3 as printed: emit re-traverses
    dict(flags=lu.F_TWO_PASS, queue_capacity=64),
    dict(flags=lu.F_ONE_CLASS), dict(flags=lu.F_ONE_CLASS | lu.F_GLOBAL_BITMAP),
    dict(flags=lu.F_FORCE_CLASSES), dict(flags=lu.F_FORCE_CLASSES | lu.F_GLOBAL_BITMAP),
    dict(flags=lu.F_FORCE_CLASSES, queue_capacity=32, rows_in_flight=7),
    dict(pool_bytes=4096),                           # pool overflow: most rows re-traversed
    dict(pool_bytes=200_000),                        # partial staging
    dict(flags=lu.F_SELF_CONT),                      # BFS self-continuation in every class
    dict(flags=lu.F_SELF_CONT, queue_capacity=32),   # ... with frontier spills
    dict(flags=lu.F_SELF_CONT | lu.F_GLOBAL_BITMAP | lu.F_FORCE_CLASSES),
    dict(flags=lu.F_SELF_CONT | lu.F_TWO_PASS, threads_per_row=1024),
    dict(flags=lu.F_NO_SELF_CONT, threads_per_row=1024, rows_in_flight=148),
    # Alg. 3 / Alg. 4 launch scheme: chunk_size = L/(6n) rows per launch (several chunks here)
    dict(flags=lu.F_PAPER_CHUNKS, scratch_budget_bytes=2_000_000),
    dict(flags=lu.F_PAPER_CHUNKS | lu.F_ONE_CLASS, scratch_budget_bytes=1_000_000),
    dict(flags=lu.F_PAPER_CHUNKS | lu.F_FORCE_CLASSES | lu.F_TWO_PASS, scratch_budget_bytes=3_000_000),
    # unified-memory variant: scratch from cudaMallocManaged, +- prefetch
    dict(flags=lu.F_MANAGED), dict(flags=lu.F_MANAGED_PREFETCH),
    dict(flags=lu.F_MANAGED | lu.F_GLOBAL_BITMAP | lu.F_FORCE_CLASSES),
    dict(flags=lu.F_MANAGED | lu.F_TWO_PASS, pool_bytes=200_000),
]


@pytest.mark.parametrize("knob", KNOBS, ids=[str(k) for k in KNOBS])
def test_knobs_do_not_change_results(knob):
    for rp, ci in (gen.lap3d(9), gen.circuit(40, 2), gen.random_pattern(700, 2.5, seed=9),
                   gen.lap2d(20)):
        check(rp, ci, tag=str(knob), **knob)


def test_pool_overflow_falls_back_to_traversal():
    g = check(*gen.circuit(64, 5), tag="pool", pool_bytes=64_000)
    assert 0 < g["stats"]["rows_retraversed"] < 4096
    g = check(*gen.circuit(64, 5), tag="pool-full")
    assert g["stats"]["rows_retraversed"] == 0 and g["stats"]["pool_bytes"] > 0


def test_row_classes():
    """Alg. 4 row classes (split visited map: low words shared, high words in HBM) on inputs
    large enough for several classes; bit-exact against the oracle."""
    for rp, ci in (gen.circuit(128, 3), gen.lap3d(20), gen.random_pattern(30000, 2.0, seed=11)):
        g = check(rp, ci, tag="classes", flags=lu.F_FORCE_CLASSES)
        assert g["stats"]["row_classes"] >= 3
        g = check(rp, ci, tag="classes+two-pass", flags=lu.F_FORCE_CLASSES | lu.F_TWO_PASS)


def test_level_schedule():
    """Fig. 1(d) form: columns grouped by level, ascending within each level."""
    import os
    A, fills, table = pins.read_fig1_golden(
        os.path.join(os.path.dirname(__file__), "golden", "fig1_fixture.txt"))
    R = [r for r, cs in A.items() for _ in cs]
    C = [c for r, cs in A.items() for c in cs]
    cases = [gen.csr_from_edges(10, R, C), gen.circuit(48, 2), gen.lap2d(12),
             gen.random_pattern(500, 2.0, seed=3)]
    d = dev()
    for k, (rp, ci) in enumerate(cases):
        h = lu.Symbolic(torch.from_numpy(rp).to(d), torch.from_numpy(ci).to(d))
        fc, rp_lu, ci_lu = h.run()
        lv, nl = h.levelize(rp_lu, ci_lu, "u")
        ptr, cols = lu.level_schedule(lv, nl)
        ptr, cols, lvh = ptr.cpu().numpy(), cols.cpu().numpy(), lv.cpu().numpy()
        assert ptr[0] == 0 and ptr[-1] == len(rp) - 1 and np.all(np.diff(ptr) > 0)
        for l in range(nl):
            seg = cols[ptr[l]:ptr[l + 1]]
            assert np.array_equal(seg, np.sort(np.nonzero(lvh == l)[0]))
        if k == 0:   # the printed table, 1-based in the paper
            got = {l: (cols[ptr[l]:ptr[l + 1]] + 1).tolist() for l in range(nl)}
            assert got == {0: [1, 2, 3, 6, 7], 1: [4, 5], 2: [8], 3: [9], 4: [10]}
        h.close()


def test_spills_are_exercised():
    g = check(*gen.lap3d(12), tag="spill", queue_capacity=32)
    assert g["stats"]["spills"] > 0


def test_repeated_runs_same_handle():
    """R25: stamps/bitmaps must not leak between passes or runs on the same handle."""
    rp, ci = gen.circuit(48, 3)
    ref = oracle.fill2(rp, ci)
    d = dev()
    h = lu.Symbolic(torch.from_numpy(rp).to(d), torch.from_numpy(ci).to(d), rows_in_flight=4)
    for _ in range(3):
        fc, rp_lu, ci_lu = h.run()
        assert np.array_equal(fc.cpu().numpy(), ref["counts"])
        assert np.array_equal(ci_lu.cpu().numpy(), ref["col_idx"])
    h.close()


def test_row_ranges():
    rp, ci = gen.circuit(40, 4)
    n = len(rp) - 1
    ref = oracle.fill2(rp, ci)
    d = dev()
    h = lu.Symbolic(torch.from_numpy(rp).to(d), torch.from_numpy(ci).to(d))
    fc = torch.full((n,), -7, dtype=torch.int32, device=d)
    h.count(100, 900, fc)
    got = fc.cpu().numpy()
    assert np.array_equal(got[100:900], ref["counts"][100:900])
    assert np.all(got[:100] == -7) and np.all(got[900:] == -7)
    # pieces assembled from disjoint ranges == the full result (the multi-GPU path's contract)
    fc = torch.zeros(n, dtype=torch.int32, device=d)
    bounds = lu.partition_rows(lu.row_cost_upper_bound(rp), 3)
    for r in range(3):
        h.count(int(bounds[r]), int(bounds[r + 1]), fc)
    rp_lu, nnz = h.scan(fc)
    ci_lu = torch.full((nnz,), -1, dtype=torch.int32, device=d)
    for r in (2, 0, 1):
        h.emit(rp_lu, ci_lu, int(bounds[r]), int(bounds[r + 1]))
    assert np.array_equal(ci_lu.cpu().numpy(), ref["col_idx"])
    h.close()


# ---------------------------------------------------------------- C-ABI error behaviour
def test_error_codes():
    d = dev()
    ok_rp, ok_ci = gen.lap2d(4)
    bad = []
    rp, ci = ok_rp.copy(), ok_ci.copy()
    ci[3], ci[4] = ci[4], ci[3]                      # unsorted row
    bad.append((rp, ci))
    rp, ci = ok_rp.copy(), ok_ci.copy()
    ci[1] = ci[0]                                    # duplicate
    bad.append((rp, ci))
    rp, ci = ok_rp.copy(), ok_ci.copy()
    ci[-1] = 99                                      # out of range
    bad.append((rp, ci))
    rp, ci = ok_rp.copy(), ok_ci.copy()
    rp[-1] += 1                                      # row_ptr[n] != nnz
    bad.append((rp, ci))
    rp, ci = ok_rp.copy(), ok_ci.copy()
    rp[5], rp[6] = rp[6], rp[5]                      # not monotone
    bad.append((rp, ci))
    for rp, ci in bad:
        with pytest.raises(lu.LuSymError) as e:
            lu.Symbolic(torch.from_numpy(rp).to(d), torch.from_numpy(ci).to(d))
        assert e.value.status == lu.LU_ERR_INPUT
    h = lu.Symbolic(torch.from_numpy(ok_rp).to(d), torch.from_numpy(ok_ci).to(d))
    fc = h.count()
    rp_lu = torch.zeros(17, dtype=torch.int64, device=d)
    with pytest.raises(lu.LuSymError) as e:
        h.emit(rp_lu, torch.zeros(10, dtype=torch.int32, device=d))
    assert e.value.status == lu.LU_ERR_STATE
    rp_lu, nnz = h.scan(fc)
    with pytest.raises(lu.LuSymError) as e:
        h.emit(rp_lu, torch.zeros(nnz - 1, dtype=torch.int32, device=d))
    assert e.value.status == lu.LU_ERR_CAPACITY
    with pytest.raises(lu.LuSymError) as e:
        h.count(3, 2)
    assert e.value.status == lu.LU_ERR_ARG
    with pytest.raises(lu.LuSymError) as e:
        lu.Symbolic(torch.from_numpy(ok_rp).to(d), torch.from_numpy(ok_ci).to(d),
                    threads_per_row=100)
    assert e.value.status == lu.LU_ERR_ARG
    with pytest.raises(lu.LuSymError) as e:
        lu.Symbolic(torch.from_numpy(ok_rp).to(d), torch.from_numpy(ok_ci).to(d),
                    scratch_budget_bytes=16)
    assert e.value.status == lu.LU_ERR_NOMEM
    h.close()


# ---------------------------------------------------------------- BASELINE configs
def test_cfg1_full():
    g = check(*gen.lap2d(64), tag="cfg1")
    assert int(g["row_ptr"][-1]) == 520_318
    assert g["levels"]["u"][1] == 4096


@pytest.mark.slow
def test_cfg2_full_bench_launch_config():
    """cfg2 (bench.py's N=1 workload) element by element against the full oracle."""
    rp, ci = gen.lap3d(40)
    ref = oracle.fill2(rp, ci)
    g = gpu_run(rp, ci, rules=("u",))
    assert int(g["row_ptr"][-1]) == pins.nnz_3d(40) == 199_868_878
    assert np.array_equal(g["counts"], ref["counts"])
    assert np.array_equal(g["row_ptr"], ref["row_ptr"])
    assert np.array_equal(g["col_idx"], ref["col_idx"])
    lv, nl = g["levels"]["u"]
    assert np.array_equal(lv, np.arange(64_000)) and nl == 64_000


@pytest.mark.slow
def test_cfg3_full():
    """cfg3 (circuit, n = 2^20, hubs last; rows deferred to the row-merge tail and the sparse
    planner class on by default): counts, row_ptr and col_idx of EVERY row against the full
    oracle, and both rules' levels of the GPU pattern against the oracle's Kahn."""
    rp, ci = gen.circuit(1024, 1)
    ref = oracle.fill2(rp, ci)
    g = gpu_run(rp, ci, rules=("u", "glu3"))
    assert np.array_equal(g["counts"], ref["counts"])
    assert np.array_equal(g["row_ptr"], ref["row_ptr"])
    assert np.array_equal(g["col_idx"], ref["col_idx"])
    assert g["stats"]["rows_deferred"] > 0          # the hubs went through the tail
    for r in ("u", "glu3"):
        lv, nl = oracle.levels(ref["row_ptr"], ref["col_idx"], r)
        assert np.array_equal(g["levels"][r][0], lv) and g["levels"][r][1] == nl


@pytest.mark.slow
@pytest.mark.parametrize("cfg", [4, 5])
def test_cfg45_closed_forms(cfg):
    """cfg4/cfg5 (2.1e9 entries): EVERY row (counts, row_ptr, col_idx) against the closed form,
    expanded on the device chunk by chunk (tests/closed_forms.py); sampled rows also against
    the oracle; levels == arange(n) (chains)."""
    from tests import closed_forms
    name, rp, ci = gen.config(cfg)
    n = len(rp) - 1
    k, kind = (1024, "2d") if cfg == 4 else (64, "3d")
    d = dev()
    h = lu.Symbolic(torch.from_numpy(rp).to(d), torch.from_numpy(ci).to(d))
    fc, rp_lu, ci_lu = h.run()
    nnz = pins.nnz_2d(k) if cfg == 4 else pins.nnz_3d(k)
    assert int(rp_lu[-1]) == nnz
    assert torch.equal(fc.to(torch.int64), closed_forms.counts(kind, k, torch, d))
    assert closed_forms.check_device(kind, k, rp_lu, ci_lu) == nnz
    rng = np.random.default_rng(cfg)
    rows = np.unique(np.concatenate([rng.choice(n, 64, replace=False), [0, 1, n - 2, n - 1]]))
    rpl = rp_lu.cpu().numpy()
    ref = oracle.fill2(rp, ci, rows=rows.astype(np.int32))
    for kk, i in enumerate(rows):
        got = ci_lu[int(rpl[i]):int(rpl[i + 1])].cpu().numpy()
        assert np.array_equal(got, ref["col_idx"][ref["row_ptr"][kk]:ref["row_ptr"][kk + 1]])
    lv, nl = h.levelize(rp_lu, ci_lu, "u")
    assert nl == n
    assert torch.equal(lv, torch.arange(n, dtype=torch.int32, device=d))
    h.close()


# ---------------------------------------------------------------- pipelined run to host memory
@pytest.mark.parametrize("nchunks,knob", [(0, {}), (1, {}), (3, {}), (17, {}), (64, {}),
                                          (5, dict(flags=lu.F_FORCE_CLASSES)),
                                          (4, dict(flags=lu.F_TWO_PASS)),
                                          (6, dict(pool_bytes=60_000)),
                                          (7, dict(queue_capacity=32, rows_in_flight=9)),
                                          (3, dict(flags=lu.F_MANAGED))])
def test_run_host_pipelined(nchunks, knob):
    """lu_sym_run_host: chunked count -> chained scan -> place -> D2H, bit-exact on the device
    and host copies, repeated on the same handle (fresh pool and scratch sets each call)."""
    d = dev()
    # a matrix whose last rows are hubs (degree > 64 x mean: the heavy-last chunk order)
    n = 3000
    rp0, ci0 = gen.random_pattern(n, 1.5, seed=70_001)
    R = [np.repeat(np.arange(n), np.diff(rp0))]
    C = [ci0.astype(np.int64)]
    for hub in range(n - 6, n):
        nb = np.random.default_rng(hub).choice(n, 900, replace=False)
        R += [np.full(nb.size, hub), nb]
        C += [nb, np.full(nb.size, hub)]
    hubs = gen.csr_from_edges(n, np.concatenate(R), np.concatenate(C))
    for rp, ci in (gen.lap3d(11), gen.circuit(48, 7), gen.random_pattern(900, 2.0, seed=5),
                   gen.lap2d(1), gen.random_pattern(40, 0.5, seed=1), hubs):
        ref = oracle.fill2(rp, ci)
        nnz = int(ref["row_ptr"][-1])
        h = lu.Symbolic(torch.from_numpy(rp).to(d), torch.from_numpy(ci).to(d), **knob)
        for rep in range(2):
            hr = torch.full((len(rp),), -7, dtype=torch.int64).pin_memory()
            hc = torch.full((nnz + 5,), -7, dtype=torch.int32).pin_memory()
            fc, rp_lu, ci_lu = h.run_host(nnz + 5, hr, hc, nchunks=nchunks)
            torch.cuda.synchronize()
            assert h.nnz_lu == nnz
            assert np.array_equal(fc.cpu().numpy(), ref["counts"])
            assert np.array_equal(rp_lu.cpu().numpy(), ref["row_ptr"])
            assert np.array_equal(ci_lu.cpu().numpy(), ref["col_idx"])
            assert np.array_equal(hr.numpy(), ref["row_ptr"])
            assert np.array_equal(hc.numpy()[:nnz], ref["col_idx"])
            lv, nl = h.levelize(rp_lu, ci_lu, "u")
            assert np.array_equal(lv.cpu().numpy(), oracle.levels(ref["row_ptr"],
                                                                  ref["col_idx"], "u")[0])
        h.close()


def test_run_host_capacity():
    d = dev()
    rp, ci = gen.lap3d(8)
    ref = oracle.fill2(rp, ci)
    nnz = int(ref["row_ptr"][-1])
    h = lu.Symbolic(torch.from_numpy(rp).to(d), torch.from_numpy(ci).to(d))
    with pytest.raises(lu.LuSymError) as e:
        h.run_host(nnz - 1, nchunks=4)
    assert e.value.status == lu.LU_ERR_CAPACITY
    fc, rp_lu, ci_lu = h.run_host(nnz, nchunks=4)   # the handle stays usable
    assert np.array_equal(ci_lu.cpu().numpy(), ref["col_idx"])
    h.close()


def test_level_types():
    """GLU3.0 level types (L208, reading R28) vs the oracle, several thresholds + defaults."""
    d = dev()
    sms = torch.cuda.get_device_properties(d).multi_processor_count
    cases = [gen.circuit(48, 2), gen.lap2d(12), gen.lap3d(6), gen.random_pattern(500, 2.0, seed=3),
             gen.random_pattern(3000, 1.2, seed=8, sym_frac=0.3), gen.lap2d(1)]
    for rp, ci in cases:
        h = lu.Symbolic(torch.from_numpy(rp).to(d), torch.from_numpy(ci).to(d))
        fc, rp_lu, ci_lu = h.run()
        for rule in ("u", "glu3"):
            lv, nl = h.levelize(rp_lu, ci_lu, rule)
            rph, cih, lvh = rp_lu.cpu().numpy(), ci_lu.cpu().numpy(), lv.cpu().numpy()
            for mc, ms in ((1, 1), (2, 3), (16, 8), (0, 0), (1000, 32)):
                typ, sub = lu.level_types(rp_lu, ci_lu, lv, nl, mc, ms)
                t_ref, s_ref, _ = oracle.level_types(rph, cih, lvh, nl, mc if mc > 0 else sms,
                                                     ms if ms > 0 else 32)
                assert np.array_equal(typ.cpu().numpy(), t_ref), (rule, mc, ms)
                assert np.array_equal(sub.cpu().numpy(), s_ref), (rule, mc, ms)
        h.close()


def test_symbolic_distributed_single_rank():
    """The row-sharded entry point on one rank (no process group): replicated and local-rows
    outputs equal the oracle's."""
    d = dev()
    rp, ci = gen.circuit(40, 4)
    ref = oracle.fill2(rp, ci)
    args = (torch.from_numpy(rp).to(d), torch.from_numpy(ci).to(d))
    fc, rp_lu, ci_lu, lv, nl = lu.symbolic_distributed(*args)
    assert np.array_equal(ci_lu.cpu().numpy(), ref["col_idx"])
    lref, nref = oracle.levels(ref["row_ptr"], ref["col_idx"], "u")
    assert nl == nref and np.array_equal(lv.cpu().numpy(), lref)
    fc, rp_lu, ci_lu, lv, nl = lu.symbolic_distributed(*args, output="local_rows")
    assert lv is None and np.array_equal(ci_lu.cpu().numpy(), ref["col_idx"])


# ---------------------------------------------------------------- deferred rows (reading G8)
def _hub_matrix(n=3000, hubs=6, deg=900, seed=70_001):
    """Random pattern whose last rows are hubs (degree >> mean): the rows fill2 serialises on."""
    rp0, ci0 = gen.random_pattern(n, 1.5, seed=seed)
    R = [np.repeat(np.arange(n), np.diff(rp0))]
    C = [ci0.astype(np.int64)]
    for hub in range(n - hubs, n):
        nb = np.random.default_rng(hub).choice(n, deg, replace=False)
        R += [np.full(nb.size, hub), nb]
        C += [nb, np.full(nb.size, hub)]
    return gen.csr_from_edges(n, np.concatenate(R), np.concatenate(C))


DEFER_KNOBS = [
    dict(defer_windows=1),                          # nearly every row with a threshold defers
    dict(defer_windows=2, defer_max=5),             # the cap: the rest finish by traversal
    dict(defer_windows=1, defer_max=4096),
    dict(defer_windows=1, pool_bytes=300_000),      # pool too small: tail rows fail -> fill2
    dict(defer_windows=3, queue_capacity=32),       # tail frontiers spill to HBM
    dict(defer_windows=1, flags=lu.F_FORCE_CLASSES),
    dict(defer_windows=1, flags=lu.F_ASCENDING),
    dict(defer_windows=2, rows_in_flight=3),
]


@pytest.mark.parametrize("knob", DEFER_KNOBS, ids=[str(k) for k in DEFER_KNOBS])
def test_deferred_rows_row_merge_tail(knob):
    """Rows abandoned by fill2 and finished by the row-merge closure over staged rows are
    bit-exact; chains of deferred rows (a row waiting for a deferred row below it) included."""
    for rp, ci in (_hub_matrix(), gen.circuit(48, 3), gen.lap3d(9), gen.lap2d(24),
                   gen.random_pattern(900, 2.5, seed=12), gen.arrow_first(300)):
        g = check(rp, ci, tag=str(knob), **knob)
        st = g["stats"]
        if knob.get("defer_windows") == 1 and "pool_bytes" not in knob:
            assert st["rows_deferred"] > 0 or len(rp) < 400, st


@pytest.mark.parametrize("variant", [("LUSYM_MERGE_HBM_BITMAP", "1"), ("LUSYM_MERGE_CLUSTER", "1"),
                                     ("LUSYM_MERGE_CLUSTER", "2"), ("LUSYM_MERGE_CLUSTER", "4"),
                                     ("LUSYM_MERGE_CLUSTER", "16"),
                                     ("LUSYM_MERGE_GRID_MAX", "100000"),
                                     ("LUSYM_MERGE_GRID_HEAD", "0"),
                                     ("LUSYM_MERGE_GRID_HEAD", "7")], ids=str)
def test_deferred_rows_tail_variants(monkeypatch, variant):
    """The tail's bitmap placements: one CTA per row with an HBM slot or a shared-memory
    bitmap, and clusters of 2/8/16 CTAs with the bitmap sliced over distributed shared memory
    (the default is 8); and the grid-wide mode (k_merge_grid) for every list however long, for
    none of the rows, or for the first 7 (the default gives it the first 2)."""
    monkeypatch.setenv(*variant)
    for rp, ci in (_hub_matrix(), gen.circuit(40, 2), gen.lap2d(24)):
        for knob in (dict(defer_windows=1), dict(defer_windows=2, queue_capacity=32)):
            g = check(rp, ci, tag=f"merge {variant} {knob}", **knob)
            assert g["stats"]["rows_deferred"] > 0


def test_deferred_rows_stats_and_row_ranges():
    """The tail only runs when every row below is staged by the handle: a count over [0, n)
    defers, a count over an upper block alone does not; both are exact."""
    rp, ci = _hub_matrix(n=4000, hubs=8, deg=1500, seed=3)
    n = len(rp) - 1
    ref = oracle.fill2(rp, ci)
    d = dev()
    h = lu.Symbolic(torch.from_numpy(rp).to(d), torch.from_numpy(ci).to(d), defer_windows=2)
    fc = torch.zeros(n, dtype=torch.int32, device=d)
    h.count(2000, n, fc)                       # rows below 2000 are not staged: no deferral
    assert h.stats()["rows_deferred"] == 0
    assert np.array_equal(fc.cpu().numpy()[2000:], ref["counts"][2000:])
    fc = h.count()
    st = h.stats()
    assert st["rows_deferred"] > 0 and st["rows_merge_failed"] == 0
    assert st["merge_entries_read"] > 0 and st["ms_tail"] > 0
    assert np.array_equal(fc.cpu().numpy(), ref["counts"])
    rp_lu, nnz = h.scan(fc)
    ci_lu = h.emit(rp_lu)
    assert np.array_equal(ci_lu.cpu().numpy(), ref["col_idx"])
    assert h.stats()["rows_retraversed"] == 0
    # two calls covering [0, n) in increasing order: the second may defer
    h.count(0, 2000, fc)
    h.count(2000, n, fc)
    assert np.array_equal(fc.cpu().numpy(), ref["counts"])
    rp_lu, nnz = h.scan(fc)
    assert np.array_equal(h.emit(rp_lu).cpu().numpy(), ref["col_idx"])
    h.close()


@pytest.mark.parametrize("nchunks", [3, 8])
def test_deferred_rows_run_host(nchunks):
    d = dev()
    for rp, ci in (_hub_matrix(), gen.circuit(48, 5)):
        ref = oracle.fill2(rp, ci)
        nnz = int(ref["row_ptr"][-1])
        h = lu.Symbolic(torch.from_numpy(rp).to(d), torch.from_numpy(ci).to(d), defer_windows=1)
        for _ in range(2):
            hr = torch.full((len(rp),), -7, dtype=torch.int64).pin_memory()
            hc = torch.full((nnz,), -7, dtype=torch.int32).pin_memory()
            fc, rp_lu, ci_lu = h.run_host(nnz, hr, hc, nchunks=nchunks)
            torch.cuda.synchronize()
            assert np.array_equal(fc.cpu().numpy(), ref["counts"])
            assert np.array_equal(hr.numpy(), ref["row_ptr"])
            assert np.array_equal(hc.numpy(), ref["col_idx"])
        h.close()


@pytest.mark.parametrize("knob", [dict(), dict(defer_windows=1), dict(queue_capacity=0, rows_in_flight=5),
                                  dict(flags=lu.F_TWO_PASS)], ids=str)
def test_sparse_class_forced(monkeypatch, knob):
    """The planner's sparse class (reading G9: 64-thread CTAs at 32 rows per SM, visited words
    in an HBM slot) replacing every shared-memory class, forced on small inputs; bit-exact."""
    monkeypatch.setenv("LUSYM_FORCE_SPARSE", "1")
    for rp, ci in (gen.lap3d(9), gen.circuit(48, 2), _hub_matrix(), gen.lap2d(20),
                   gen.random_pattern(700, 2.5, seed=9)):
        g = check(rp, ci, tag=f"sparse {knob}", **knob)
        assert g["stats"]["visited_in_smem"] == 0
        assert g["stats"]["row_classes"] == 1
        assert g["stats"]["sample_mean_sv"] == 0.0


@pytest.mark.parametrize("budget", [2_500_000, 6_000_000, 40_000_000])
def test_scratch_budget_is_enforced(budget):
    """Every allocation of the handle (row classes running concurrently, the staging pool, the
    row-merge tail, lu_sym_run_host's extra scratch sets) stays within scratch_budget_bytes
    (ADVICE r1); results stay exact."""
    d = dev()
    for rp, ci in (gen.lap3d(20), gen.circuit(64, 2), _hub_matrix()):
        ref = oracle.fill2(rp, ci)
        nnz = int(ref["row_ptr"][-1])
        h = lu.Symbolic(torch.from_numpy(rp).to(d), torch.from_numpy(ci).to(d),
                        scratch_budget_bytes=budget, flags=lu.F_FORCE_CLASSES)
        fc, rp_lu, ci_lu = h.run()
        assert np.array_equal(ci_lu.cpu().numpy(), ref["col_idx"])
        hc = torch.empty(nnz, dtype=torch.int32).pin_memory()
        fc, rp_lu, ci_lu = h.run_host(nnz, None, hc, nchunks=4)
        torch.cuda.synchronize()
        assert np.array_equal(hc.numpy(), ref["col_idx"])
        st = h.stats()
        assert st["scratch_bytes"] <= budget, (budget, st["scratch_bytes"])
        h.close()


def test_smem_base_fallback(monkeypatch):
    """If a kernel's dynamic shared memory did not start at the base the shared-bitmap kernels
    assume, the planner falls back to the HBM-bitmap kernels (no trap); forced here."""
    monkeypatch.setenv("LUSYM_ASSUME_SMEM_BASE_MISMATCH", "1")
    for rp, ci in (gen.lap3d(9), gen.circuit(40, 2), _hub_matrix()):
        g = check(rp, ci, tag="smem-base-fallback")
        assert g["stats"]["visited_in_smem"] == 0


@pytest.mark.parametrize("defer_windows", [1, 3, 0])
def test_deferred_rows_across_shards(defer_windows):
    """Reading G8 across GPUs (F_DEFER_GLOBAL), two "ranks" simulated by two handles in one
    process: each counts its block deferring rows whose rows below live on the other handle,
    counts and flags are summed (all-reduce), the pattern of the other rows is assembled, then
    lu_sym_merge_deferred finishes the deferred rows on either handle; bit-exact."""
    d = dev()
    for rp, ci in (_hub_matrix(), _hub_matrix(n=4000, hubs=9, deg=1500, seed=3),
                   gen.circuit(48, 3), gen.lap3d(9)):
        ref = oracle.fill2(rp, ci)
        n = len(rp) - 1
        A = (torch.from_numpy(rp).to(d), torch.from_numpy(ci).to(d))
        hs = [lu.Symbolic(*A, flags=lu.F_DEFER_GLOBAL, defer_windows=defer_windows)
              for _ in range(2)]
        b = [0, n // 2, n]
        fc = torch.zeros(n, dtype=torch.int32, device=d)
        flags = torch.zeros(n, dtype=torch.int32, device=d)
        for r in range(2):
            part = torch.zeros(n, dtype=torch.int32, device=d)
            hs[r].count(b[r], b[r + 1], part)
            fc += part
            flags |= hs[r].deferred_flags()
        rp_lu, nnz = hs[0].scan(fc)
        hs[1].scan(fc)
        ci_lu = torch.zeros(nnz, dtype=torch.int32, device=d)
        for r in range(2):
            hs[r].emit(rp_lu, ci_lu, b[r], b[r + 1])
        if defer_windows:
            assert int(flags.sum()) > 0
        for r in (1, 0):       # either handle finishes the same rows identically
            fcr, rpr = fc.clone(), rp_lu.clone()
            nnz2 = hs[r].merge_deferred(flags, fcr, rpr, ci_lu)
            assert nnz2 == int(ref["row_ptr"][-1])
            out = hs[r].emit(rpr, torch.empty(nnz2, dtype=torch.int32, device=d))
            assert np.array_equal(fcr.cpu().numpy(), ref["counts"])
            assert np.array_equal(rpr.cpu().numpy(), ref["row_ptr"])
            assert np.array_equal(out.cpu().numpy(), ref["col_idx"])
        for h in hs:
            h.close()
        # the one-process form of the same protocol
        h = lu.Symbolic(*A, flags=lu.F_DEFER_GLOBAL, defer_windows=defer_windows)
        fc, rp_lu, ci_lu = lu.sharded_pass(h, 0, n, [0, n])
        assert np.array_equal(ci_lu.cpu().numpy(), ref["col_idx"])
        h.close()


@pytest.mark.parametrize("knob", [dict(), dict(flags=lu.F_NO_BATCH), dict(flags=lu.F_SELF_CONT),
                                  dict(flags=lu.F_GLOBAL_BITMAP), dict(flags=lu.F_FORCE_CLASSES),
                                  dict(queue_capacity=32), dict(threads_per_row=1024),
                                  dict(threads_per_row=1025, queue_capacity=2048)], ids=str)
def test_stats_are_the_methods_work_units(knob):
    """The library's own counters are the method's work (reading R24): scanned
    vertices (every threshold once + every BFS vertex) and, with F_COUNT_TE, traversed edges
    (seed row + every scanned vertex's row, diagonal included) equal the oracle's per-row TE /
    SV summed — checked with and without diagonals, heavy rows and the knobs that change the
    traversal's schedule."""
    d = dev()
    knob = dict(knob)
    flags = knob.pop("flags", 0) | lu.F_COUNT_TE | lu.F_NO_DEFER
    for rp, ci in (gen.lap3d(9), gen.lap2d(20), gen.circuit(40, 2), _hub_matrix(),
                   gen.random_pattern(700, 2.5, seed=9),
                   gen.random_pattern(500, 2.2, seed=3, zero_free_diag=False)):
        ref = oracle.fill2(rp, ci, emit=False)
        h = lu.Symbolic(torch.from_numpy(rp).to(d), torch.from_numpy(ci).to(d), flags=flags,
                        **knob)
        fc = h.count()
        st = h.stats()
        assert np.array_equal(fc.cpu().numpy(), ref["counts"])
        assert st["vertices_scanned_count"] == int(ref["sv"].sum()), (knob, st)
        assert st["edges_read_count"] == int(ref["te"].sum()), (knob, st)
        h.close()
