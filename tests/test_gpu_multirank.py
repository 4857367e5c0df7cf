"""S7 / SURVEY 8(e) on the GPU: the row-sharded path (symbolic_distributed: partition, count of
the own rows, all-reduce of the counts, scan, emit of the own rows, all-gather of the pattern,
replicated levels) with 2 and 3 ranks sharing cuda:0 over gloo, every rank's result compared
bit-exactly with the oracle.  Also the measured-cost partition (cycles of a profiled pass).
These ranks share one GPU, so nothing here is a performance number."""
import os
import socket

import numpy as np
import pytest

pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _hubs(n=3000, hubs=6, deg=900):
    from inputs import gen
    rp0, ci0 = gen.random_pattern(n, 1.5, seed=70_001)
    R = [np.repeat(np.arange(n), np.diff(rp0))]
    C = [ci0.astype(np.int64)]
    for hub in range(n - hubs, n):
        nb = np.random.default_rng(hub).choice(n, deg, replace=False)
        R += [np.full(nb.size, hub), nb]
        C += [nb, np.full(nb.size, hub)]
    return gen.csr_from_edges(n, np.concatenate(R), np.concatenate(C))


def _worker(rank, world, port, q):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import torch
    import torch.distributed as dist
    import oracle
    import paper_conf_ppopp_xia0ar23_b200 as lu
    from inputs import gen
    try:
        torch.cuda.set_device(0)
        dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank,
                                world_size=world)
        d = torch.device("cuda", 0)
        out = []
        for name, (rp, ci) in (("lap3d9", gen.lap3d(9)), ("circuit48", gen.circuit(48, 3)),
                               ("hubs", _hubs()), ("random", gen.random_pattern(800, 2.2, seed=4))):
            ref = oracle.fill2(rp, ci)
            args = (torch.from_numpy(rp).to(d), torch.from_numpy(ci).to(d))
            for rule in ("u", "glu3"):
                lref, nref = oracle.levels(ref["row_ptr"], ref["col_idx"], rule)
                # rows deferred on any rank (F_DEFER_GLOBAL, set for N > 1) are finished after
                # the pattern exchange; defer_windows=2 defers many rows
                fc, rp_lu, ci_lu, lv, nl = lu.symbolic_distributed(
                    *args, rule=rule, options=lu.Options(defer_windows=2 if rule == "u" else 0))
                ok = (np.array_equal(fc.cpu().numpy(), ref["counts"])
                      and np.array_equal(rp_lu.cpu().numpy(), ref["row_ptr"])
                      and np.array_equal(ci_lu.cpu().numpy(), ref["col_idx"])
                      and np.array_equal(lv.cpu().numpy(), lref) and nl == nref)
                out.append((name, rule, ok))
            # partition by measured per-row cycles, then the same path again
            h = lu.Symbolic(*args)
            cost = lu.measured_row_cost(h)
            fc, rp_lu, ci_lu, lv, nl = lu.symbolic_distributed(*args, handle=h, cost=cost)
            ok = (np.array_equal(ci_lu.cpu().numpy(), ref["col_idx"])
                  and np.array_equal(fc.cpu().numpy(), ref["counts"]))
            b = lu.partition_rows(cost, world)
            out.append((name, "measured", ok and b[0] == 0 and b[-1] == len(rp) - 1))
            # local rows only: this rank's block, no exchange of the pattern
            fc, rp_lu, ci_lu, lv, nl = lu.symbolic_distributed(*args, handle=h,
                                                               output="local_rows")
            bounds = lu.partition_rows(lu.row_cost_upper_bound(rp), world)
            a, e = int(ref["row_ptr"][bounds[rank]]), int(ref["row_ptr"][bounds[rank + 1]])
            out.append((name, "local", np.array_equal(ci_lu.cpu().numpy()[a:e],
                                                       ref["col_idx"][a:e]) and lv is None))
            h.close()
        q.put((rank, out))
        dist.destroy_process_group()
    except Exception as e:  # pragma: no cover
        import traceback
        q.put((rank, traceback.format_exc()))


@pytest.mark.parametrize("world", [2, 3])
def test_symbolic_distributed_ranks_share_cuda0(world):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=600) for _ in range(world)]
    for p in procs:
        p.join(timeout=120)
    for rank, out in res:
        assert isinstance(out, list), out
        bad = [x for x in out if not bool(x[2])]
        assert not bad, (rank, bad)
