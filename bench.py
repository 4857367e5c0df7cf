#!/usr/bin/env python
"""Benchmark of the symbolic LU hot path (fill2 count -> scan -> allocate -> fill2 emit ->
levelize) on synthetic BASELINE.json workloads.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config C] [--impl ours|reference]

One step = one pass of the whole hot path (SURVEY §8(a) S1-S9 minus the create-time S1/S2,
which are timed in the e2e number) over the workload, inputs resident in HBM.  For N > 1 the
script runs under torchrun, one rank per GPU, rows sharded (strong scaling of one matrix):
count own rows, all-reduce counts, scan, emit own rows, allgatherv the pattern, levelize.
Timed with CUDA events on the launching stream, K steps bracketed by barrier + synchronize,
max over ranks.  L2 is flushed (256 MiB write) between timed steps, outside the events.

Prints ONE JSON line (rank 0).  metric = fill entries/s = nnz(L+U) / step time.
--impl reference times the CPU oracle (the only reference this tier has), bounded samples.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

from inputs import gen  # noqa: E402

METRIC = "fill entries/s"
UNIT = "entries/s"
L2_FLUSH_BYTES = 256 << 20


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", type=int, default=2, help="BASELINE.json configs[C-1]")
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--rule", default="u", choices=["u", "glu3"])
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--e2e-mode", default="pipelined", choices=["pipelined", "plain"],
                    help="pipelined: lu_sym_run_host (pattern copied to the host behind the "
                         "traversal, 1 GPU); plain: count/scan/emit then copies")
    ap.add_argument("--e2e-chunks", type=int, default=0, help="lu_sym_run_host chunks (0 = the library default, 16)")
    ap.add_argument("--cpu-sample-stride", type=int, default=0,
                    help="oracle sample: every s-th row (0 = auto, ~10-30 s of CPU work)")
    ap.add_argument("--profile", action="store_true", help="short run for ncu (no extras)")
    ap.add_argument("--no-numeric", action="store_true",
                    help="skip the side measurement of the numeric phase (SURVEY 8(f4))")
    ap.add_argument("--flags", type=int, default=0, help="lu_sym_opts.flags (LU_F_*)")
    ap.add_argument("--threads-per-row", type=int, default=0)
    ap.add_argument("--queue-capacity", type=int, default=0)
    return ap.parse_args()


# --------------------------------------------------------------------------- work units
def work_units(rp, cfg=None):
    """Method work of one traversal (reading R24): TE traversed edges, SV
    scanned vertices.  Exact values per config come from tests/golden/work_units.json
    (scripts/work_units.py: oracle counts, or the pinned grid closed forms TE = sum
    row_ptr[i+1], SV = n(n-1)/2); without an entry the grid closed forms are used (upper
    bounds for other inputs)."""
    n = len(rp) - 1
    try:
        wu = json.load(open(os.path.join(ROOT, "tests", "golden", "work_units.json")))
        e = wu.get(f"cfg{cfg}")
        if e and e["n"] == n and e["nnz_a"] == int(rp[-1]):
            return int(e["te"]), int(e["sv"])
    except Exception:
        pass
    return int(rp[1:].sum()), n * (n - 1) // 2


def alg_bytes_per_pass(te, sv, n, nnz_lu, emit):
    """4 B per traversed edge + 1 bit visited test-and-set, 8 B offsets + 8 B
    queue push/pop per scanned vertex; per row 4 B count (count pass) or 8 B offset read and
    4 B per emitted entry (emit pass)."""
    b = 4 * te + te / 8 + 16 * sv
    if emit:
        b += 8 * (n + 1) + 4 * nnz_lu
    else:
        b += 4 * n
    return b


# --------------------------------------------------------------------------- clocks
REASONS = ["gpu_idle", "applications_clocks_setting", "sw_power_cap", "hw_slowdown",
           "sync_boost", "sw_thermal_slowdown", "hw_thermal_slowdown", "hw_power_brake_slowdown",
           "display_clock_setting"]


class ClockSampler:
    """SM clock + clock-event reasons sampled DURING the timed region: NVML in a thread every
    10 ms (nvidia-smi -lms as the fallback), so even a ~0.2 s region gets a dozen samples.
    Reason bits follow nvmlClocksEventReason* (the same bits nvidia-smi reports)."""

    PERIOD_S = 0.01

    def __init__(self, index):
        self.index = index
        self.samples = []  # (sm_mhz, max_mhz, reasons_bitmask, busy)
        self.proc = None
        self.stop = threading.Event()
        self.thread = None

    def __enter__(self):
        try:
            import pynvml
            pynvml.nvmlInit()
            hd = pynvml.nvmlDeviceGetHandleByIndex(self._nvml_index())
            self.thread = threading.Thread(target=self._nvml, args=(pynvml, hd), daemon=True)
            self.thread.start()
            return self
        except Exception:
            pass
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index),
                 "--query-gpu=clocks.sm,clocks.max.sm,clocks_event_reasons.active,"
                 "utilization.gpu", "--format=csv,noheader,nounits", "-lms", "100"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.thread = threading.Thread(target=self._read, daemon=True)
            self.thread.start()
        except Exception:
            self.proc = None
        return self

    def _nvml_index(self):
        # CUDA_VISIBLE_DEVICES may remap: take the physical index of the visible device
        ids = [v.strip() for v in os.environ.get("CUDA_VISIBLE_DEVICES", "").split(",")
               if v.strip()]
        if ids and self.index < len(ids) and ids[self.index].isdigit():
            return int(ids[self.index])
        return self.index

    def _nvml(self, pynvml, hd):
        mx = pynvml.nvmlDeviceGetMaxClockInfo(hd, pynvml.NVML_CLOCK_SM)
        while not self.stop.is_set():
            try:
                c = pynvml.nvmlDeviceGetClockInfo(hd, pynvml.NVML_CLOCK_SM)
                r = pynvml.nvmlDeviceGetCurrentClocksEventReasons(hd)
                self.samples.append((float(c), float(mx), int(r), not (r & 1)))
            except Exception:
                pass
            self.stop.wait(self.PERIOD_S)

    def _read(self):
        for line in self.proc.stdout:
            parts = [p.strip() for p in line.split(",")]
            try:
                r = int(parts[2], 16)
                self.samples.append((float(parts[0]), float(parts[1]), r,
                                     float(parts[3]) > 0 or not (r & 1)))
            except (ValueError, IndexError):
                continue

    def __exit__(self, *a):
        self.stop.set()
        if self.proc is not None:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()
        if self.thread is not None:
            self.thread.join(timeout=5)

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unavailable"]}
        sm, mx, reasons = [], None, set()
        for c, m, r, busy in self.samples:
            mx = m
            if busy:
                sm.append(c)
            for b, name in enumerate(REASONS):
                if r & (1 << b) and name != "gpu_idle":
                    reasons.add(name)
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": mx,
                "reasons": sorted(reasons), "samples": len(self.samples),
                "source": "nvml" if self.proc is None else "nvidia-smi"}


# --------------------------------------------------------------------------- CPU oracle
def cpu_oracle_sample(rp, ci, stride, rule="u", te_total=None, threads=None):
    """Time the oracle (as it stands) on every stride-th row (both passes, all host cores by
    default) and extrapolate the symbolic time by TE share (te_total: the exact per-config TE
    of tests/golden/work_units.json, else the grid closed form sum row_ptr[i+1])."""
    import oracle
    n = len(rp) - 1
    rows = np.arange(n - 1, -1, -stride, dtype=np.int32)
    threads = threads or os.cpu_count() or 1
    t0 = time.perf_counter()
    r = oracle.fill2(rp, ci, rows=rows, emit=True, threads=threads)
    t_sym = time.perf_counter() - t0
    if te_total is None:
        te_total = int(rp[1:].sum())
    te_sample = int(r["te"].sum())
    scale = te_total / max(te_sample, 1)
    t_sym_full = t_sym * scale
    return dict(rows=rows, t_sample=t_sym, t_sym_full=t_sym_full, threads=threads,
                entries_sample=int(r["counts"].sum()), te_sample=te_sample, scale=scale)


def cpu_one_core_rate(rp, ci, te_total, seconds=1.0):
    """the oracle on ONE thread over a row sample of about `seconds` of work ->
    traversed edges per second per core (both passes)."""
    stride = max(1, int(round(te_total / (3e8 * seconds))))
    s = cpu_oracle_sample(rp, ci, stride, te_total=te_total, threads=1)
    return {"te_per_s": 2 * s["te_sample"] / max(s["t_sample"], 1e-9), "rows": len(s["rows"]),
            "seconds": s["t_sample"]}


def cpu_levels_time(rp, ci, rule, nnz_hint=None):
    """Full-pattern oracle Kahn time (needs the full pattern: computed once, untimed)."""
    import oracle
    full = oracle.fill2(rp, ci, emit=True, threads=os.cpu_count() or 1)
    t0 = time.perf_counter()
    oracle.levels(full["row_ptr"], full["col_idx"], rule)
    return time.perf_counter() - t0, int(full["row_ptr"][-1])


def auto_stride(n, te_total):
    """Row stride of the oracle sample: about 10-30 s of CPU work on the box's host cores.
    The oracle visits ~6e8 TE/s per core over its two passes (count + emit)."""
    cores = os.cpu_count() or 1
    target = 6e8 * cores * 15.0 / 2
    return max(1, int(round(te_total / target)))


# --------------------------------------------------------------------------- reference arm
def numeric_side(reps=5, warmup=2):
    """Side measurement of the numeric phase (Alg. 2) on cfg1's pattern: not part of
    `value`.  lu_numeric_factor timed with CUDA events on the current stream (median of reps,
    after warm-up); the scatter of A's values is outside the events.  Latency-bound: one
    grid barrier per GLU3 level."""
    import numpy as np
    import torch
    import paper_conf_ppopp_xia0ar23_b200 as lu
    from inputs import gen
    d = torch.device("cuda", torch.cuda.current_device())
    rp, ci = gen.lap2d(64)
    val = gen.dominant_values(rp, ci, 1, dtype=np.float32)
    trp, tci, tv = (torch.from_numpy(x).to(d) for x in (rp, ci, val))
    h = lu.Symbolic(trp, tci)
    _, rp_lu, ci_lu = h.run()
    level, nl = lu.levelize(rp_lu, ci_lu, rule="glu3", handle=h)
    h.close()
    lptr, lcols = lu.level_schedule(level, nl)
    rph, cih = rp_lu.cpu().numpy(), ci_lu.cpu().numpy()
    n = len(rph) - 1
    row = np.repeat(np.arange(n), np.diff(rph))
    updates = int((np.bincount(cih[cih < row], minlength=n).astype(np.int64)
                   * np.bincount(row[cih > row], minlength=n)).sum())
    s = torch.cuda.current_stream()
    ts = []
    for r in range(warmup + reps):
        v = lu.numeric_scatter(trp, tci, tv, rp_lu, ci_lu)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        lu.numeric_factor(rp_lu, ci_lu, lptr, lcols, v)
        e1.record(s)
        torch.cuda.synchronize()
        if r >= warmup:
            ts.append(e0.elapsed_time(e1))
    ms = float(np.median(ts))
    return {"workload": "cfg1 lap2d_k64, numeric phase (Alg. 2, float), not in value",
            "ms": ms, "updates": updates, "gflops": 2 * updates / ms / 1e6,
            "levels_glu3": nl, "us_per_level": 1e3 * ms / max(nl, 1),
            "bound": "latency: one grid barrier per GLU3 level (DESIGN.md 6.1)",
            "parity": "tests/test_gpu_numeric.py vs oracle/numeric.py (float64)"}


def run_reference(args, rank, world):
    if rank != 0:
        return
    name, rp, ci = gen.config(args.config)
    n = len(rp) - 1
    te, _ = work_units(rp, args.config)
    stride = args.cpu_sample_stride or auto_stride(n, te)
    times, entries = [], None
    for k in range(args.warmup + args.steps):
        s = cpu_oracle_sample(rp, ci, stride, te_total=te)
        if k >= args.warmup:
            times.append(s["t_sym_full"])
        entries = s
    t_lev, nnz = cpu_levels_time(rp, ci, args.rule)
    t_step = float(np.mean(times)) + t_lev
    value = nnz / t_step
    out = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": t_step * 1e3,
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "int32",
        "data": "synthetic",
        "config": {"workload": f"cfg{args.config} {name}", "n": n, "nnz_a": int(rp[-1]),
                   "nnz_lu": nnz},
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": entries["threads"],
                         "kind": "oracle",
                         "sample": f"fill2 count+emit on every {stride}-th row "
                                   f"({len(entries['rows'])} rows, descending), extrapolated by "
                                   f"exact TE share x{entries['scale']:.2f}; Kahn on the full "
                                   f"pattern ({t_lev:.2f} s, 1 thread)"},
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(out), flush=True)


# --------------------------------------------------------------------------- our arm
def run_ours(args, rank, world, local_rank):
    import torch
    import torch.distributed as dist
    import paper_conf_ppopp_xia0ar23_b200 as lu

    dev = torch.device("cuda", local_rank)
    torch.cuda.set_device(dev)
    stream = torch.cuda.current_stream()
    name, rp_np, ci_np = gen.config(args.config)
    n = len(rp_np) - 1
    te, sv = work_units(rp_np, args.config)
    rp = torch.from_numpy(rp_np).to(dev)
    ci = torch.from_numpy(ci_np).to(dev)
    sym_opts = dict(flags=args.flags, threads_per_row=args.threads_per_row,
                    queue_capacity=args.queue_capacity)
    h = lu.Symbolic(rp, ci, **sym_opts)
    cost = lu.row_cost_upper_bound(rp_np)
    bounds = lu.partition_rows(cost, world)
    rb, re_ = int(bounds[rank]), int(bounds[rank + 1])
    flush = torch.empty(L2_FLUSH_BYTES // 4, dtype=torch.int32, device=dev)

    def barrier():
        if world > 1:
            dist.barrier()

    state = {}

    def step():
        state.clear()  # let the allocator reuse the previous step's output blocks
        fc = torch.zeros(n, dtype=torch.int32, device=dev)
        h.count(rb, re_, fc)                                     # S3 (symbolic_1)
        if world > 1:
            lu.assemble_counts(fc)                               # S7 (counts)
        rp_lu, nnz = h.scan(fc)                                  # S4
        ci_lu = torch.empty(nnz, dtype=torch.int32, device=dev)  # S5
        h.emit(rp_lu, ci_lu, rb, re_)                            # S6 (symbolic_2)
        if world > 1:
            lu.assemble_pattern(ci_lu, rp_lu, bounds)            # S7 (pattern)
        level, nl = h.levelize(rp_lu, ci_lu, args.rule)          # S8 + S9
        state.update(nnz=nnz, nl=nl, rp_lu=rp_lu, ci_lu=ci_lu, level=level, fc=fc)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    launches0 = h.stats()["kernel_launches"]
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
          for _ in range(args.steps)]
    k_ms = {"count": [], "scan": [], "emit": [], "levelize": []}
    barrier()
    torch.cuda.synchronize()
    with ClockSampler(local_rank) as clk:
        for k in range(args.steps):
            flush.fill_(k)                                   # L2 flush, outside the events
            ev[k][0].record(stream)
            step()
            ev[k][1].record(stream)
            st = h.stats()
            for key in k_ms:
                k_ms[key].append(st["ms_" + key])
        barrier()
        torch.cuda.synchronize()
    launches = h.stats()["kernel_launches"] - launches0
    step_ms = [a.elapsed_time(b) for a, b in ev]
    tot = torch.tensor([sum(step_ms)], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(tot, op=dist.ReduceOp.MAX)
    ms_per_step = float(tot.item()) / args.steps
    nnz = state["nnz"]
    value = nnz / (ms_per_step / 1e3)
    stats = h.stats()
    if args.profile:
        if rank == 0:
            print(json.dumps({"profile": True, "ms_per_step": ms_per_step, "stats": stats}))
        return

    # ---- roofline of the dominant kernel (fill2 traversal; events around its launch)
    avg = {k: float(np.mean(v)) for k, v in k_ms.items()}
    rows_mine = re_ - rb
    frac_rows = cost[rb:re_].sum() / max(cost.sum(), 1)
    te_mine, sv_mine = te * frac_rows, sv * frac_rows
    # the count pass runs the traversal and stages every row (staged mode), so its algorithmic
    # bytes are the traversal's plus the pattern it writes; emit is then a placement copy
    staged = stats["pool_bytes"] > 0
    b_count = alg_bytes_per_pass(te_mine, sv_mine, rows_mine, nnz * frac_rows, staged)
    b_emit = (8.0 * nnz * frac_rows + 8 * rows_mine) if staged else \
        alg_bytes_per_pass(te_mine, sv_mine, rows_mine, nnz * frac_rows, True)
    dom = "emit" if avg["emit"] >= avg["count"] else "count"
    b_dom = b_emit if dom == "emit" else b_count
    kname = {"count": "stage" if staged else "count", "emit": "place" if staged else "emit"}[dom]
    peaks = {}
    try:
        peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        pass
    peak = float(peaks.get("hbm_gbs", 6650.0))
    achieved = b_dom / (avg[dom] / 1e3) / 1e9
    traffic = None
    try:
        prof = json.load(open(os.path.join(ROOT, "profiles", "traffic.json")))
        traffic = prof.get(f"cfg{args.config}", {}).get(
            f"fill2_{kname}" if kname in ("stage", "count", "emit") else "k_place")
    except Exception:
        pass
    roofline = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                "frac": achieved / peak, "traffic": traffic,
                "kernel": f"fill2_kernel<{kname}>" if kname != "place" else "k_place",
                "peak_source": "MEASURED_PEAKS.json hbm_gbs" if peaks else "fallback",
                "alg_bytes_per_launch": b_dom, "ms_per_launch": avg[dom]}

    # ---- e2e through the public API with host buffers
    e2e = None
    if not args.no_e2e:
        rp_h = torch.from_numpy(rp_np).pin_memory()
        ci_h = torch.from_numpy(ci_np).pin_memory()
        out_rp = torch.empty(n + 1, dtype=torch.int64).pin_memory()
        out_ci = torch.empty(nnz, dtype=torch.int32).pin_memory()
        out_lv = torch.empty(n, dtype=torch.int32).pin_memory()
        e_ms = []
        e_phase = {}
        pipelined = args.e2e_mode == "pipelined" and world == 1
        for k in range(args.e2e_steps + 1):
            barrier()
            torch.cuda.synchronize()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            marks = []

            def mark(tag):
                ev_ = torch.cuda.Event(enable_timing=True)
                ev_.record(stream)
                marks.append((tag, ev_))

            a.record(stream)
            rpd = rp_h.to(dev, non_blocking=True)
            cid = ci_h.to(dev, non_blocking=True)
            mark("h2d")
            he = lu.Symbolic(rpd, cid, **sym_opts)             # S1 + S2 (validate, plan)
            mark("create")
            if pipelined:
                # S3-S6 with the pattern streamed to pinned host memory behind the traversal
                fc, rp_lu, ci_lu = he.run_host(nnz, out_rp, out_ci, nchunks=args.e2e_chunks)
                mark("count+scan+emit+d2h(pattern)")
                level, _ = he.levelize(rp_lu, ci_lu, args.rule)
                mark("levelize")
                out_lv.copy_(level, non_blocking=True)
            else:
                fc = torch.zeros(n, dtype=torch.int32, device=dev)
                he.count(rb, re_, fc)
                if world > 1:
                    lu.assemble_counts(fc)
                mark("count")
                rp_lu, nz = he.scan(fc)
                ci_lu = torch.empty(nz, dtype=torch.int32, device=dev)
                mark("scan+alloc")
                he.emit(rp_lu, ci_lu, rb, re_)
                if world > 1:
                    lu.assemble_pattern(ci_lu, rp_lu, bounds)
                mark("emit")
                level, _ = he.levelize(rp_lu, ci_lu, args.rule)
                mark("levelize")
                if rank == 0:
                    out_rp.copy_(rp_lu, non_blocking=True)
                    out_ci.copy_(ci_lu, non_blocking=True)
                    out_lv.copy_(level, non_blocking=True)
            b.record(stream)
            torch.cuda.synchronize()
            he.close()
            if k > 0:
                e_ms.append(a.elapsed_time(b))
                prev = a
                for tag, ev_ in marks + [("d2h", b)]:
                    e_phase.setdefault(tag, []).append(prev.elapsed_time(ev_))
                    prev = ev_
        t = torch.tensor([float(np.mean(e_ms))], dtype=torch.float64, device=dev)
        if world > 1:
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
        e2e = {"value": nnz / (float(t.item()) / 1e3), "unit": UNIT,
               "h2d_bytes_per_step": int(rp_np.nbytes + ci_np.nbytes),
               "d2h_bytes_per_step": int((n + 1) * 8 + nnz * 4 + n * 4) if rank == 0 else 0,
               "ms_per_step": float(t.item()),
               "phases_ms": {k: float(np.mean(v)) for k, v in e_phase.items()},
               "mode": "lu_sym_run_host (chunked count/scan/place, pattern D2H behind the "
                       "traversal)" if pipelined else "count, scan, alloc, emit, then copies",
               "includes": "H2D of A, create (validate+adjacency+plan), count, scan, alloc, "
                           "emit, levelize, D2H of row_ptr/col_idx/level"}

    if rank != 0:
        return
    cpu = None
    if world == 1 and not args.no_cpu_baseline:
        stride = args.cpu_sample_stride or auto_stride(n, te)
        s = cpu_oracle_sample(rp_np, ci_np, stride, te_total=te)
        one = cpu_one_core_rate(rp_np, ci_np, te)
        import oracle
        rpl = state["rp_lu"].cpu().numpy()
        cil = state["ci_lu"].cpu().numpy()
        t0 = time.perf_counter()
        oracle.levels(rpl, cil, args.rule)
        t_lev = time.perf_counter() - t0
        t_cpu = s["t_sym_full"] + t_lev
        cpu = {"value": nnz / t_cpu, "unit": UNIT, "cores": s["threads"], "kind": "oracle",
               "sample": f"fill2 count+emit on every {stride}-th row ({len(s['rows'])} rows) in "
                         f"{s['t_sample']:.2f} s, extrapolated by exact TE share "
                         f"x{s['scale']:.2f}; Kahn levels on the full pattern {t_lev:.2f} s "
                         f"(1 thread)",
               "one_core": {"traversed_edges_per_s": one["te_per_s"], "rows": one["rows"],
                            "note": "oracle on 1 thread, count+emit (2 traversals per row)"}}
    out = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "int32", "data": "synthetic",
        "config": {"workload": f"cfg{args.config} {name}", "n": n, "nnz_a": int(rp_np[-1]),
                   "nnz_lu": nnz, "num_levels": state["nl"], "rule": args.rule,
                   "parallelism": f"rows sharded over {world} GPU(s)" if world > 1 else "1 GPU",
                   "l2": "flushed between timed steps (256 MiB write, outside the events)"},
        "phases_ms": avg,
        "symbolic_s": (avg["count"] + avg["scan"] + avg["emit"]) / 1e3,
        "levelize_s": avg["levelize"] / 1e3,
        "teps": te / ((avg["count"] + avg["scan"] + avg["emit"]) / 1e3),
        "traversed_edges_per_pass": te, "scanned_vertices_per_pass": sv,
        "roofline": roofline,
        "cpu_baseline": cpu,
        "e2e": e2e,
        "gpu_launches": int(launches),
        "clocks": clk.summary(),
        "numeric": None if (world > 1 or args.no_numeric) else numeric_side(),
        "plan": {k: stats[k] for k in ("rows_in_flight", "threads_per_row", "smem_bytes_per_row",
                                        "visited_in_smem", "ell_width", "queue_capacity",
                                        "row_classes", "pool_bytes", "rows_retraversed",
                                        "levelize_wide_levels", "levelize_narrow_levels",
                                        "spills")},
    }
    print(json.dumps(out), flush=True)


def main():
    args = parse()
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    # test hook: run every rank on one GPU over gloo (exercises the N>1 path where only one GPU
    # exists); never used for a reported number
    if os.environ.get("LUSYM_BENCH_ONE_GPU"):
        local_rank = 0
    if args.impl == "reference":
        run_reference(args, rank, world)
        return
    if world > 1:
        import torch
        import torch.distributed as dist
        torch.cuda.set_device(local_rank)
        backend = os.environ.get("LUSYM_BENCH_BACKEND", "nccl")
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local_rank))
        else:
            dist.init_process_group(backend)
    try:
        run_ours(args, rank, world, local_rank)
    finally:
        if world > 1:
            import torch.distributed as dist
            dist.destroy_process_group()


if __name__ == "__main__":
    main()
