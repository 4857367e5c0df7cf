"""Row sharding of the symbolic factorization across the GPUs of one node.

PAPER.md L100: "symbolic factorization from each source row is independent", so the rows of A
are split into contiguous blocks, one per rank, with A replicated on every rank (it is <= 30 MB
on every config).  The exchange steps are real data dependencies of the path, not inventions:
  * the prefix sum of the per-row counts (Alg. 3 line 7, L262) needs every row's count
    -> all_reduce(SUM) of the count array (each row is non-zero on exactly one rank);
  * levelization (Alg. 5) needs the whole pattern -> one all-gather of the ranks' blocks of
    col_idx_lu, in place (an allgatherv over NVLink), after which each rank levelizes the
    identical pattern locally (the DAG is global and, on chains, strictly serial: "replicas
    only").
Blocks are balanced by a cost per row: the a-priori traversal bound row_ptr[i+1] (exact on the
grids), or the cycles each row took in a profiled pass of the same matrix (measured_row_cost),
which is what a repeated factorization of one pattern uses (circuit simulation re-factors the
same pattern many times).
torch.distributed supplies the communicator (NCCL on GPUs, gloo in the CPU tests).
"""
from __future__ import annotations

import numpy as np
import torch


def row_cost_upper_bound(row_ptr) -> np.ndarray:
    """Traversal cost bound of row i: |A(i,:)| + sum_{v<i} |A(v,:)| = row_ptr[i+1].

    fill2 reads the seed row plus the rows of scanned vertices, all of which are < i, each at
    most once (SURVEY reading R24); the bound is exact on connected natural-order grids."""
    rp = row_ptr.cpu().numpy() if isinstance(row_ptr, torch.Tensor) else np.asarray(row_ptr)
    return rp[1:].astype(np.float64)


def measured_row_cost(handle, row_begin: int = 0, row_end: int | None = None,
                      fill_count=None, group=None) -> np.ndarray:
    """Cycles each row of [row_begin, row_end) took in one profiled count pass on this rank
    (lu_sym_set_row_profile), summed over the ranks of `group` when distributed (disjoint
    rows), + 1 so that no row is free.  A cost for partition_rows."""
    import torch.distributed as dist
    n = handle.n
    row_end = n if row_end is None else row_end
    prof = torch.zeros(4 * n, dtype=torch.int64, device=handle.device)
    handle.set_row_profile(prof)
    try:
        handle.count(row_begin, row_end, fill_count)
    finally:
        handle.set_row_profile(None)
    if dist.is_initialized() and dist.get_world_size(group) > 1:
        _all_reduce(prof, group)
    return prof.view(n, 4)[:, 0].double().cpu().numpy() + 1.0


def partition_rows(cost, world: int) -> np.ndarray:
    """Contiguous row blocks with (nearly) equal total cost.  Returns bounds[world+1]."""
    cost = np.asarray(cost, dtype=np.float64)
    n = cost.size
    if world < 1:
        raise ValueError("world must be >= 1")
    pref = np.concatenate([[0.0], np.cumsum(cost)])
    total = pref[-1]
    bounds = np.zeros(world + 1, dtype=np.int64)
    for r in range(1, world):
        bounds[r] = int(np.searchsorted(pref, total * r / world, side="left"))
    bounds[world] = n
    bounds = np.maximum.accumulate(np.clip(bounds, 0, n))
    return bounds


def _device_collectives(t: torch.Tensor, group=None) -> bool:
    """NCCL handles device tensors directly; gloo (the CPU tests, and the one-GPU multi-rank
    test) gets host copies."""
    import torch.distributed as dist
    return not t.is_cuda or dist.get_backend(group) == "nccl"


def _all_reduce(t: torch.Tensor, group=None):
    import torch.distributed as dist
    if _device_collectives(t, group):
        dist.all_reduce(t, op=dist.ReduceOp.SUM, group=group)
    else:
        h = t.cpu()
        dist.all_reduce(h, op=dist.ReduceOp.SUM, group=group)
        t.copy_(h)
    return t


def assemble_counts(fill_count: torch.Tensor, group=None) -> torch.Tensor:
    """All ranks end with every row's count (disjoint supports -> SUM)."""
    return _all_reduce(fill_count, group)


def assemble_pattern(col_idx_lu: torch.Tensor, row_ptr_lu: torch.Tensor, bounds,
                     group=None) -> torch.Tensor:
    """In-place allgatherv of the per-rank column blocks of the L+U CSR: ONE all_gather call
    whose outputs are the ranks' slices of col_idx_lu itself (uneven sizes; NCCL runs it as one
    group of broadcasts).  gloo: the same call on padded host buffers."""
    import torch.distributed as dist
    world = len(bounds) - 1
    rank = dist.get_rank(group)
    idx = torch.as_tensor(np.asarray(bounds, dtype=np.int64), device=row_ptr_lu.device)
    offs = row_ptr_lu.index_select(0, idx).cpu().numpy()
    sizes = np.diff(offs)
    mx = max(int(sizes.max()), 1)
    if _device_collectives(col_idx_lu, group) and dist.get_backend(group) == "nccl":
        views = [col_idx_lu[int(offs[r]):int(offs[r + 1])] for r in range(world)]
        try:
            dist.all_gather(views, views[rank], group=group)
        except (RuntimeError, ValueError):
            # a torch without uneven all_gather: one padded all_gather_into_tensor on the device
            send = torch.zeros(mx, dtype=col_idx_lu.dtype, device=col_idx_lu.device)
            send[:sizes[rank]] = views[rank]
            recv = torch.empty(world * mx, dtype=col_idx_lu.dtype, device=col_idx_lu.device)
            dist.all_gather_into_tensor(recv, send, group=group)
            for r in range(world):
                if r != rank and sizes[r]:
                    views[r].copy_(recv[r * mx:r * mx + sizes[r]])
        return col_idx_lu
    send = torch.zeros(mx, dtype=col_idx_lu.dtype)
    send[:sizes[rank]] = col_idx_lu[int(offs[rank]):int(offs[rank + 1])].cpu()
    recv = [torch.empty(mx, dtype=col_idx_lu.dtype) for _ in range(world)]
    dist.all_gather(recv, send, group=group)
    for r in range(world):
        if r != rank and sizes[r]:
            col_idx_lu[int(offs[r]):int(offs[r + 1])].copy_(recv[r][:sizes[r]])
    return col_idx_lu
