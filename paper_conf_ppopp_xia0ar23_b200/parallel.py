"""Row sharding of the symbolic factorization across the GPUs of one node.

PAPER.md L100: "symbolic factorization from each source row is independent", so the rows of A
are split into contiguous blocks, one per rank, balanced by an a-priori cost bound, with A
replicated on every rank (it is <= 30 MB on every config).  The exchange steps are real data
dependencies of the path, not inventions:
  * the prefix sum of the per-row counts (Alg. 3 line 7, L262) needs every row's count
    -> all_reduce(SUM) of the count array (each row is non-zero on exactly one rank);
  * levelization (Alg. 5) needs the whole pattern -> every rank broadcasts its block of
    col_idx_lu (an allgatherv over NVLink), after which each rank levelizes the identical
    pattern locally (the DAG is global and, on chains, strictly serial: "replicas only").
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


def assemble_counts(fill_count: torch.Tensor, group=None) -> torch.Tensor:
    """All ranks end with every row's count (disjoint supports -> SUM)."""
    import torch.distributed as dist
    dist.all_reduce(fill_count, op=dist.ReduceOp.SUM, group=group)
    return fill_count


def assemble_pattern(col_idx_lu: torch.Tensor, row_ptr_lu: torch.Tensor, bounds,
                     group=None) -> torch.Tensor:
    """In-place allgatherv of the per-rank column blocks of the L+U CSR."""
    import torch.distributed as dist
    world = len(bounds) - 1
    idx = torch.as_tensor(np.asarray(bounds, dtype=np.int64), device=row_ptr_lu.device)
    offs = row_ptr_lu.index_select(0, idx).cpu().numpy()
    for r in range(world):
        a, b = int(offs[r]), int(offs[r + 1])
        if b <= a:
            continue
        src = r if group is None else dist.get_global_rank(group, r)
        dist.broadcast(col_idx_lu[a:b], src=src, group=group)
    return col_idx_lu
