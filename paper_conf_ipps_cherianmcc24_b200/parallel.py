"""Host-side plumbing for row-block sharding over torch.distributed.

Destination vertices are split into contiguous blocks holding ≈E/P in-edges each
(nnz-balanced on a snapshot's in-CSR row pointer); the forward aggregation of a
rank produces the rows of its block, which an all-gather assembles; the backward
aggregation of a rank over its local edges produces partial sums for every
source, which an all-reduce (or reduce-scatter to the owners) combines.  The
device-side partitioner is ``stg_partition_rows`` (same bounds, see the GPU
test); these helpers are the host logic and the collectives only — no compute.
"""
from __future__ import annotations

import numpy as np
import torch
import torch.distributed as dist


def row_blocks(rowptr: np.ndarray, world: int) -> list:
    """bounds[k] = first row r with rowptr[r] >= ceil(k·E/world); bounds[0]=0, bounds[world]=V."""
    rowptr = np.asarray(rowptr, dtype=np.int64)
    V = rowptr.size - 1
    E = int(rowptr[-1])
    b = [0]
    for k in range(1, world):
        target = (E * k + world - 1) // world
        b.append(int(np.searchsorted(rowptr[:V], target, side="left")))
    b.append(V)
    for k in range(1, world + 1):          # non-decreasing (empty blocks allowed)
        b[k] = max(b[k], b[k - 1])
    return b


def base_row_blocks(V: int, src0, dst0, world: int, self_loops: bool = True) -> list:
    """Row blocks of a graph given as an edge list (the DTDG base S_0 in bench.py): the
    in-degrees of the edge SET (duplicates removed, plus the self-loops the library adds
    with STG_SELF_LOOPS) -> row pointer -> row_blocks."""
    k = np.unique(np.asarray(src0, np.int64) * V + np.asarray(dst0, np.int64))
    s, d = k // V, k % V
    if self_loops:
        d = d[s != d]
    deg = np.bincount(d, minlength=V) + (1 if self_loops else 0)
    return row_blocks(np.concatenate([[0], np.cumsum(deg)]), world)


def local_in_csr(rowptr: np.ndarray, col: np.ndarray, lo: int, hi: int):
    """The in-CSR rows [lo, hi) of a snapshot (local row pointer, global column ids)."""
    rp = np.asarray(rowptr, dtype=np.int64)
    s, e = int(rp[lo]), int(rp[hi])
    return (rp[lo:hi + 1] - s).astype(np.int32), np.asarray(col[s:e], dtype=np.int32)


def local_out_csr(in_rowptr: np.ndarray, in_col: np.ndarray, V: int, lo: int, hi: int):
    """Out-CSR (rows = all sources) of the edges whose destination lies in [lo, hi)."""
    rp = np.asarray(in_rowptr, dtype=np.int64)
    dst = np.repeat(np.arange(lo, hi), np.diff(rp[lo:hi + 1]))
    src = np.asarray(in_col[rp[lo]:rp[hi]], dtype=np.int64)
    order = np.lexsort((dst, src))
    src, dst = src[order], dst[order]
    out_rowptr = np.zeros(V + 1, np.int64)
    np.add.at(out_rowptr, src + 1, 1)
    return np.cumsum(out_rowptr).astype(np.int32), dst.astype(np.int32)


def allgather_rows(local: torch.Tensor, bounds: list, group=None) -> torch.Tensor:
    """Concatenate every rank's row block (variable sizes) on every rank."""
    world = len(bounds) - 1
    sizes = [bounds[k + 1] - bounds[k] for k in range(world)]
    m = max(sizes) if sizes else 0
    pad = torch.zeros((m,) + tuple(local.shape[1:]), dtype=local.dtype, device=local.device)
    pad[: local.shape[0]] = local
    bufs = [torch.empty_like(pad) for _ in range(world)]
    dist.all_gather(bufs, pad, group=group)
    return torch.cat([bufs[k][: sizes[k]] for k in range(world)], dim=0)


def allreduce_sum_(t: torch.Tensor, group=None) -> torch.Tensor:
    dist.all_reduce(t, op=dist.ReduceOp.SUM, group=group)
    return t
