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

import ctypes

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


# ---------------------------------------------------------------- sharded mode over peer memory
def stream_barrier(device=None):
    """Cross-rank ordering point for the peer buffers (include/stg.h): with NCCL a
    one-element all-reduce on the current stream (stream-ordered, no host sync);
    with gloo (CPU tests, ranks sharing one GPU) a device synchronize + barrier."""
    if dist.get_world_size() == 1:                # no peers: stream order suffices
        return
    if dist.get_backend() == "nccl":
        t = torch.zeros(1, device=device or torch.device("cuda", torch.cuda.current_device()))
        dist.all_reduce(t)
    else:
        torch.cuda.synchronize()
        dist.barrier()


class PeerGroup:
    """One IPC-shared fp32 row matrix over the ranks of the default process group:
    this rank's PeerBuffer ([rows, cols]; rows = its block, or V with full=True)
    plus every peer's buffer mapped into this process (stg_peer_open)."""

    def __init__(self, bounds, cols: int, full: bool = False):
        from paper_conf_ipps_cherianmcc24_b200 import PeerBuffer, PeerRows, stg_peer_open
        self.rank, self.world = dist.get_rank(), dist.get_world_size()
        self.bounds = list(bounds)
        rows = self.bounds[-1] if full else self.bounds[self.rank + 1] - self.bounds[self.rank]
        self.buf = PeerBuffer(rows, cols)
        handles = [None] * self.world
        dist.all_gather_object(handles, self.buf.handle_bytes())
        self._opened = []
        self.ptrs = []
        for k, h in enumerate(handles):
            if k == self.rank:
                self.ptrs.append(self.buf.ptr)
            else:
                p = stg_peer_open(h)
                self._opened.append(p)
                self.ptrs.append(p)
        self.rows = PeerRows(self.bounds, self.ptrs, cols)

    @property
    def tensor(self) -> torch.Tensor:
        return self.buf.tensor

    def close(self):
        from paper_conf_ipps_cherianmcc24_b200 import stg_peer_close
        for p in self._opened:
            stg_peer_close(p)
        self._opened = []
        self.buf.close()


class PeerTGCN:
    """Algorithm 1 for one rank in sharded mode: X is row-sharded,
    P' = diag(n_src)XW is computed for the local rows only and gathered from the
    owners inside the aggregation (stg_tgcn_step_peer); the backward's partial
    dP of the local edges is reduce-scattered to the owners over peer loads
    (stg_reduce_scatter_rows) before dW += X_locᵀ dP_loc.  Two buffers per
    exchanged matrix alternate per timestep.

    native=True (DTDG sources): the whole sequence runs in the library
    (stg_tgcn_train_sequence_peer) with the cross-rank ordering done by device-side
    counters in peer memory (stream wait / write operations) — no host barrier or
    collective per timestep.  native=False: the Python loop below, one stream
    barrier (a one-element NCCL all-reduce) per exchange."""

    def __init__(self, stg, bounds, V: int, F: int, H: int, S: int, native: bool = True):
        self.stg = stg
        self.bounds = list(bounds)
        self.rank = dist.get_rank()
        self.world = dist.get_world_size()
        self.V, self.F, self.H, self.S = V, F, H, S
        self.R = self.bounds[self.rank + 1] - self.bounds[self.rank]
        self.P = [PeerGroup(self.bounds, 3 * H) for _ in range(2)]
        self.dP = [PeerGroup(self.bounds, 3 * H, full=True) for _ in range(2)]
        self.dP_loc = torch.empty(max(self.R, 1), 3 * H, device="cuda")
        self.G = torch.empty(2, max(self.R, 1), H, device="cuda")
        self.stack = stg.stg_state_stack_create(S * max(self.R, 1) * 3 * H * 4 + (1 << 20))
        self.native = native
        if native:
            # every rank's 4 exchange counters (zero-initialised peer memory)
            self.flags = PeerGroup([0] + [1] * self.world, 4, full=True)
            px = stg.stg_peer_exchange()
            px.world, px.rank = self.world, self.rank
            self._bounds_c = (ctypes.c_int32 * (self.world + 1))(*self.bounds)
            px.bounds = self._bounds_c
            for b in range(2):
                for k in range(self.world):
                    px.P[b][k] = self.P[b].ptrs[k]
                    px.dP[b][k] = self.dP[b].ptrs[k]
            for k in range(self.world):
                px.flags[k] = self.flags.ptrs[k]
            self.px = px

    def train_sequence(self, source, t0, params, w_o, b_o, X_loc, Y_loc, H0, H_seq, grads, dw_o, db_o, loss,
                       barrier=stream_barrier):
        stg, S, R, H = self.stg, len(X_loc), self.R, self.H
        dyn = isinstance(source, stg.Dtdg)
        if self.native and dyn:
            stg.stg_tgcn_train_sequence_peer(source, t0, params, w_o, b_o, X_loc, Y_loc, H0, H_seq, self.G,
                                             self.dP_loc, grads, dw_o, db_o, loss, self.stack, self.px)
            return

        def view(t, backward):
            if not dyn:
                return source.view()
            part = stg.STG_PART_OUT if backward else stg.STG_PART_IN
            return stg.stg_dtdg_get_snapshot_parts(source, t, part, backward=backward)

        for i in range(S):                                     # forward, lines 7-16
            v = view(t0 + i, False)
            buf = self.P[i & 1]
            stg.stg_tgcn_project(v, params, X_loc[i], buf.buf.ptr)
            barrier()                                          # every owner's P' rows written
            Hp = H0 if i == 0 else H_seq[i - 1]
            stg.stg_tgcn_step_peer(v, params, buf.rows, Hp, H_seq[i], self.stack)
            stg.stg_mse_head(H_seq[i], Y_loc[i], w_o, b_o, loss_accum=loss, V_total=self.V)
        G, Gn = self.G[0][:R], self.G[1][:R]
        G.zero_()
        for i in range(S - 1, -1, -1):                         # backward, lines 18-25
            v = view(t0 + i, True)
            stg.stg_mse_head(H_seq[i], Y_loc[i], w_o, b_o, dH=G, accumulate=True, dw_o=dw_o, db_o=db_o,
                             V_total=self.V)
            dpg = self.dP[i & 1]
            stg.stg_tgcn_step_backward_peer(v, params, G, Gn, grads, dpg.buf.ptr, self.stack)
            barrier()                                          # every rank's partial dP written
            stg.stg_reduce_scatter_rows(self.bounds, dpg.ptrs, 3 * H, self.rank, 3 * H, self.dP_loc[:R])
            stg.stg_tgcn_dw(params, X_loc[i], self.dP_loc[:R], grads, self.stack)
            G, Gn = Gn, G

    def close(self):
        for g in self.P + self.dP:
            g.close()


class PeerTGCN2:
    """Algorithm 1 for one rank with the ORIGINAL T-GCN cell in sharded mode (NEXT-2):
    the gate and candidate convolutions gather rows that carry H from their owners,
    so hidden-state rows cross ranks every timestep (stg_tgcn2_peer_fwd / _bwd, one
    stream barrier between phases).  Buffers alternate by timestep as in PeerTGCN."""

    def __init__(self, stg, bounds, V: int, F: int, H: int, S: int):
        self.stg = stg
        self.bounds = list(bounds)
        self.rank = dist.get_rank()
        self.V, self.F, self.H = V, F, H
        self.R = self.bounds[self.rank + 1] - self.bounds[self.rank]
        self.Zg = [PeerGroup(self.bounds, 2 * H) for _ in range(2)]
        self.Zc = [PeerGroup(self.bounds, H) for _ in range(2)]
        self.Dc = [PeerGroup(self.bounds, H, full=True) for _ in range(2)]
        self.Dg = [PeerGroup(self.bounds, 2 * H, full=True) for _ in range(2)]
        self.G = torch.empty(2, max(self.R, 1), H, device="cuda")
        self.stack = stg.stg_state_stack_create(S * max(self.R, 1) * 3 * H * 4 + (1 << 20))

    def train_sequence(self, source, t0, params, w_o, b_o, X_loc, Y_loc, H0, H_seq, grads, dw_o, db_o, loss,
                       barrier=stream_barrier):
        stg, S, R = self.stg, len(X_loc), self.R
        dyn = isinstance(source, stg.Dtdg)

        def view(t, backward):
            if not dyn:
                return source.view()
            part = stg.STG_PART_OUT if backward else stg.STG_PART_IN
            return stg.stg_dtdg_get_snapshot_parts(source, t, part, backward=backward)

        for i in range(S):
            v = view(t0 + i, False)
            Hp = H0 if i == 0 else H_seq[i - 1]
            zg, zc = self.Zg[i & 1], self.Zc[i & 1]
            stg.stg_tgcn2_peer_fwd(0, v, params, X_loc[i], Hp, Z_loc=zg.buf.ptr, stack=self.stack)
            barrier()                                          # every owner's Zg rows written
            stg.stg_tgcn2_peer_fwd(1, v, params, X_loc[i], Hp, rows=zg.rows, Z_loc=zc.buf.ptr, stack=self.stack)
            barrier()                                          # every owner's Zc rows written
            stg.stg_tgcn2_peer_fwd(2, v, params, X_loc[i], Hp, rows=zc.rows, H_next=H_seq[i], stack=self.stack)
            stg.stg_mse_head(H_seq[i], Y_loc[i], w_o, b_o, loss_accum=loss, V_total=self.V)
        G, Gn = self.G[0][:R], self.G[1][:R]
        G.zero_()
        for i in range(S - 1, -1, -1):
            v = view(t0 + i, True)
            stg.stg_mse_head(H_seq[i], Y_loc[i], w_o, b_o, dH=G, accumulate=True, dw_o=dw_o, db_o=db_o,
                             V_total=self.V)
            dc, dg = self.Dc[i & 1], self.Dg[i & 1]
            stg.stg_tgcn2_peer_bwd(0, v, params, X_loc[i], G, Gn, grads, self.rank, self.bounds, None, dc.buf.ptr,
                                   self.stack)
            barrier()                                          # every rank's partial dY_c written
            stg.stg_tgcn2_peer_bwd(1, v, params, X_loc[i], None, Gn, grads, self.rank, self.bounds, dc.ptrs,
                                   dg.buf.ptr, self.stack)
            barrier()                                          # every rank's partial dY_g written
            stg.stg_tgcn2_peer_bwd(2, v, params, X_loc[i], None, Gn, grads, self.rank, self.bounds, dg.ptrs, None,
                                   self.stack)
            G, Gn = Gn, G

    def close(self):
        for g in self.Zg + self.Zc + self.Dc + self.Dg:
            g.close()
