"""Multi-GPU sharding of the sub-filters — plumbing only.

Sub-filters shard naturally: rank r owns a contiguous range (ring) or a band
of grid rows (2D torus).  The only cross-rank data per step are

* the exchange halo: the best-t mailbox rows of the boundary sub-filters,
  sent to the neighbouring rank before the next step (Alg.2 l.10–14,
  PAPER.md:16; "exchanged particles are unique to neighbor pairs",
  PAPER.md:20 §VI-E), and
* the global estimate: every rank's best record (u64 key + state), gathered
  and reduced by the exact, order-free max of pf_reduce_records (R6).

Both go through ``torch.distributed`` (NCCL on GPUs, gloo in the CPU tests).
The halo *plan* (which mailbox rows go where) is a pure function shared by the
NCCL path, the single-process loopback used on one GPU, and the gloo tests;
the kernel side of the same layout is ``neighbor_row`` in csrc/pf_kernels.cuh
and the pf_shard comment in include/pf.h.
"""
from __future__ import annotations

import os
from dataclasses import dataclass

import torch
import torch.distributed as dist

RING, TORUS, ALL2ALL = "ring", "torus", "all2all"


@dataclass(frozen=True)
class Transfer:
    """nrows mailbox rows [src_row, src_row + nrows) of rank src -> rows
    [dst_row, dst_row + nrows) of rank dst (rows of t entries)."""
    src: int
    src_row: int
    dst: int
    dst_row: int
    nrows: int
    what: str


def torus_shape(n_filters: int, rows: int = 0, cols: int = 0) -> tuple[int, int]:
    """R = 2^floor(log2(N)/2), C = N / R unless given (reading R4)."""
    if rows > 0 and cols > 0:
        return rows, cols
    lg = n_filters.bit_length() - 1
    R = 1 << (lg // 2)
    return R, n_filters // R


def shard_geometry(topo: str, n_filters: int, world: int, rank: int, R: int = 0, C: int = 0):
    """(g0, n_local, n_ext) of a rank — the same rule as pf.h / pf_runtime.cu."""
    if topo == TORUS:
        R, C = torus_shape(n_filters, R, C)
        rows = R // world
        return rank * rows * C, rows * C, rows * C + (2 * C if world > 1 else 0)
    n_local = n_filters // world
    extra = (2 if (world > 1 and topo == RING) else 0) + ((world + 1 if world > 1 else 1) if topo == ALL2ALL else 0)
    return rank * n_local, n_local, n_local + extra


def halo_plan(topo: str, n_filters: int, world: int, R: int = 0, C: int = 0) -> list[Transfer]:
    """Every transfer of one exchange, in a canonical order.

    ring : rank r's first row -> rank r-1's row n_local+1 ("right" halo),
           rank r's last row  -> rank r+1's row n_local ("left" halo);
    torus: rank r's first grid row -> rank r-1's rows n_local+C.. ("below"),
           rank r's last grid row  -> rank r+1's rows n_local.. ("above").
    """
    if world <= 1 or topo not in (RING, TORUS):
        return []
    out = []
    for r in range(world):
        _, n_local, _ = shard_geometry(topo, n_filters, world, r, R, C)
        prev, nxt = (r - 1) % world, (r + 1) % world
        if topo == RING:
            out.append(Transfer(r, 0, prev, n_local + 1, 1, "first->prev.right"))
            out.append(Transfer(r, n_local - 1, nxt, n_local, 1, "last->next.left"))
        else:
            _, Cc = torus_shape(n_filters, R, C)
            out.append(Transfer(r, 0, prev, n_local + Cc, Cc, "first->prev.below"))
            out.append(Transfer(r, n_local - Cc, nxt, n_local, Cc, "last->next.above"))
    return out


def _ordered_ops(plan: list[Transfer], rank: int):
    """This rank's sends and receives, ordered so that the k-th send to a
    peer matches the k-th receive of that peer (NCCL matches point-to-point
    operations between a pair in issue order)."""
    sends = [t for t in plan if t.src == rank]
    recvs = [t for t in plan if t.dst == rank]
    # order receives from each peer like that peer orders its sends to us
    recvs.sort(key=lambda t: (t.src, [s for s in plan if s.src == t.src and s.dst == rank].index(t)))
    return sends, recvs


def exchange_halos(mailbox_parity: torch.Tensor, plan: list[Transfer], rank: int, group=None) -> None:
    """Fill this rank's halo rows of one mailbox parity [n_ext, t, E] from the
    neighbouring ranks (torch.distributed point-to-point, one batch)."""
    sends, recvs = _ordered_ops(plan, rank)
    ops = []
    for t in sends:
        ops.append(dist.P2POp(dist.isend, mailbox_parity[t.src_row:t.src_row + t.nrows].contiguous(), t.dst,
                              group=group))
    for t in recvs:   # rows are the leading dimension: the slice is contiguous
        ops.append(dist.P2POp(dist.irecv, mailbox_parity[t.dst_row:t.dst_row + t.nrows], t.src, group=group))
    if ops:
        for w in dist.batch_isend_irecv(ops):
            w.wait()


def gather_pool(mailbox_parity: torch.Tensor, n_local: int, rank: int, world: int, group=None) -> None:
    """All-to-All: all-gather every rank's best-t row (row n_local + rank) into
    rows [n_local, n_local + world) of one mailbox parity (in place)."""
    rows = mailbox_parity[n_local:n_local + world]
    dist.all_gather_into_tensor(rows.reshape(-1), rows[rank].reshape(-1).clone(), group=group)


def loopback_exchange(mailboxes: list[torch.Tensor], plan: list[Transfer]) -> None:
    """The same plan between shards held by one process (e.g. on one GPU)."""
    for t in plan:
        mailboxes[t.dst][t.dst_row:t.dst_row + t.nrows].copy_(mailboxes[t.src][t.src_row:t.src_row + t.nrows])


def connect_peers(pf, group=None) -> bool:
    """Peer transport (include/pf.h): every rank exports its CUDA IPC blob, the
    blobs are all-gathered (host objects, any backend), every rank opens its
    neighbours' mailboxes and all peer blocks.  Returns False on every rank
    (nothing connected: the NCCL path stays) if any rank cannot export."""
    try:
        blob, ok = pf.peer_export(), True
    except Exception:   # e.g. no CUDA IPC on this system
        blob, ok = b"", False
    got = [None] * pf.world
    dist.all_gather_object(got, (ok, blob), group=group)
    if not all(g[0] for g in got):
        return False
    pf.peer_connect(b"".join(g[1] for g in got))
    dist.barrier(group=group)   # every rank connected before anyone steps
    return True


class DistributedFilter:
    """One rank of a filter sharded over ``world`` processes (one per GPU).

    transport "p2p" (default): the step kernel itself writes the boundary rows
    into the neighbours' halo rows (All-to-All: its pool row into every rank's
    peer block) and reduces the global estimate (and pool) through the ranks'
    peer blocks (NVLink peer memory, include/pf.h pf_peer_*), so step() is the
    kernel launch alone.  transport "nccl": halo exchange of the previous step's mailbox through
    torch.distributed, the step kernel, then all-gather of the per-rank
    estimate records and their exact reduce, all on the filter's CUDA stream.
    """

    def __init__(self, pf, group=None, transport: str | None = None):
        self.pf, self.group = pf, group
        self.rank, self.world = pf.rank, pf.world
        s = pf.shard
        self.plan = halo_plan(pf.topo, pf.n_filters, pf.world, int(s.torus_rows), int(s.torus_cols))
        self.k = 0
        self._records = torch.empty(self.world, s.record_floats, dtype=torch.float32, device=pf.device)
        transport = transport or os.environ.get("PF_TRANSPORT", "p2p")
        self.p2p = False
        if self.world > 1 and transport == "p2p":
            self.p2p = connect_peers(pf, group)

    def step(self, z, u) -> None:
        if self.p2p:   # halo + global estimate inside the kernel
            self.pf.step(z, u)
            self.k += 1
            return
        if self.world > 1 and self.k >= 1:
            exchange_halos(self.pf.mailbox[self.k & 1], self.plan, self.rank, self.group)
        self.pf.step(z, u)
        self.k += 1
        if self.world > 1:
            if self.pf.topo == ALL2ALL and self.pf.t > 0:
                gather_pool(self.pf.mailbox[self.k & 1], int(self.pf.shard.n_local), self.rank, self.world,
                            self.group)
                self.pf.reduce_pool()
            dist.all_gather_into_tensor(self._records, self.pf.record, group=self.group)
            self.pf.reduce_records(self._records)

    def estimate(self):
        return self.pf.estimate()

    def estimate_mean(self):
        """Weighted-average estimate (R22) of the whole sharded filter: every
        rank's partial record (with the global L of the reduced record) is
        all-gathered and summed in rank order."""
        if self.world == 1:
            return self.pf.estimate_mean()
        part = self.pf.mean_partial()
        gathered = torch.empty(self.world * part.numel(), dtype=torch.float64, device=part.device)
        dist.all_gather_into_tensor(gathered, part.contiguous(), group=self.group)
        return self.pf.reduce_means(gathered.view(self.world, part.numel()))
