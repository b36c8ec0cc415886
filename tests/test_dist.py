"""Multi-rank host logic on CPU (gloo, world_size 2..4): the halo plan and
its exchange fill every halo row with the right neighbour sub-filter's
mailbox entries (Alg.2 l.10–14; sharding SURVEY §8(e)), and the
per-rank estimate records reduce to the oracle's global argmax (R6)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_ipps_chitchianasks13_b200 import distributed as Dd


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _expected_halo_ids(topo, N, world, rank, R=0, C=0):
    g0, n_local, n_ext = Dd.shard_geometry(topo, N, world, rank, R, C)
    if topo == "ring":
        return {n_local: (g0 - 1) % N, n_local + 1: (g0 + n_local) % N}
    R, C = Dd.torus_shape(N, R, C)
    r0, rows = g0 // C, n_local // C
    out = {}
    for c in range(C):
        out[n_local + c] = ((r0 - 1) % R) * C + c
        out[n_local + C + c] = ((r0 + rows) % R) * C + c
    return out


def _worker(rank, world, port, cases, ret):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        for topo, N, t, E in cases:
            g0, n_local, n_ext = Dd.shard_geometry(topo, N, world, rank)
            mb = torch.full((n_ext, t, E), -1.0)
            for row in range(n_local):
                mb[row] = float(g0 + row)          # entry = global sub-filter id
            plan = Dd.halo_plan(topo, N, world)
            Dd.exchange_halos(mb, plan, rank)
            for row, gid in _expected_halo_ids(topo, N, world, rank).items():
                assert torch.all(mb[row] == float(gid)), (topo, N, rank, row, gid, mb[row].flatten()[:3])
            for row in range(n_local):
                assert torch.all(mb[row] == float(g0 + row))
        # All-to-All pool rows: every rank's best-t row gathered in place
        g0, n_local, n_ext = Dd.shard_geometry("all2all", 4 * world, world, rank)
        assert n_ext == n_local + world + 1
        mb = torch.full((n_ext, 2, 5), -1.0)
        mb[n_local + rank] = float(100 + rank)
        Dd.gather_pool(mb, n_local, rank, world)
        for r in range(world):
            assert torch.all(mb[n_local + r] == float(100 + r))
        # estimate protocol: ordered key of every rank's best, all-gather, max
        rng = np.random.default_rng(7)
        w = np.round(rng.normal(-20, 5, 64 * world) * 2).astype(np.float32) / 2   # ties across ranks
        lo = rank * 64
        mine = w[lo:lo + 64]

        def key(v, p):
            b = np.array([v], np.float32).view(np.uint32)[0]
            o = (~b & 0xFFFFFFFF) if b & 0x80000000 else (b | 0x80000000)
            return (int(o) << 32) | (0xFFFFFFFF - p)

        best = max(key(v, lo + i) for i, v in enumerate(mine))
        keys = torch.zeros(world, dtype=torch.float64)
        out = [torch.zeros(2, dtype=torch.int64) for _ in range(world)]
        dist.all_gather(out, torch.tensor([best >> 32, best & 0xFFFFFFFF], dtype=torch.int64))
        win = max((int(a) << 32) | int(b) for a, b in out)
        idx = 0xFFFFFFFF - (win & 0xFFFFFFFF)
        ref = max(range(len(w)), key=lambda p: (w[p], -p))
        assert idx == ref
        ret[rank] = True
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3, 4])
def test_halo_exchange_gloo(world):
    cases = [("ring", 4 * world, 1, 11), ("ring", world, 2, 8)]
    if world in (2, 4):
        cases += [("torus", 16, 1, 11), ("torus", 64, 2, 6)]
    ctx = mp.get_context("spawn")
    ret = ctx.Manager().dict()
    mp.start_processes(_worker, args=(world, _free_port(), cases, ret), nprocs=world, join=True,
                       start_method="spawn")
    assert len(ret) == world


def test_loopback_matches_plan():
    # the single-process loopback applies the same plan
    for topo, N, world in [("ring", 8, 2), ("ring", 12, 4), ("torus", 16, 2), ("torus", 64, 4)]:
        mbs = []
        for r in range(world):
            g0, n_local, n_ext = Dd.shard_geometry(topo, N, world, r)
            mb = torch.full((n_ext, 1, 3), -1.0)
            mb[:n_local] = torch.arange(g0, g0 + n_local, dtype=torch.float32)[:, None, None]
            mbs.append(mb)
        Dd.loopback_exchange(mbs, Dd.halo_plan(topo, N, world))
        for r in range(world):
            for row, gid in _expected_halo_ids(topo, N, world, r).items():
                assert torch.all(mbs[r][row] == float(gid))


def test_plan_shapes():
    assert Dd.halo_plan("ring", 8, 1) == []
    assert Dd.halo_plan("none", 8, 4) == []
    p = Dd.halo_plan("torus", 64, 4)      # R = C = 8, 2 grid rows per rank
    assert len(p) == 8 and all(t.nrows == 8 for t in p)
    assert Dd.shard_geometry("torus", 64, 4, 3) == (48, 16, 32)
    assert Dd.shard_geometry("ring", 64, 4, 1) == (16, 16, 18)


class _FakeShard:
    """Host stand-in for a ParticleFilter shard: the partial record of R22
    (pf_mean_partial) computed on the host from the global L."""

    def __init__(self, state, logw, L, rank, world, orc):
        self.state, self.logw, self.L, self.orc = state, logw, L, orc
        self.rank, self.world = rank, world

    def mean_partial(self):
        q = np.array([self.orc.s_expq(float(v - self.L)) for v in self.logw], np.float64)
        S = (self.state.astype(np.float64) * q).sum(axis=1)
        Q = int(q.sum())
        return torch.tensor(np.concatenate([np.array([Q], np.int64).view(np.float64), S]))

    def reduce_means(self, parts):
        p = parts.numpy()
        Q = int(p[:, 0].copy().view(np.int64).sum())
        return (p[:, 1:].sum(axis=0) / Q).astype(np.float32)


def _mean_worker(rank, world, port, ret):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from oracle import orc
        orc.build()
        rng = np.random.default_rng(3)
        state = rng.normal(0, 1, (6, 40 * world)).astype(np.float32)
        logw = (-rng.exponential(3.0, 40 * world)).astype(np.float32)
        sl = slice(rank * 40, (rank + 1) * 40)
        df = Dd.DistributedFilter.__new__(Dd.DistributedFilter)
        df.pf, df.group, df.rank, df.world = _FakeShard(state[:, sl], logw[sl], logw.max(), rank, world, orc), None, \
            rank, world
        got = df.estimate_mean()
        np.testing.assert_allclose(got, orc.weighted_mean(state, logw), rtol=1e-6, atol=1e-7)
        ret[rank] = True
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_mean_protocol_gloo(world):
    # R22 across ranks: every rank's partial record (global L) all-gathered in
    # rank order and reduced = the weighted mean of the whole set
    ctx = mp.get_context("spawn")
    ret = ctx.Manager().dict()
    mp.start_processes(_mean_worker, args=(world, _free_port(), ret), nprocs=world, join=True, start_method="spawn")
    assert len(ret) == world


class _FakePeerShard:
    """Host stand-in for the peer-transport handshake of a shard: export may
    fail (no CUDA IPC), connect records the blobs it was given."""

    def __init__(self, rank, world, can_export):
        self.rank, self.world, self.can_export, self.connected = rank, world, can_export, None

    def peer_export(self):
        if not self.can_export:
            raise RuntimeError("no CUDA IPC")
        return bytes([self.rank]) * 160

    def peer_connect(self, blobs):
        self.connected = blobs


def _peer_worker(rank, world, port, fail_rank, ret):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        pf = _FakePeerShard(rank, world, rank != fail_rank)
        ok = Dd.connect_peers(pf)
        ret[rank] = (ok, pf.connected)
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,fail_rank", [(2, -1), (3, -1), (2, 1), (3, 0)])
def test_peer_handshake_gloo(world, fail_rank):
    # every rank connects with all blobs in rank order, or (one rank cannot
    # export) no rank connects and all stay on the NCCL transport
    ctx = mp.get_context("spawn")
    ret = ctx.Manager().dict()
    mp.start_processes(_peer_worker, args=(world, _free_port(), fail_rank, ret), nprocs=world, join=True,
                       start_method="spawn")
    expect = b"".join(bytes([r]) * 160 for r in range(world))
    for r in range(world):
        ok, blobs = ret[r]
        if fail_rank < 0:
            assert ok and blobs == expect
        else:
            assert not ok and blobs is None
