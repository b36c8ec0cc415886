"""Peer transport (include/pf.h pf_peer_*): the halo rows (or the All-to-All
pool rows) and the global estimate cross ranks inside the step kernel (peer stores + a device-side flag
rendezvous) instead of NCCL around it.  On one device: (1) `world` shards in
one process, each stepping on its own stream, connected without IPC; (2) two
processes sharing the device, connected through CUDA IPC with the blobs
all-gathered over gloo (the path DistributedFilter takes on a multi-GPU node).
Bar: every rank's estimate equals the oracle's at every step and the
concatenated shards equal the oracle's particle set bit for bit (global Philox
counters, exact max reduce — SURVEY.md §8(e))."""
import os
import subprocess
import sys
import textwrap

import numpy as np
import pytest

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def P():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_ipps_chitchianasks13_b200 import build, filter as F
    build.build()
    return F


@pytest.mark.timeout(120)
@pytest.mark.parametrize("topo,N,world,t", [("ring", 16, 2, 1), ("ring", 8, 4, 1), ("torus", 64, 2, 1),
                                            ("torus", 16, 4, 1), ("ring", 4, 4, 1), ("all2all", 16, 2, 2),
                                            ("all2all", 8, 4, 1), ("all2all", 32, 4, 3),
                                            ("ring", 16, 8, 1), ("torus", 64, 8, 1), ("all2all", 16, 8, 2)])   # 8 ranks
def test_peer_transport_local(P, orc, W, topo, N, world, t):
    import torch
    nj, m, T = 5, 64, 6
    tr = W.make_trajectory(nj, T, 5)
    kw = dict(m=m, n_filters=N, t=t, topo=topo, resampler="rws", seed=31)
    shards = [P.ParticleFilter(tr["mu0"], tr["sigma0"], P.ArmModel(n_joints=nj), rank=r, world=world,
                               stream=torch.cuda.Stream(), **kw) for r in range(world)]
    P.ParticleFilter.peer_connect_local(shards)
    assert all(s.peer_connected for s in shards)
    o = orc.Filter(orc.Config(**kw), orc.Model(n_joints=nj), tr["mu0"], tr["sigma0"])
    for k in range(1, T + 1):
        for s in shards:          # every shard launched before any estimate is awaited
            s.step(tr["Z"][k], tr["U"][k - 1])
        o.step(tr["Z"][k], tr["U"][k - 1])
        xo, lo, io = o.estimate()
        for s in shards:
            xg, lg, ig = s.estimate()
            assert ig == io, (k, ig, io)
            np.testing.assert_array_equal(xg, xo)
    so, wo, _ = o.get()
    parts = [s.get_particles() for s in shards]
    np.testing.assert_array_equal(np.concatenate([p[0] for p in parts], axis=1), so)
    np.testing.assert_array_equal(np.concatenate([p[1] for p in parts]), wo)
    for s in shards:
        s.close()


_TWO_PROC = textwrap.dedent(r"""
    import os, sys
    sys.path.insert(0, os.environ["PF_ROOT"])
    import numpy as np, torch, torch.distributed as dist
    from paper_conf_ipps_chitchianasks13_b200 import filter as F, workload as W, distributed as D
    from oracle import orc
    rank, world = int(os.environ["RANK"]), int(os.environ["WORLD_SIZE"])
    dist.init_process_group("gloo", rank=rank, world_size=world)
    torch.cuda.set_device(0)
    nj, m, N, T, topo = 5, 64, 16, 5, os.environ["PF_TOPO"]
    tr = W.make_trajectory(nj, T, 6)
    kw = dict(m=m, n_filters=N, t=2 if topo == "all2all" else 1, topo=topo, resampler="vose", seed=13)
    pf = F.ParticleFilter(tr["mu0"], tr["sigma0"], F.ArmModel(n_joints=nj), rank=rank, world=world, **kw)
    df = D.DistributedFilter(pf, transport="p2p")
    assert df.p2p and pf.peer_connected
    o = orc.Filter(orc.Config(**kw), orc.Model(n_joints=nj), tr["mu0"], tr["sigma0"])
    for k in range(1, T + 1):
        df.step(tr["Z"][k], tr["U"][k - 1])
        o.step(tr["Z"][k], tr["U"][k - 1])
        xg, lg, ig = df.estimate()
        xo, lo, io = o.estimate()
        assert ig == io and np.array_equal(xg, xo), (rank, k, ig, io)
    so, _, _ = o.get()
    g0 = int(pf.shard.g0) * m
    sg = pf.get_particles()[0]
    assert np.array_equal(sg, so[:, g0:g0 + sg.shape[1]]), rank
    dist.barrier()
    pf.close()
    print("rank", rank, "ok")
""")


@pytest.mark.timeout(300)
@pytest.mark.parametrize("topo", ["ring", "torus", "all2all"])
def test_peer_transport_two_processes_ipc(P, topo, tmp_path):
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    script = tmp_path / "peer2.py"
    script.write_text(_TWO_PROC)
    procs = []
    for r in range(2):
        env = dict(os.environ, RANK=str(r), WORLD_SIZE="2", MASTER_ADDR="127.0.0.1", MASTER_PORT="29617",
                   PF_ROOT=root, PF_TOPO=topo)
        procs.append(subprocess.Popen([sys.executable, str(script)], env=env, stdout=subprocess.PIPE,
                                      stderr=subprocess.STDOUT, text=True))
    outs = []
    for p in procs:
        try:
            out, _ = p.communicate(timeout=240)
        except subprocess.TimeoutExpired:
            for q in procs:
                q.kill()
            raise
        outs.append(out)
    for r, (p, out) in enumerate(zip(procs, outs)):
        assert p.returncode == 0, f"rank {r}:\n{out[-3000:]}"
        assert f"rank {r} ok" in out


@pytest.mark.timeout(120)
@pytest.mark.parametrize("topo,t", [("ring", 1), ("all2all", 2)])
def test_peer_back_to_back_skewed(P, orc, W, topo, t):
    # steps launched back to back with NO host synchronization between them,
    # one shard's stream delayed by a sleep before every other step, each
    # step's record captured on the device: every step's estimate must still
    # equal the oracle's (double-buffered records / pool rows)
    import torch
    nj, m, N, world, T = 5, 64, 16, 2, 10
    tr = W.make_trajectory(nj, T, 2)
    kw = dict(m=m, n_filters=N, t=t, topo=topo, resampler="rws", seed=17)
    shards = [P.ParticleFilter(tr["mu0"], tr["sigma0"], P.ArmModel(n_joints=nj), rank=r, world=world,
                               stream=torch.cuda.Stream(), **kw) for r in range(world)]
    P.ParticleFilter.peer_connect_local(shards)
    # load the sleep kernel's module now: a lazily loaded module can only be
    # loaded between kernels, so loading it while rank 0's step kernel waits
    # at the rendezvous would stall the one host thread that must launch
    # rank 1's step (caught by the rendezvous timeout, PF_ETIMEOUT)
    torch.cuda._sleep(1)
    torch.cuda.synchronize()
    recs = [[] for _ in shards]
    for k in range(1, T + 1):
        for r, s in enumerate(shards):
            if r == 1 and k % 2 == 0:
                with torch.cuda.stream(s.stream):
                    torch.cuda._sleep(2_000_000)      # ~1 ms: rank 1 reaches the rendezvous late
            s.step(tr["Z"][k], tr["U"][k - 1])
            with torch.cuda.stream(s.stream):
                recs[r].append(s.record.clone())
    torch.cuda.synchronize()
    o = orc.Filter(orc.Config(**kw), orc.Model(n_joints=nj), tr["mu0"], tr["sigma0"])
    for k in range(1, T + 1):
        o.step(tr["Z"][k], tr["U"][k - 1])
        xo, lo, io = o.estimate()
        for r in range(world):
            rec = recs[r][k - 1].cpu().numpy()
            idx = 0xFFFFFFFF - int(rec[:1].view(np.uint32)[0])
            assert idx == io, (r, k, idx, io)
            assert rec[3:4].view(np.uint32)[0] == 0          # status ok
            np.testing.assert_array_equal(rec[4:4 + nj + 4], xo)
    for s in shards:
        s.close()


@pytest.mark.timeout(120)
def test_peer_rendezvous_timeout_is_reported(P, W, monkeypatch):
    # a rank that never arrives: the waiting rank's kernel gives up after
    # PF_PEER_TIMEOUT_MS and pf_estimate returns PF_ETIMEOUT (sticky) — the
    # GPU does not hang
    import torch
    monkeypatch.setenv("PF_PEER_TIMEOUT_MS", "300")
    nj = 2
    tr = W.make_trajectory(nj, 4, 0)
    kw = dict(m=64, n_filters=4, t=1, topo="ring", seed=1)
    shards = [P.ParticleFilter(tr["mu0"], tr["sigma0"], P.ArmModel(n_joints=nj), rank=r, world=2,
                               stream=torch.cuda.Stream(), **kw) for r in range(2)]
    P.ParticleFilter.peer_connect_local(shards)
    shards[0].step(tr["Z"][1], tr["U"][0])          # rank 1 never steps
    with pytest.raises(P.B.PFError, match="timed out"):
        shards[0].estimate()
    with pytest.raises(P.B.PFError):                # sticky
        shards[0].step(tr["Z"][2], tr["U"][1])
    for s in shards:
        s.close()
