"""Dev diagnostic: back-to-back peer steps with a delayed rank; prints per-step record vs oracle."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np, torch
from paper_conf_ipps_chitchianasks13_b200 import filter as F, workload as W
from oracle import orc
topo = sys.argv[1] if len(sys.argv) > 1 else "ring"
sleep = int(sys.argv[2]) if len(sys.argv) > 2 else 2_000_000
sync = len(sys.argv) > 3 and sys.argv[3] == "sync"
nj, m, N, world, T = 5, 64, 16, 2, 10
tr = W.make_trajectory(nj, T, 2)
kw = dict(m=m, n_filters=N, t=1, topo=topo, resampler="rws", seed=17)
shards = [F.ParticleFilter(tr["mu0"], tr["sigma0"], F.ArmModel(n_joints=nj), rank=r, world=world,
                           stream=torch.cuda.Stream(), **kw) for r in range(world)]
F.ParticleFilter.peer_connect_local(shards)
torch.cuda._sleep(1); torch.cuda.synchronize()   # module loaded before any rendezvous
recs = [[] for _ in shards]
for k in range(1, T + 1):
    for r, s in enumerate(shards):
        if r == 1 and k % 2 == 0 and sleep:
            with torch.cuda.stream(s.stream):
                torch.cuda._sleep(sleep)
        s.step(tr["Z"][k], tr["U"][k - 1])
        with torch.cuda.stream(s.stream):
            recs[r].append(s.record.clone())
    if sync:
        torch.cuda.synchronize()
torch.cuda.synchronize()
o = orc.Filter(orc.Config(**kw), orc.Model(n_joints=nj), tr["mu0"], tr["sigma0"])
for k in range(1, T + 1):
    o.step(tr["Z"][k], tr["U"][k - 1])
    xo, lo, io = o.estimate()
    row = []
    for r in range(world):
        rec = recs[r][k - 1].cpu().numpy()
        idx = 0xFFFFFFFF - int(rec[:1].view(np.uint32)[0])
        row.append((idx, float(rec[2]), int(rec[3:4].view(np.uint32)[0])))
    print(k, "oracle", io, lo, "gpu", row, "OK" if all(x[0] == io for x in row) else "BAD")
