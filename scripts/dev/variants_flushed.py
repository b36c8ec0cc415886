"""Dev: flushed per-step time (bench-style) of every PF_VARIANT of one config."""
import os, subprocess, sys, json
nj, m, N, res = sys.argv[1:5]
nvar = int(sys.argv[5]) if len(sys.argv) > 5 else 12
child = r'''
import os, sys, statistics
sys.path.insert(0, os.getcwd())
import torch
from paper_conf_ipps_chitchianasks13_b200 import filter as F, workload as W
nj, m, N, res = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3]), sys.argv[4]
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
for _ in range(200): flush.zero_()
tr = W.make_trajectory(nj, 60, 0)
g = F.ParticleFilter(tr["mu0"], tr["sigma0"], F.ArmModel(n_joints=nj), m=m, n_filters=N, resampler=res, device_inputs=True)
zs = torch.tensor(tr["Z"][1:], device="cuda"); us = torch.tensor(tr["U"][:-1], device="cuda")
for k in range(5): g.step(zs[k], us[k])
torch.cuda.synchronize()
ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(40)]
for i in range(40):
    with torch.cuda.stream(g.stream): flush.zero_()
    ev[i][0].record(g.stream); g.step(zs[5 + i], us[5 + i]); ev[i][1].record(g.stream)
torch.cuda.synchronize()
print("RES", statistics.median(a.elapsed_time(b) * 1e3 for a, b in ev))
'''
for v in range(nvar):
    env = dict(os.environ, PF_VARIANT=str(v))
    r = subprocess.run([sys.executable, "-c", child, nj, m, N, res], env=env, capture_output=True, text=True)
    line = [l for l in r.stdout.splitlines() if l.startswith("RES")]
    print(f"variant {v}: {line[0][4:] if line else 'fail ' + r.stderr[-300:]}", flush=True)
