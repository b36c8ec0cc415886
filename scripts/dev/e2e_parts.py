"""Dev: where the host-clock e2e step time goes (pf_step enqueue vs pf_estimate wait)."""
import os, sys, time, statistics
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np, torch
from paper_conf_ipps_chitchianasks13_b200 import filter as F, workload as W
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
for _ in range(200): flush.zero_()
tr = W.make_trajectory(5, 80, 0)
g = F.ParticleFilter(tr["mu0"], tr["sigma0"], F.ArmModel(n_joints=5), m=256, n_filters=4096, t=1, topo="ring", seed=1)
Z = np.ascontiguousarray(tr["Z"][1:], np.float32); U = np.ascontiguousarray(tr["U"][:-1], np.float32)
for k in range(5):
    g.step(Z[k], U[k]); g.estimate()
a, b, c = [], [], []
for i in range(5, 65):
    flush.zero_(); torch.cuda.synchronize()
    t0 = time.perf_counter(); g.step(Z[i], U[i]); t1 = time.perf_counter(); g.estimate(); t2 = time.perf_counter()
    a.append(t1 - t0); b.append(t2 - t1); c.append(t2 - t0)
print("step enqueue %.1f us, estimate wait %.1f us, total %.1f us" % tuple(1e6 * statistics.median(x) for x in (a, b, c)))
# the same without the L2 flush (real-time loop: previous step's data in L2)
a, b, c = [], [], []
for i in range(5, 65):
    torch.cuda.synchronize()
    t0 = time.perf_counter(); g.step(Z[i], U[i]); t1 = time.perf_counter(); g.estimate(); t2 = time.perf_counter()
    a.append(t1 - t0); b.append(t2 - t1); c.append(t2 - t0)
print("no flush: step enqueue %.1f us, estimate wait %.1f us, total %.1f us" % tuple(1e6 * statistics.median(x) for x in (a, b, c)))
h = g.h
from paper_conf_ipps_chitchianasks13_b200 import binding as B
L = B.lib()
zp, up = Z.ctypes.data, U.ctypes.data
x = np.zeros(9, np.float32)
t0 = time.perf_counter()
for i in range(200):
    L.pf_step(h, Z[i % 60].ctypes.data, U[i % 60].ctypes.data)
    L.pf_estimate(h, x.ctypes.data, None, None)
print("raw ctypes loop: %.1f us/step" % ((time.perf_counter() - t0) / 200 * 1e6))
# host cost of one trivial ctypes call and of pf_step alone on a tiny filter (GPU keeps up)
t0 = time.perf_counter()
for i in range(2000):
    L.pf_last_error(h)
print("ctypes trivial call: %.2f us" % ((time.perf_counter() - t0) / 2000 * 1e6))
gt = F.ParticleFilter(tr["mu0"], tr["sigma0"], F.ArmModel(n_joints=5), m=32, n_filters=4, t=1, topo="ring", seed=1)
for k in range(5):
    gt.step(Z[k], U[k]); gt.estimate()
torch.cuda.synchronize()
t0 = time.perf_counter()
for i in range(300):
    L.pf_step(gt.h, Z[i % 60].ctypes.data, U[i % 60].ctypes.data)
t1 = time.perf_counter()
torch.cuda.synchronize()
t2 = time.perf_counter()
print("tiny filter: pf_step enqueue %.2f us/call (drain %.1f us)" % ((t1 - t0) / 300 * 1e6, (t2 - t1) * 1e6))
zp0, up0 = Z.ctypes.data, U.ctypes.data
zs0, us0 = Z.strides[0], U.strides[0]
ptrs = [(zp0 + (i % 60) * zs0, up0 + (i % 60) * us0) for i in range(300)]
torch.cuda.synchronize()
t0 = time.perf_counter()
for zz, uu in ptrs:
    L.pf_step(gt.h, zz, uu)
t1 = time.perf_counter()
torch.cuda.synchronize()
print("tiny filter: pf_step with precomputed pointers %.2f us/call" % ((t1 - t0) / 300 * 1e6))
t0 = time.perf_counter()
for i in range(2000):
    _ = Z[i % 60].ctypes.data
print("numpy view + .ctypes.data: %.2f us" % ((time.perf_counter() - t0) / 2000 * 1e6))
