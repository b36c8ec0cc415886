"""Dev tool: where does the per-launch fixed cost go?  Times (flush, e0, X, e1)
for X = an empty torch op, the step at N = 16 and at C2, the bench's way.
usage: overhead.py [steps]"""
import os, sys, statistics
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_chitchianasks13_b200 import filter as F, workload as W

K = int(sys.argv[1]) if len(sys.argv) > 1 else 30
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
tr = W.make_trajectory(5, K + 20, 0)
zs = torch.tensor(tr["Z"][1:], device="cuda"); us = torch.tensor(tr["U"][:-1], device="cuda")
small = torch.zeros(16, device="cuda")


def timed(fn, stream, do_flush=True):
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(K)]
    for i in range(K):
        if do_flush:
            with torch.cuda.stream(stream):
                flush.zero_()
        ev[i][0].record(stream)
        fn(i)
        ev[i][1].record(stream)
    torch.cuda.synchronize()
    return statistics.median(s.elapsed_time(e) * 1e3 for s, e in ev)


s = torch.cuda.Stream()
with torch.cuda.stream(s):
    print(f"empty torch op after flush: {timed(lambda i: small.add_(1), s):.1f} us")
for N in (16, 4096):
    for mapped in (1, 0):
        if not mapped:
            os.environ["PF_NO_MAPPED"] = "1"
        else:
            os.environ.pop("PF_NO_MAPPED", None)
        g = F.ParticleFilter(tr["mu0"], tr["sigma0"], F.ArmModel(n_joints=5), m=256, n_filters=N, device_inputs=True)
        for k in range(5):
            g.step(zs[k], us[k])
        torch.cuda.synchronize()
        t_f = timed(lambda i: g.step(zs[5 + i], us[5 + i]), g.stream)
        t_n = timed(lambda i: g.step(zs[5 + i], us[5 + i]), g.stream, do_flush=False)
        print(f"N={N} mapped={mapped}: flushed {t_f:.1f} us, back-to-back-ish (no flush, own events) {t_n:.1f} us")
        g.close()
