"""Dev tool: per-sub-filter timeline of one step-kernel launch (needs a PF_TIMELINE
build loaded through PF_LIB, see build_variant.py).  usage: timeline.py nj m N res [flush]
Prints the kernel span, the ramp (first data arrival), mean phase durations per
sub-filter and the tail (how long the last 10% of groups run alone)."""
import ctypes as C, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_ipps_chitchianasks13_b200 import binding, filter as F, workload as W

nj, m, N, res = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3]), sys.argv[4]
flush_l2 = len(sys.argv) <= 5 or sys.argv[5] != "0"
host_in = len(sys.argv) > 6 and sys.argv[6] == "host"   # z / u through the launch (the e2e path)
tr = W.make_trajectory(nj, 20, 0)
g = F.ParticleFilter(tr["mu0"], tr["sigma0"], F.ArmModel(n_joints=nj), m=m, n_filters=N, resampler=res,
                     device_inputs=not host_in)
zs = torch.tensor(tr["Z"][1:], device="cuda"); us = torch.tensor(tr["U"][:-1], device="cuda")
L = binding.lib()
fn = L.pf_debug_timeline
fn.argtypes = [C.c_void_p, C.c_longlong, C.c_int]
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
for k in range(5):
    g.step(*((tr["Z"][k + 1], tr["U"][k]) if host_in else (zs[k], us[k])))
torch.cuda.synchronize()
for rep in range(3):
    if flush_l2:
        flush.zero_()
    torch.cuda.synchronize()
    fn(None, 0, 1)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    if host_in:
        zh, uh = tr["Z"][6 + rep], tr["U"][5 + rep]
        e0.record(g.stream); g.step(zh, uh); e1.record(g.stream)
    else:
        e0.record(g.stream); g.step(zs[5 + rep], us[5 + rep]); e1.record(g.stream)
    torch.cuda.synchronize()
    buf = np.zeros(1 + 8 * 65536, np.uint64)
    fn(buf.ctypes.data, buf.size, 0)
    t2 = np.zeros(4, np.uint64)
    fn(t2.ctypes.data, -1, 0)
    n = int(buf[0]); r = buf[1:1 + 8 * n].reshape(n, 8).astype(np.int64)
    t3 = np.zeros(3 * 4096, np.uint64)
    fn(t3.ctypes.data, -2, 0)
    t3 = t3.reshape(4096, 3).astype(np.int64)
    t3 = t3[t3[:, 0] > 0]
    if len(t3):   # per-CTA prologue: entry -> after griddepcontrol.wait -> after the prologue barrier
        e0_ = t3[:, 0].min()
        q = lambda v: f"p50 {np.median(v)/1e3:.2f} p90 {np.percentile(v, 90)/1e3:.2f} max {v.max()/1e3:.2f}"
        print(f"  CTAs {len(t3)}: entry (from first) {q(t3[:, 0] - e0_)}; wait {q(t3[:, 1] - t3[:, 0])}; "
              f"prologue {q(t3[:, 2] - t3[:, 1])}; ready-to-loop (from first entry) {q(t3[:, 2] - e0_)}")
    tmin = int(r[:, 1].min())
    print(f"  first CTA entry -> first group start {(tmin - int(t2[0]))/1e3:.2f} us; last group end -> "
          f"epilogue (last CTA) start {(int(t2[1]) - int(r[:, 7].max()))/1e3:.2f} us; epilogue {(int(t2[2]) - int(t2[1]))/1e3:.2f} us")
    t0 = r[:, 1].min()
    start, w0, ready, merged, resd, smp, end = (r[:, i] - t0 for i in range(1, 8))
    grp = (r[:, 0] >> 40)
    span = end.max()
    print(f"rep {rep}: event {e0.elapsed_time(e1)*1e3:.1f} us, kernel span (first CTA start -> last sub-filter end) {span/1e3:.1f} us, "
          f"{n} sub-filters, {len(np.unique(grp))} groups")
    print(f"  CTA start spread {np.ptp(start)/1e3:.2f} us; first data ready {ready.min()/1e3:.2f} us, "
          f"median first ready {np.median([ready[grp == q].min() for q in np.unique(grp)])/1e3:.2f} us")
    print(f"  per sub-filter (mean us): wait {np.mean(ready - w0)/1e3:.2f}  exchange {np.mean(merged - ready)/1e3:.2f}  "
          f"resample {np.mean(resd - merged)/1e3:.2f}  sample {np.mean(smp - resd)/1e3:.2f}  reduce+finish {np.mean(end - smp)/1e3:.2f}"
          f"  total {np.mean(end - ready)/1e3:.2f}")
    ends = np.sort([end[grp == q].max() for q in np.unique(grp)])
    print(f"  group end times (us): p10 {ends[len(ends)//10]/1e3:.1f} p50 {ends[len(ends)//2]/1e3:.1f} "
          f"p90 {ends[9*len(ends)//10]/1e3:.1f} max {ends[-1]/1e3:.1f}")
    cnt = np.bincount(np.unique(grp, return_inverse=True)[1])
    print(f"  sub-filters per group: {np.bincount(cnt)}")
    # concurrency profile: busy groups in 2-us bins
    bins = np.arange(0, span + 2000, 2000)
    busy = [int(np.sum((ready <= b + 1000) & (end > b + 1000))) for b in bins[:-1]]
    print("  busy sub-filters per 2 us:", busy)
    if rep == 2:   # one machine-readable line (the Fig. 4-style per-phase breakdown)
        import json
        print("TIMELINE " + json.dumps({
            "n_joints": nj, "m": m, "N": N, "particles": m * N, "resampler": res, "flush_l2": flush_l2,
            "event_us": e0.elapsed_time(e1) * 1e3, "kernel_span_us": span / 1e3,
            "epilogue_us": (int(t2[2]) - int(t2[1])) / 1e3, "first_data_us": ready.min() / 1e3,
            "groups": int(len(np.unique(grp))), "sub_filters": n,
            "per_sub_filter_us": {"wait": float(np.mean(ready - w0)) / 1e3, "exchange": float(np.mean(merged - ready)) / 1e3,
                                  "normalise_resample": float(np.mean(resd - merged)) / 1e3,
                                  "sample_weight_store": float(np.mean(smp - resd)) / 1e3,
                                  "reduce_finish": float(np.mean(end - smp)) / 1e3},
            "group_end_us": {"p10": ends[len(ends) // 10] / 1e3, "p50": ends[len(ends) // 2] / 1e3,
                             "p90": ends[9 * len(ends) // 10] / 1e3, "max": ends[-1] / 1e3}}), flush=True)
g.close()
