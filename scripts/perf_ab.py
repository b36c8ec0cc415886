"""Dev tool: A/B device timing of two library builds (or one), bench-style (L2
flushed before every step, CUDA events on the filter stream), interleaved.
usage: perf_ab.py LIB_A [LIB_B] [--reps R] [--quick]
A library path of '-' means the in-tree libpf_b200.so."""
import json, os, statistics, subprocess, sys

CONFIGS = [  # nj, m, N, resampler, topo, t
    (5, 256, 4096, "rws", "ring", 1), (5, 256, 4096, "vose", "ring", 1),
    (5, 256, 65536, "rws", "ring", 1), (5, 256, 65536, "vose", "ring", 1),
    (28, 256, 65536, "rws", "ring", 1), (28, 256, 65536, "vose", "ring", 1),
    (5, 256, 16384, "rws", "torus", 1), (5, 256, 16384, "rws", "ring", 0),
    (5, 1048576, 1, "rws", "none", 0), (5, 1048576, 1, "vose", "none", 0),   # centralized filter (NEXT-2)
]


def child(cfgs, K):
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import torch
    from paper_conf_ipps_chitchianasks13_b200 import filter as F, workload as W
    flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
    out = {}
    for nj, m, N, res, topo, t in cfgs:
        tr = W.make_trajectory(nj, K + 20, 0)
        g = F.ParticleFilter(tr["mu0"], tr["sigma0"], F.ArmModel(n_joints=nj), m=m, n_filters=N, resampler=res,
                             topo=topo, t=t, device_inputs=True)
        zs = torch.tensor(tr["Z"][1:], device="cuda"); us = torch.tensor(tr["U"][:-1], device="cuda")
        for k in range(5):
            g.step(zs[k], us[k])
        torch.cuda.synchronize()
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(K)]
        for i in range(K):
            with torch.cuda.stream(g.stream):
                flush.zero_()
            ev[i][0].record(g.stream)
            g.step(zs[5 + i], us[5 + i])
            ev[i][1].record(g.stream)
        torch.cuda.synchronize()
        out[f"nj{nj} m{m} N{N} {res} {topo} t{t}"] = statistics.median(s.elapsed_time(e) * 1e3 for s, e in ev)
        g.close()
    print("RESULT " + json.dumps(out), flush=True)


def main():
    args = [a for a in sys.argv[1:] if not a.startswith("--")]
    reps = 3
    if "--reps" in sys.argv:
        reps = int(sys.argv[sys.argv.index("--reps") + 1])
        args = [a for a in args if a != str(reps)]
    cfgs = CONFIGS[:3] if "--quick" in sys.argv else CONFIGS
    res = {a: {} for a in args}
    for r in range(reps):
        for lib in args:
            env = dict(os.environ)
            if lib != "-":
                env["PF_LIB"] = os.path.abspath(lib)
            p = subprocess.run([sys.executable, __file__, "--child", json.dumps(cfgs)], env=env, capture_output=True,
                               text=True)
            line = [l for l in p.stdout.splitlines() if l.startswith("RESULT ")]
            if not line:
                print(lib, "FAILED", p.stderr[-2000:])
                continue
            for k, v in json.loads(line[0][7:]).items():
                res[lib].setdefault(k, []).append(v)
    keys = list(res[args[0]].keys())
    for k in keys:
        cells = []
        for lib in args:
            v = res[lib].get(k, [])
            cells.append(f"{statistics.median(v):8.1f}" if v else "     n/a")
        ratio = ""
        if len(args) == 2 and res[args[0]].get(k) and res[args[1]].get(k):
            ratio = f"  B/A {statistics.median(res[args[1]][k]) / statistics.median(res[args[0]][k]):.3f}"
        print(f"{k:32s} " + " ".join(cells) + " us" + ratio)


if __name__ == "__main__":
    if len(sys.argv) > 1 and sys.argv[1] == "--child":
        child([tuple(c) for c in json.loads(sys.argv[2])], 20)
    else:
        main()
