"""A/B timing of PF_VARIANT choices, interleaved, several repeats: ab.py NJ M N RES v1 v2 [reps]"""
import os, subprocess, sys, statistics
nj, m, N, res, va, vb = sys.argv[1:7]
reps = int(sys.argv[7]) if len(sys.argv) > 7 else 3
t = {va: [], vb: []}
for r in range(reps):
    for v in (va, vb):
        out = subprocess.run([sys.executable, os.path.join(os.path.dirname(__file__), "time_one.py"), nj, m, N, res, "30"],
                             env=dict(os.environ, PF_VARIANT=v), capture_output=True, text=True).stdout
        t[v].append(float(out.split("rws:" if res == "rws" else "vose:")[1].split("us")[0]))
for v in (va, vb):
    print(f"nj={nj} m={m} N={N} {res} variant {v}: median {statistics.median(t[v]):.1f} us  {t[v]}")
