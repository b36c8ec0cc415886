"""Dev tool: flushed step time of every PF_VARIANT for one config.  usage: variants_one.py nj m N res nvar"""
import os, subprocess, sys, json
nj, m, N, res, nv = sys.argv[1:6]   # nv: a count or a comma list of variant indices
here = os.path.dirname(os.path.abspath(__file__))
for v in (range(int(nv)) if "," not in nv else [int(x) for x in nv.split(",")]):
    env = dict(os.environ, PF_VARIANT=str(v))
    r = subprocess.run([sys.executable, os.path.join(here, "perf_ab.py"), "--child",
                        json.dumps([[int(nj), int(m), int(N), res, "ring", 1]])], env=env, capture_output=True, text=True)
    print(f"variant {v}: {[l for l in r.stdout.splitlines() if l.startswith('RESULT')]} {r.stderr[-300:] if r.returncode else ''}", flush=True)
