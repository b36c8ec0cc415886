"""Time every compiled variant (PF_VARIANT) of a config: usage NJ M N RES [T]."""
import os, subprocess, sys
nj, m, N, res = sys.argv[1:5]
T = sys.argv[5] if len(sys.argv) > 5 else "30"
for v in range(int(os.environ.get("NVAR", "8"))):
    env = dict(os.environ, PF_VARIANT=str(v))
    r = subprocess.run([sys.executable, os.path.join(os.path.dirname(__file__), "time_one.py"), nj, m, N, res, T],
                       env=env, capture_output=True, text=True)
    print(f"variant {v}: {r.stdout.strip()} {r.stderr.strip()[-200:] if r.returncode else ''}", flush=True)
