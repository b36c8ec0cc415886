"""A/B timing of an environment toggle, interleaved: ab_env.py NJ M N RES VAR [reps]"""
import os, subprocess, sys, statistics
nj, m, N, res, var = sys.argv[1:6]
reps = int(sys.argv[6]) if len(sys.argv) > 6 else 3
t = {"off": [], "on": []}
for r in range(reps):
    for k in ("off", "on"):
        env = dict(os.environ)
        if k == "on":
            env[var] = "1"
        out = subprocess.run([sys.executable, os.path.join(os.path.dirname(__file__), "time_one.py"), nj, m, N, res, "30"],
                             env=env, capture_output=True, text=True).stdout
        t[k].append(float(out.split(res + ":")[1].split("us")[0]))
for k in t:
    print(f"nj={nj} m={m} N={N} {res} {var}={k}: median {statistics.median(t[k]):.1f} us {t[k]}")
