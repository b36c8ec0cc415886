"""Dev tool: aggregate an ncu source page (instructions executed, stall samples by reason)
over line ranges of pf_kernels.cuh.  usage: ncu_regions.py report name:lo-hi ..."""
import csv, subprocess, sys, collections
rep = sys.argv[1]
regions = []
for a in sys.argv[2:]:
    n, r = a.split(":"); lo, hi = map(int, r.split("-")); regions.append((n, lo, hi))
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source=cuda,sass"], capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
cur = None; hdr = None
agg = collections.defaultdict(lambda: collections.Counter())
for r in rows:
    if len(r) == 2 and r[0] in ("File Path", "File Name"):
        cur = r[1].split("/")[-1]; continue
    if r and r[0] == "Line No":
        hdr = r; continue
    if hdr and len(r) > 8 and r[0].isdigit():
        d = {"Instructions Executed": r[7], "Warp Stall Sampling (All Samples)": r[4]}; ln = int(r[0])
        name = "other:" + (cur or "?")
        if cur == "pf_kernels.cuh":
            for n, lo, hi in regions:
                if lo <= ln < hi: name = n
        for k, v in d.items():
            try: agg[name][k] += float(v)
            except ValueError: pass
keys = ["Instructions Executed", "Warp Stall Sampling (All Samples)"]
tot = {k: sum(a[k] for a in agg.values()) for k in keys}
print(f"{'region':28s} {'inst%':>6s} {'stall%':>7s}")
for n, a in sorted(agg.items(), key=lambda x: -x[1][keys[1]]):
    print(f"{n:28s} {100*a[keys[0]]/max(tot[keys[0]],1):6.1f} {100*a[keys[1]]/max(tot[keys[1]],1):7.1f}")
