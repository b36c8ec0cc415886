"""Executed-instruction histogram by SASS opcode from an ncu report (source page, sass rows).
usage: ncu_opcodes.py report.ncu-rep particles [top]"""
import csv, subprocess, sys, re, collections
rep, parts = sys.argv[1], float(sys.argv[2])
top = int(sys.argv[3]) if len(sys.argv) > 3 else 40
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source=sass"], capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
hdr = None; agg = collections.Counter(); tot = 0
for r in rows:
    if r and r[0] == "Address": hdr = r; continue
    if hdr and len(r) == len(hdr):
        d = dict(zip(hdr, r))
        try: ie = int(d.get("Instructions Executed", "0") or 0)
        except ValueError: continue
        src = d.get("Source", "")
        op = re.sub(r"^@!?U?P\w+\s+", "", src.strip()).split(" ")[0]
        agg[op.split(".")[0]] += ie; tot += ie
print(f"total {tot*32/parts:.0f} lane-instr/particle")
for op, n in agg.most_common(top):
    print(f"  {op:12s} {n*32/parts:8.1f}")
