"""Summarise an ncu source page by CUDA line: instructions executed and stall samples.
usage: ncu_lines.py report.ncu-rep [top]"""
import csv, subprocess, sys
rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source=cuda,sass"],
                     capture_output=True, text=True).stdout
cur = None; agg = []; tot_i = tot_s = 0
for r in csv.reader(out.splitlines()):
    if len(r) == 2 and r[0] in ("File Path", "File Name"):
        cur = r[1].split("/")[-1]; continue
    if len(r) > 8 and r[0].isdigit():
        try:
            ie = int(r[7]); ss = int(r[4])
        except ValueError:
            continue
        if ie or ss:
            agg.append((ie, ss, cur, int(r[0]), r[1].strip()[:90])); tot_i += ie; tot_s += ss
agg.sort(reverse=True)
print(f"total warp-inst {tot_i}  stall samples {tot_s}")
for ie, ss, f, ln, src in agg[:top]:
    print(f"{100*ie/tot_i:5.1f}% {100*ss/max(tot_s,1):5.1f}%  {f}:{ln:<4} {src}  [{ie} {ss}]")
