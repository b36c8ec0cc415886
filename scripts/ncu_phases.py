"""Per-phase instruction and stall accounting of the step kernel from an ncu source-line table
(scripts/ncu_lines.py report N output, every line): executed warp-instructions -> lane-instructions per
particle and stall samples, grouped by the phase each CUDA source line belongs to.
usage: ncu_phases.py lines.txt particles"""
import re, sys
src, particles = sys.argv[1], int(sys.argv[2])
K = {  # pf_kernels.cuh line ranges (this revision) -> phase
    "exchange (a6)": [(672, 698), (1241, 1367)],
    "normalise + resample (a7, a8)": [(348, 671), (1368, 1470)],
    "sample loop glue: gather, stores (a9, a10)": [(699, 876), (1471, 1583)],
    "local reduce + global key (a4, a5)": [(1584, 1668)],
    "epilogue: last CTA, peers (a5)": [(877, 1023), (1669, 99999)],
    "group helpers (barriers, warp reductions, slot / smem addressing), scheduling, TMA": [(1, 347), (1024, 1240)],
}
D = {  # pf_device.cuh line ranges -> contract part
    "Philox4x32-10 (R12, F1)": [(23, 67)],
    "Box-Muller (F2-F4, F6) + joint sin/cos of the kinematics (F5)": [(69, 165), (187, 356)],
    "expq normalise (F7)": [(166, 186), (357, 375)],
    "order keys": [(376, 389)],
}
acc, tot_i, tot_s = {}, 0, 0
for line in open(src):
    m = re.match(r"\s*([\d.]+)%\s+([\d.]+)%\s+(\S+):(\d+)", line)
    if not m:
        h = re.match(r"total warp-inst (\d+)\s+stall samples (\d+)", line)
        if h:
            tot_i, tot_s = int(h.group(1)), int(h.group(2))
        continue
    pi, ps, f, ln = float(m.group(1)), float(m.group(2)), m.group(3), int(m.group(4))
    raw = re.search(r"\[(\d+) (\d+)\]\s*$", line)   # exact counts when ncu_lines.py printed them
    if raw and tot_i:
        pi, ps = 100.0 * int(raw.group(1)) / tot_i, 100.0 * int(raw.group(2)) / max(tot_s, 1)
    table = K if f == "pf_kernels.cuh" else D if f == "pf_device.cuh" else None
    name = "model hooks: sample, forward kinematics, likelihood (F8-F10)" if f == "pf_model.cuh" else f"other ({f})"
    if table:
        name = next((k for k, rs in table.items() if any(a <= ln <= b for a, b in rs)), f"other ({f})")
    a = acc.setdefault(name, [0.0, 0.0])
    a[0] += pi
    a[1] += ps
lane = tot_i * 32 / particles   # (source-page warp-instructions x 32: includes predicated-off lanes)
W = 84
print(f"{'phase (CUDA source line of the executed instruction; inlined helpers count where they are written)':{W}s} {'instr %':>8s} {'lane-instr/particle':>20s} {'stall %':>8s}")
for k, (pi, ps) in sorted(acc.items(), key=lambda kv: -kv[1][0]):
    print(f"{k:{W}s} {pi:8.1f} {pi * lane / 100:20.1f} {ps:8.1f}")
print(f"{'total':{W}s} {100:8.1f} {lane:20.1f} {100:8.1f}")
