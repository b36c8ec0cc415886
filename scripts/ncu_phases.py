"""Per-phase instruction and stall accounting of the step kernel from an ncu source-line table
(scripts/ncu_lines.py report N output, every line): executed warp-instructions -> lane-instructions per
particle and stall samples, grouped by the phase each CUDA source line belongs to.
usage: ncu_phases.py lines.txt particles"""
import os, re, sys
src, particles = sys.argv[1], int(sys.argv[2])
# pf_kernels.cuh line ranges -> phase, found from the section markers of the source file itself
KSRC = open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                         "paper_conf_ipps_chitchianasks13_b200", "csrc", "pf_kernels.cuh")).read().split("\n")


def _at(pat, start=0):
    for i in range(start, len(KSRC)):
        if pat in KSRC[i]:
            return i + 1   # 1-based line number
    raise SystemExit(f"marker not found: {pat}")


_scan = _at("X slot_scan_smem(") - 1
_nbr = _at("long long neighbor_row(")
_noise = _at("struct NoiseGen {")
_peer = _at("static __device__ void peer_halo_rows(")
_kern = _at(") pf_step_kernel(")
_mbf0 = _at("auto mb_fetch = ", _kern)
_mbf1 = _at("  };", _mbf0)
_a6 = _at("// ---- a6 exchange", _kern)
_a7 = _at("// ---- a7 normalise", _a6)
_a9 = _at("// ---- a9 gather", _a7)
_a4 = _at("// ---- a4 local reduce", _a9)
_a5 = _at("// ---- a5: the last CTA", _a4)
_end = _at("pf_resample_debug_kernel(", _a5)
K = {
    "exchange (a6)": [(_nbr, _noise - 1), (_mbf0, _mbf1), (_a6, _a7 - 1)],
    "normalise + resample (a7, a8)": [(_scan, _nbr - 1), (_a7, _a9 - 1)],
    "sample loop glue: gather, stores (a9, a10)": [(_noise, _peer - 1), (_a9, _a4 - 1)],
    "local reduce + global key (a4, a5)": [(_a4, _a5 - 1)],
    "epilogue: last CTA, peers (a5)": [(_peer, _kern - 1), (_a5, _end)],
    "group helpers (barriers, warp reductions, slot / smem addressing), scheduling, TMA": [(1, _scan - 1), (_kern, _a6 - 1)],
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
