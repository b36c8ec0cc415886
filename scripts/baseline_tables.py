"""Regenerate the Results section of BASELINE.md from profiles/r01_bench_c2.json,
profiles/r01_bench_reference.json, profiles/ncu_summary.json and profiles/r01_sweeps.jsonl."""
import json, os, re
R = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
b = json.load(open(os.path.join(R, "profiles/r01_bench_c2.json")))
ref = json.load(open(os.path.join(R, "profiles/r01_bench_reference.json")))
ncu = json.load(open(os.path.join(R, "profiles/ncu_summary.json")))
sw = [json.loads(l) for l in open(os.path.join(R, "profiles/r01_sweeps.jsonl"))]
big = {(d["n_joints"], d["N"], d["resampler"]): d for d in sw if d["sweep"] in ("res", "count", "dim")}
c5 = big[(5, 65536, "rws")]; e8 = big[(5, 390625, "rws")]
peak = b["roofline"]["peak"]
L = []
L.append("## Results (round 1, one B200, `profiles/r01_*`)\n")
L.append("Headline (`bench.py`, config C2: medium arm d = 9, 4096 × 256 = 2²⁰ particles, ring t = 1, RWS; L2 flushed")
L.append(f"before every timed step; SM clock {b['clocks']['sm_mhz']:.0f} MHz, throttle reasons {b['clocks']['reasons'] or 'none'}):\n")
L.append("| Quantity | Value |\n|---|---|")
L.append(f"| State estimates/s at 1M particles (device-resident inputs) | **{b['estimates_per_s']:.0f}** ({1e3*b['ms_per_step']:.1f} µs/step; target ≥ 1 000) |")
L.append(f"| Particle-steps/s | {b['value']:.3g} |")
L.append(f"| End to end through the C ABI (host z/u in, estimate out, every step) | {b['e2e']['estimates_per_s']:.0f} estimates/s ({1e3*b['e2e']['ms_per_step']:.1f} µs/step) |")
L.append(f"| Vose instead of RWS | {b['vose']['estimates_per_s']:.0f} estimates/s |")
L.append(f"| L2-resident back-to-back steps (no flush; context) | {b['l2_resident']['estimates_per_s']:.0f} estimates/s |")
L.append(f"| Step-kernel HBM roofline (algorithmic {b['roofline']['bytes_per_launch']/1e6:.1f} MB / launch) | {b['roofline']['achieved']:.0f} GB/s = {100*b['roofline']['frac']:.0f} % of the measured {peak:.0f} GB/s; ncu DRAM traffic {ncu['C2']['dram_bytes_per_launch']/1e6:.1f} MB / launch |")
L.append(f"| Issue roofline (the binding one, DESIGN.md §6) | {b['roofline_issue']['instr_per_particle']:.0f} lane-instructions / particle, {100*b['roofline_issue']['frac']:.0f} % of 148 × 4 × 32 per clock |")
for key, lab in (("C5_nj5_16M", "16M particles d = 9 (RWS)"), ("C4_nj28_16M_rws", "16M particles d = 32 (RWS)"), ("C4_nj28_16M_vose", "16M particles d = 32 (Vose, config C4)")):
    v = ncu[key]
    d = 9 if "nj5" in key else 32
    alg = 16777216 * 8 * (d + 1)
    t = v["gpu__time_duration.sum"] * (1e-6 if v["gpu__time_duration.sum"] > 10 else 1e-3)
    L.append(f"| {lab}, ncu | {1e6*t:.0f} µs = {alg/t/1e9:.0f} GB/s algorithmic ({100*alg/t/1e9/peak:.0f} % of HBM), "
             f"{v['lane_instr_per_particle']:.0f} lane-instr/particle, issue active {v['smsp__issue_active.avg.pct_of_peak_sustained_active']:.0f} % |")
L.append(f"| 10⁸ particles (d = 9, sweep) | {e8['us_per_step']:.0f} µs/step = {e8['hbm_gbs_algorithmic']:.0f} GB/s ({100*e8['hbm_gbs_algorithmic']/peak:.0f} %) |")
L.append(f"| CPU oracle (plain C, 1 core) | {b['cpu_baseline']['value']:.3g} particle-steps/s ({b['cpu_baseline']['sample']}); reference arm {ref['value']:.3g} |")
L.append("| 2 ranks sharing one GPU (peer transport, functional check; `profiles/r01_bench_2rank_shared_gpu.json`) | completes; time-sliced on one device, not a scaling number |")
L.append("| Paper (GTX 580/680, HD 7970; Table III) | \"a few hundred\" estimates/s at 1M (context only) |\n")
L.append("Sweeps (`scripts/sweeps.py`, device-resident inputs, L2 flushed per step):\n")
L.append("| Sweep | d | m | N | particles | resampler | X, t | policy | µs/step | particle-steps/s | alg. HBM GB/s |")
L.append("|---|---|---|---|---|---|---|---|---|---|---|")
for d in sw:
    pol = d["policy"] if d["policy"] == "always" else f"{d['policy']} {d['policy_value']}"
    L.append(f"| {d['sweep']} | {d['d']} | {d['m']} | {d['N']} | {d['particles']} | {d['resampler']} | {d['topo']} {d['t']} | {pol} | "
             f"{d['us_per_step']:.1f} | {d['particle_steps_per_s']:.3g} | {d['hbm_gbs_algorithmic']:.0f} |")
txt = open(os.path.join(R, "BASELINE.md")).read()
a = txt.index("## Results (round 1")
z = txt.index("### Estimation accuracy on B200")
open(os.path.join(R, "BASELINE.md"), "w").write(txt[:a] + "\n".join(L) + "\n\n" + txt[z:])
print("\n".join(L[:20]))
