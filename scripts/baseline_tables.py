"""Regenerate the Results section of BASELINE.md from profiles/r02_bench.json,
profiles/r02_bench_reference.json, profiles/ncu_summary.json and profiles/r02_sweeps.jsonl."""
import json, os, re
R = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
b = json.loads(open(os.path.join(R, "profiles/r02_bench.json")).read().strip().splitlines()[-1])
ref = json.loads(open(os.path.join(R, "profiles/r02_bench_reference.json")).read().strip().splitlines()[-1])
ncu = json.load(open(os.path.join(R, "profiles/ncu_summary.json")))
sw = [json.loads(l) for l in open(os.path.join(R, "profiles/r02_sweeps.jsonl"))]
big = {(d["n_joints"], d["N"], d["resampler"]): d for d in sw if d["sweep"] in ("res", "count", "dim")}
c5 = big[(5, 65536, "rws")]; e8 = big[(5, 390625, "rws")]
peak = b["roofline"]["peak"]
L = []
L.append("## Results (round 2, one B200, `profiles/r02_*`)\n")
L.append("Headline (`bench.py`, config C2: medium arm d = 9, 4096 × 256 = 2²⁰ particles, ring t = 1, RWS; L2 flushed")
L.append(f"before every timed step; SM clock {b['clocks']['sm_mhz']:.0f} MHz, throttle reasons {b['clocks']['reasons'] or 'none'}):\n")
L.append("| Quantity | Value |\n|---|---|")
L.append(f"| State estimates/s at 1M particles (device-resident inputs) | **{b['estimates_per_s']:.0f}** ({1e3*b['ms_per_step']:.1f} µs/step; target ≥ 1 000) |")
L.append(f"| Particle-steps/s | {b['value']:.3g} |")
L.append(f"| End to end through the C ABI (host z/u in, estimate out, every step; host clock) | {b['e2e']['estimates_per_s']:.0f} estimates/s ({1e3*b['e2e']['ms_per_step']:.1f} µs/step) |")
L.append(f"| Vose instead of RWS | {b['vose']['estimates_per_s']:.0f} estimates/s |")
L.append(f"| L2-resident back-to-back steps (no flush; context) | {b['l2_resident']['estimates_per_s']:.0f} estimates/s |")
L.append(f"| Step-kernel HBM roofline (algorithmic {b['roofline']['bytes_per_launch']/1e6:.1f} MB / launch) | {b['roofline']['achieved']:.0f} GB/s = {100*b['roofline']['frac']:.0f} % of the measured {peak:.0f} GB/s; ncu DRAM traffic {ncu['C2']['dram_bytes_per_launch']/1e6:.1f} MB / launch |")
L.append(f"| Issue roofline (the binding one, DESIGN.md §6) | {b['roofline_issue']['instr_per_particle']:.0f} lane-instructions / particle, {100*b['roofline_issue']['frac']:.0f} % of 148 × 4 × 32 per clock |")
for blk, lab in (("c5_weak", "C5 shard (bench, device-timed): 16M particles d = 9, RWS"), ("c4_strong", "C4 (bench, device-timed): 16M particles d = 32, Vose")):
    v = b[blk]
    L.append(f"| {lab} | {1e3*v['ms_per_step']:.0f} µs/step = {v['particle_steps_per_s']:.3g} particle-steps/s; {v['roofline']['achieved']:.0f} GB/s = {100*v['roofline']['frac']:.0f} % of HBM |")
for key, lab in (("C2_vose", "C2 with Vose"), ("C5_nj5_16M", "16M particles d = 9 (RWS)"), ("C5_nj5_16M_vose", "16M particles d = 9 (Vose)"), ("C4_nj28_16M_rws", "16M particles d = 32 (RWS)"), ("C4_nj28_16M_vose", "16M particles d = 32 (Vose, config C4)")):
    v = ncu[key]
    d = 32 if "nj28" in key else 9
    n = 1048576 if key.startswith("C2") else 16777216
    alg = n * 8 * (d + 1)
    t = v["gpu__time_duration.sum"] * (1e-6 if v["gpu__time_duration.sum"] > 10 else 1e-3)
    L.append(f"| {lab}, ncu | {1e6*t:.0f} µs = {alg/t/1e9:.0f} GB/s algorithmic ({100*alg/t/1e9/peak:.0f} % of HBM), "
             f"{v['lane_instr_per_particle']:.0f} lane-instr/particle, issue active {v['smsp__issue_active.avg.pct_of_peak_sustained_active']:.0f} % |")
L.append(f"| 10⁸ particles (d = 9, sweep) | {e8['us_per_step']:.0f} µs/step = {e8['hbm_gbs_algorithmic']:.0f} GB/s ({100*e8['hbm_gbs_algorithmic']/peak:.0f} %) |")
L.append(f"| CPU oracle on all {b['cpu_baseline']['cores']} host cores ({b['cpu_baseline']['cpu_model']}) | {b['cpu_baseline']['value']:.3g} particle-steps/s (one process per core); 1 core {b['cpu_baseline']['single_core']['value']:.3g}; reference arm {ref['value']:.3g} |")
cen = [json.loads(l) for l in open(os.path.join(R, "profiles/r02_central_sweep.jsonl"))]
cz = {(d["particles"], d["resampler"]): d["us_per_step"] for d in cen}
L.append(f"| Centralized filter, 2²⁰ particles (NEXT-2; round 1: RWS 113, Vose 149 µs) | RWS {cz[(1048576, 'rws')]:.0f} µs, Vose {cz[(1048576, 'vose')]:.0f} µs per step (Vose faster, the paper's Fig. 5 finding) |")
L.append("| 2 ranks sharing one GPU (peer transport, functional check; `profiles/r02_bench_2rank.json`) | completes; time-sliced on one device, not a scaling number |")
L.append("| Paper (GTX 580/680, HD 7970; Table III) | \"a few hundred\" estimates/s at 1M (context only) |\n")
L.append("Sweeps (`scripts/sweeps.py`, device-resident inputs, L2 flushed per step):\n")
L.append("| Sweep | d | m | N | particles | resampler | X, t | policy | µs/step | particle-steps/s | alg. HBM GB/s |")
L.append("|---|---|---|---|---|---|---|---|---|---|---|")
for d in sw:
    pol = d["policy"] if d["policy"] == "always" else f"{d['policy']} {d['policy_value']}"
    L.append(f"| {d['sweep']} | {d['d']} | {d['m']} | {d['N']} | {d['particles']} | {d['resampler']} | {d['topo']} {d['t']} | {pol} | "
             f"{d['us_per_step']:.1f} | {d['particle_steps_per_s']:.3g} | {d['hbm_gbs_algorithmic']:.0f} |")
txt = open(os.path.join(R, "BASELINE.md")).read()
a = txt.index("## Results (round")
z = txt.index("### Estimation accuracy on B200")
open(os.path.join(R, "BASELINE.md"), "w").write(txt[:a] + "\n".join(L) + "\n\n" + txt[z:])
print("\n".join(L[:20]))
