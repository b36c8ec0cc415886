"""Summarise ncu reports into profiles/: key raw metrics per kernel launch.
usage: ncu_summary.py name=report.ncu-rep[:particles] ... > out.txt ; also updates profiles/ncu_summary.json"""
import csv, json, os, subprocess, sys
KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "smsp__inst_executed.sum",
        "sm__warps_active.avg.per_cycle_active", "launch__registers_per_thread", "launch__grid_size",
        "launch__block_size", "launch__shared_mem_per_block_dynamic", "launch__occupancy_limit_registers",
        "launch__occupancy_limit_shared_mem", "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active", "sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "sm__cycles_elapsed.avg.per_second",
        "smsp__average_warps_issue_stalled_barrier_per_issue_active.ratio",
        "smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio",
        "smsp__average_warps_issue_stalled_wait_per_issue_active.ratio",
        "smsp__average_warps_issue_stalled_no_instruction_per_issue_active.ratio",
        "smsp__average_warps_issue_stalled_math_pipe_throttle_per_issue_active.ratio",
        "smsp__average_warps_issue_stalled_not_selected_per_issue_active.ratio"]
root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
js_path = os.path.join(root, "profiles", "ncu_summary.json")
js = json.load(open(js_path)) if os.path.exists(js_path) else {}
for arg in sys.argv[1:]:
    name, rest = arg.split("=", 1)
    rep, parts = (rest.split(":") + [None])[:2]
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    h, units, v = rows[0], rows[1], rows[2]
    print(f"== {name}: {rep} ({v[h.index('Kernel Name')][:90]})")
    rec = {}
    for k in KEYS:
        if k in h:
            i = h.index(k)
            print(f"  {k:75s} {v[i]:>16s} {units[i]}")
            try:
                val = float(v[i].replace(",", ""))
            except ValueError:
                continue
            rec[k] = val
            unit = units[i]
            if k.startswith("dram__bytes"):
                scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(unit, 1)
                rec[k + ".bytes"] = val * scale
            if k == "gpu__time_duration.sum":
                rec["duration_s"] = val * {"nsecond": 1e-9, "usecond": 1e-6, "msecond": 1e-3, "second": 1}.get(unit, 1)
    if "dram__bytes_read.sum.bytes" in rec:
        rec["dram_bytes_per_launch"] = rec["dram__bytes_read.sum.bytes"] + rec["dram__bytes_write.sum.bytes"]
        print(f"  dram bytes per launch = {rec['dram_bytes_per_launch']:.4g}")
    if parts:
        rec["lane_instr_per_particle"] = rec["smsp__inst_executed.sum"] * 32 / float(parts)
        print(f"  lane instructions per particle = {rec['lane_instr_per_particle']:.0f}")
    js[name] = rec
json.dump(js, open(js_path, "w"), indent=1)
