"""Summarise the centralized filter's ncu captures (gpurun_out/r02_central_launches_*.csv: launch list;
gpurun_out/r02_ncu_central_*.csv: --set full raw page) into profiles/r02_ncu_central.txt."""
import collections, csv, os
R = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
G = os.path.join(R, "gpurun_out")
out = open(os.path.join(R, "profiles", "r02_ncu_central.txt"), "w")
out.write("# Centralized filter (NEXT-2), 2^20 particles, d = 9: every kernel of the measured steps.\n"
          "# (1) ncu launch list (gpu__time_duration, DRAM bytes; ncu default cache control, --clock-control none),\n"
          "#     steps 3..6 of scripts/prof_one.py 5 1048576 1 <res> none 0 6;\n"
          "# (2) ncu --set full of one step's kernels (issue activity, warps, registers, long-scoreboard stalls).\n"
          "# RWS: cz_tile_scan + cz_step (the tile prefix is folded into cz_step's prologue below 4M particles).\n")
for res in ("rws", "vose"):
    rows = [r for r in csv.reader(open(os.path.join(G, f"r02_central_launches_{res}.csv"))) if len(r) > 10]
    h = rows[0]; ki = h.index("Kernel Name"); vi = h.index("Metric Value"); ii = h.index("ID"); mi = h.index("Metric Name")
    d = collections.OrderedDict()
    for r in rows[1:]:
        d.setdefault(r[ii], {"k": r[ki].split("(")[0].replace("void ", "").replace("pf::<unnamed>::", "")})[r[mi]] = \
            float(r[vi].replace(",", ""))
    out.write(f"\n== {res.upper()}: launch list (last steps)\n")
    out.write(f"{'kernel':34s} {'us':>8s} {'DRAM rd MB':>11s} {'DRAM wr MB':>11s}\n")
    for k, v in list(d.items())[-10:]:
        out.write(f"{v['k'][:34]:34s} {v['gpu__time_duration.sum']/1e3:8.1f} {v['dram__bytes_read.sum']/1e6:11.2f} "
                  f"{v['dram__bytes_write.sum']/1e6:11.2f}\n")
    rows = list(csv.reader(open(os.path.join(G, f"r02_ncu_central_{res}.csv"))))
    h = rows[0]
    out.write(f"== {res.upper()}: ncu --set full, one step\n")
    cols = ["gpu__time_duration.sum", "smsp__issue_active.avg.pct_of_peak_sustained_active",
            "sm__warps_active.avg.per_cycle_active", "launch__registers_per_thread", "launch__grid_size",
            "smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio", "dram__bytes_read.sum"]
    out.write(f"{'kernel':34s} {'us':>8s} {'issue%':>7s} {'warps':>6s} {'regs':>5s} {'grid':>5s} {'lsb/iss':>8s} {'DRAM rd MB':>10s}\n")
    for r in rows[2:]:
        if len(r) < len(h):
            continue
        k = r[h.index("Kernel Name")].split("(")[0].replace("void ", "").replace("unnamed>::", "")
        v = [r[h.index(c)] for c in cols]
        out.write(f"{k[:34]:34s} {float(v[0]):8.1f} {float(v[1]):7.1f} {float(v[2]):6.1f} {v[3]:>5s} {v[4]:>5s} "
                  f"{float(v[5]):8.2f} {float(v[6]):10.2f}\n")
out.close()
print(open(os.path.join(R, "profiles", "r02_ncu_central.txt")).read())
