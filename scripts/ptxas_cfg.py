"""Dev tool: registers / spill bytes of every pf_step_kernel instantiation in build/*.ptxas.log,
keyed by model and KCfg (m, res, gw, s, nstage, unr, minb).  usage: ptxas_cfg.py [filter]"""
import glob, os, re, sys
root = os.environ.get("PTXAS_DIR") or os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "paper_conf_ipps_chitchianasks13_b200", "build")
flt = sys.argv[1] if len(sys.argv) > 1 else ""
for f in sorted(glob.glob(os.path.join(root, "*.ptxas.log"))):
    cur, spill = None, "?"
    for line in open(f):
        m = re.search(r"Compiling entry function '(\S+)'", line)
        if m:
            n = m.group(1)
            k = re.search(r"pf_step_kernelINS_4KCfgINS_\d+(\w+?)EELi(\d+)ELi(\d)ELi(\d)ELi(\d+)ELi(\d)ELi(\d+)ELi(\d+)E", n)
            cur = (f"{os.path.basename(f)[:12]:12s} {k.group(1)[:22]:22s} m={k.group(2):>4} res={k.group(3)} gw={k.group(4)} "
                   f"s={k.group(5)} nst={k.group(6)} unr={k.group(7)} minb={k.group(8)}") if k else None
            continue
        m = re.search(r"(\d+) bytes spill stores", line)
        if m and cur: spill = m.group(1)
        m = re.search(r"Used (\d+) registers", line)
        if m and cur:
            if flt in cur:
                print(f"{cur}  regs={m.group(1):>4} spill={spill}")
            cur = None
