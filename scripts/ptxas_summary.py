"""Print registers / spills / smem per step-kernel instantiation from build/*.ptxas.log."""
import glob, os, re, sys
root = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "paper_conf_ipps_chitchianasks13_b200", "build")
for f in sorted(glob.glob(os.path.join(root, "*.ptxas.log"))):
    cur = None
    for line in open(f):
        m = re.search(r"Compiling entry function '(\S+)'", line)
        if m:
            n = m.group(1)
            k = re.search(r"pf_step_kernelILi(\d+)ELi(\d+)ELi(\d)E", n)
            r = re.search(r"resample_debug_kernelILi(\d+)ELi(\d)E", n)
            cur = f"step nj={k.group(1)} m={k.group(2)} res={k.group(3)}" if k else (f"rdebug m={r.group(1)} res={r.group(2)}" if r else n[:40])
            continue
        m = re.search(r"(\d+) bytes spill stores", line)
        if m and cur: spill = m.group(1)
        m = re.search(r"Used (\d+) registers", line)
        if m and cur:
            print(f"{cur:32s} regs={m.group(1):>4} spill={spill}")
            cur = None
