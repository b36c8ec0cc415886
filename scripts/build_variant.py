"""Dev tool: build an alternative libpf_b200 with extra -D defines for A/B timing
(e.g. PF_X2_DEFAULT=0), loaded through PF_LIB=<path>.  Not used by tests/bench."""
import os, subprocess, sys, concurrent.futures as cf
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_chitchianasks13_b200 import build as B

def main(out, defs):
    bdir = out + ".objs"
    os.makedirs(bdir, exist_ok=True)
    def comp(src):
        obj = os.path.join(bdir, src.replace(".cu", ".o"))
        subprocess.check_call([B.NVCC, *B.FLAGS, *[f"-D{d}" for d in defs], "-c", os.path.join(B.CSRC, src), "-o", obj],
                              stdout=subprocess.DEVNULL, stderr=subprocess.DEVNULL)
        return obj
    with cf.ThreadPoolExecutor(len(B.SOURCES)) as ex:
        objs = list(ex.map(comp, B.SOURCES))
    subprocess.check_call([B.NVCC, "-shared", "-gencode", "arch=compute_100a,code=sm_100a", "-o", out, *objs, "-lcudart"])
    import shutil; shutil.rmtree(bdir)

if __name__ == "__main__":
    main(os.path.abspath(sys.argv[1]), sys.argv[2:])
