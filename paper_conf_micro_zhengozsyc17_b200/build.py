"""Build libvp.so in-tree with nvcc for sm_100a (no torch JIT, no cache dir)."""
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
# VP_LIB_NAME: dev variants (e.g. libvp_m4.so built with other VP_NVCC_EXTRA), still in-tree
LIB_NAME = os.environ.get("VP_LIB_NAME", "libvp.so")
LIB = os.path.join(HERE, LIB_NAME)
OBJDIR = os.path.join(HERE, "build" if LIB_NAME == "libvp.so" else "build_" + LIB_NAME.split(".")[0])
SOURCES = ["vp_host.cu", "vp_tune.cu", "fam_basic.cu", "fam_reyes.cu", "fam_raster.cu", "fam_pyramid.cu", "fam_cfd.cu", "fam_facedet.cu", "fam_qbench.cu", "fam_ldpc.cu", "vp_microbench.cu"]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
FLAGS = ["-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo", "-std=c++17",
         # no FMA contraction, IEEE div/sqrt, no fast math -> bit-exact vs oracle
         "-fmad=false", "-prec-div=true", "-prec-sqrt=true",
         "-Xcompiler", "-fPIC", "-Xptxas", "-v", "--expt-relaxed-constexpr"]
FLAGS += os.environ.get("VP_NVCC_EXTRA", "").split()


def _stale():
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    deps = [os.path.join(CSRC, f) for f in os.listdir(CSRC)] + [os.path.join(HERE, "..", "include", "vp.h")]
    return any(os.path.getmtime(d) > t for d in deps)


def build(force=False, verbose=False, jobs=None):
    if not force and not _stale():
        return LIB
    objs = []
    procs = []
    os.makedirs(OBJDIR, exist_ok=True)
    for src in SOURCES:
        obj = os.path.join(OBJDIR, src.replace(".cu", ".o"))
        cmd = [NVCC, *FLAGS, "-c", os.path.join(CSRC, src), "-o", obj]
        procs.append((src, subprocess.Popen(cmd, stdout=subprocess.PIPE, stderr=subprocess.STDOUT, text=True)))
        objs.append(obj)
    logs = []
    for src, p in procs:
        out, _ = p.communicate()
        logs.append(f"== {src}\n{out}")
        if p.returncode != 0:
            sys.stderr.write(out)
            raise RuntimeError(f"nvcc failed for {src}")
    with open(os.path.join(OBJDIR, "ptxas.log"), "w") as f:
        f.write("\n".join(logs))
    cmd = [NVCC, "-shared", "-gencode", "arch=compute_100a,code=sm_100a", "-o", LIB, *objs, "-lcudart"]
    subprocess.run(cmd, check=True)
    if verbose:
        print("\n".join(logs))
    return LIB


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose="-v" in sys.argv)
    print(LIB)
