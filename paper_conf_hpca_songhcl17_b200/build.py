"""Build libpcnn.so in-tree with nvcc for sm_100a (no JIT, no torch extension).

    python -m paper_conf_hpca_songhcl17_b200.build [--force] [--verbose]

Objects are compiled in parallel into build/ and linked into
paper_conf_hpca_songhcl17_b200/libpcnn.so (static cudart, so the library has
no runtime dependency beyond the CUDA driver).
"""
import concurrent.futures as cf
import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
BUILD = os.path.join(ROOT, "build", "pcnn")
LIB = os.path.join(PKG, "libpcnn.so")
# experiments variant (tcgen05 barrier-wait counters and the PCNN_* tuning /
# A-B environment switches compiled in), used by tools/ through PCNN_LIB;
# never the product library
PROF_LIB = os.path.join(ROOT, "build", "prof", "libpcnn_prof.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")

ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
FLAGS = ["-O3", "-std=c++17", "-lineinfo", "-Xcompiler", "-fPIC",
         "-I" + os.path.join(ROOT, "include")]
SOURCES = ["kernels_tc.cu", "kernels_fc.cu", "kernels_simt.cu", "runtime.cu", "svd.cpp"]
HEADERS = ["pcnn_internal.h", "budget.cuh", "svd.h", "lrn_math.cuh", "tc_ptx.cuh"]


def _newer(src_list, target):
    if not os.path.exists(target):
        return True
    t = os.path.getmtime(target)
    return any(os.path.getmtime(s) > t for s in src_list)


def build(force=False, verbose=False, prof=False):
    bdir = BUILD + ("_prof" if prof else "")
    lib = PROF_LIB if prof else LIB
    flags = FLAGS + (["-DPCNN_TC_PROF=1", "-DPCNN_EXPERIMENTS=1"] if prof else [])
    os.makedirs(bdir, exist_ok=True)
    os.makedirs(os.path.dirname(lib), exist_ok=True)
    hdrs = [os.path.join(CSRC, h) for h in HEADERS] + [
        os.path.join(ROOT, "include", "pcnn.h")]
    objs, jobs = [], []
    for src in SOURCES:
        s = os.path.join(CSRC, src)
        o = os.path.join(bdir, src + ".o")
        objs.append(o)
        if force or _newer([s] + hdrs, o):
            extra = ["-Xptxas", "-v"] if verbose and src.endswith(".cu") else []
            jobs.append([NVCC] + ARCH + flags + extra + ["-c", s, "-o", o])

    def run(cmd):
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError("nvcc failed:\n%s\n%s" % (" ".join(cmd), r.stderr))
        return r.stderr

    with cf.ThreadPoolExecutor(max_workers=len(SOURCES)) as ex:
        for out in ex.map(run, jobs):
            if verbose and out:
                sys.stderr.write(out)
    if force or jobs or _newer(objs, lib):
        tmp = lib + ".tmp%d" % os.getpid()
        run([NVCC] + ARCH + ["-shared", "-o", tmp] + objs + ["-lpthread"])
        os.replace(tmp, lib)
    return lib


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose="--verbose" in sys.argv,
                prof="--prof" in sys.argv))
