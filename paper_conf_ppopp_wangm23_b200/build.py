"""Build libtg.so in-tree with nvcc for sm_100a (no JIT cache, no torch extension).

    python -m paper_conf_ppopp_wangm23_b200.build [--force]

TG_TRACE=1 builds the debug variant libtg_trace.so (GEMM clock64 trace, see
k_gemm_tc.cu; loaded only when TG_LIB points at it, e.g. by tools/gemm_trace.py).
"""
import concurrent.futures as cf
import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
TRACE = os.environ.get("TG_TRACE") == "1"
LIB = os.path.join(PKG, "libtg_trace.so" if TRACE else "libtg.so")
BUILD = os.path.join(CSRC, "build_trace" if TRACE else "build")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
FLAGS = ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC", "-Xptxas", "-v",
         "--expt-relaxed-constexpr", "-I", os.path.join(ROOT, "include")]
if TRACE:
    FLAGS.append("-DTG_TC_TRACE")
# NOTE: no --use_fast_math: Eq. 8 needs the accurate cosf and uncontracted mul/add (R5).


def sources():
    return sorted(os.path.join(CSRC, f) for f in os.listdir(CSRC) if f.endswith(".cu"))


def _stale():
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    deps = [os.path.join(CSRC, f) for f in os.listdir(CSRC)] + [os.path.join(ROOT, "include", "tg.h")]
    return any(os.path.getmtime(d) > t for d in deps)


def _compile(src, log):
    obj = os.path.join(BUILD, os.path.basename(src)[:-3] + ".o")
    extra = os.environ.get("TG_EXTRA_FLAGS_" + os.path.basename(src)[:-3].upper(), "").split()  # experiments
    cmd = [NVCC, *ARCH, *FLAGS, *extra, "-c", src, "-o", obj]
    r = subprocess.run(cmd, capture_output=True, text=True)
    with open(log, "a") as f:
        f.write(" ".join(cmd) + "\n" + r.stdout + r.stderr + "\n")
    if r.returncode != 0:
        raise RuntimeError(f"nvcc failed for {src}:\n{r.stderr[-4000:]}")
    return obj


def build(force=False, verbose=False):
    if not force and not _stale():
        return LIB
    os.makedirs(BUILD, exist_ok=True)
    log = os.path.join(BUILD, "ptxas.log")
    open(log, "w").close()
    with cf.ThreadPoolExecutor(max_workers=min(8, os.cpu_count() or 1)) as ex:
        objs = list(ex.map(lambda s: _compile(s, log), sources()))
    tmp = LIB + ".tmp"
    cmd = [NVCC, *ARCH, "-shared", "-o", tmp, *objs]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"link failed:\n{r.stderr[-4000:]}")
    os.replace(tmp, LIB)
    if verbose:
        print(open(log).read())
    return LIB


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv))
