"""Build libsshopm.so in-tree for sm_100a.

    python -m paper_conf_ipps_ballardkp11_b200.build [--force] [-j N] [--ptxas-v]

Compiles csrc/sshopm_instance.cu once per SHAPE(m, n) line of csrc/shapes.def
(-DSSHOPM_M/-DSSHOPM_N), plus the API / dedup / host-pipeline units, and links
them into paper_conf_ipps_ballardkp11_b200/_lib/libsshopm.so.  Objects go to
build/ (git-ignored); a unit is rebuilt when any csrc/ or include/ file is
newer than its object.
"""
import argparse
import glob
import os
import re
import shutil
import subprocess
import sys
from concurrent.futures import ThreadPoolExecutor

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
INCLUDE = os.path.join(ROOT, "include")
# SSHOPM_BUILD_DIR / SSHOPM_LIB_OUT: build a variant library elsewhere (tools/ sweeps), never over the product .so
BUILD = os.environ.get("SSHOPM_BUILD_DIR") or os.path.join(ROOT, "build")
LIB = os.environ.get("SSHOPM_LIB_OUT") or os.path.join(PKG, "_lib", "libsshopm.so")
LIBDIR = os.path.dirname(LIB)

ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
NVCC_FLAGS = ["-O3", "-std=c++17", "-lineinfo", "-Xcompiler", "-fPIC", "--expt-relaxed-constexpr",
              "-I" + INCLUDE, "-I" + CSRC] + ARCH + os.environ.get("SSHOPM_NVCC_EXTRA", "").split()


def nvcc():
    for c in (os.environ.get("NVCC"), "/usr/local/cuda/bin/nvcc", shutil.which("nvcc")):
        if c and os.path.exists(c):
            return c
    raise RuntimeError("nvcc not found")


def shapes():
    with open(os.path.join(CSRC, "shapes.def")) as f:
        sh = [(int(a), int(b)) for a, b in re.findall(r"^SHAPE\((\d+),\s*(\d+)\)", f.read(), re.M)]
    return sh


def _newest_source():
    files = glob.glob(os.path.join(CSRC, "*")) + glob.glob(os.path.join(INCLUDE, "*"))
    return max(os.path.getmtime(f) for f in files)


def _units():
    u = []
    for m, n in shapes():
        u.append((os.path.join(CSRC, "sshopm_instance.cu"), os.path.join(BUILD, f"inst_{m}_{n}.o"),
                  [f"-DSSHOPM_M={m}", f"-DSSHOPM_N={n}"]))
    for src in ("sshopm_api.cu", "host_pipeline.cu", "general.cu", "blocked.cu"):
        u.append((os.path.join(CSRC, src), os.path.join(BUILD, src.replace(".cu", ".o")), []))
    return u


def build(force=False, jobs=None, ptxas_v=False, verbose=False):
    os.makedirs(BUILD, exist_ok=True)
    os.makedirs(LIBDIR, exist_ok=True)
    newest = _newest_source()
    todo = [u for u in _units() if force or not os.path.exists(u[1]) or os.path.getmtime(u[1]) < newest]
    cc = nvcc()

    def run(u):
        src, obj, defs = u
        cmd = [cc, "-c", src, "-o", obj] + NVCC_FLAGS + defs + (["-Xptxas", "-v"] if ptxas_v else [])
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"nvcc failed for {os.path.basename(obj)}:\n{' '.join(cmd)}\n{r.stdout}\n{r.stderr}")
        return obj, r.stderr

    if todo:
        with ThreadPoolExecutor(max_workers=jobs or os.cpu_count() or 4) as ex:
            for obj, err in ex.map(run, todo):
                if verbose or ptxas_v:
                    print(f"== {os.path.basename(obj)}\n{err}")
    objs = [u[1] for u in _units()]
    if todo or not os.path.exists(LIB) or os.path.getmtime(LIB) < max(os.path.getmtime(o) for o in objs):
        cmd = [cc, "-shared", "-o", LIB] + objs + ARCH + ["-Xcompiler", "-fPIC"]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"link failed:\n{' '.join(cmd)}\n{r.stdout}\n{r.stderr}")
    return LIB


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--force", action="store_true")
    ap.add_argument("-j", type=int, default=None)
    ap.add_argument("--ptxas-v", action="store_true")
    a = ap.parse_args()
    print(build(a.force, a.j, a.ptxas_v))


if __name__ == "__main__":
    sys.exit(main())
