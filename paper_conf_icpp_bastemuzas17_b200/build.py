"""Build libtiles.so in-tree for sm_100a (nvcc + g++), no torch involved.

    python paper_conf_icpp_bastemuzas17_b200/build.py [--force]   (standalone: does not import the package)

Outputs paper_conf_icpp_bastemuzas17_b200/libtiles.so. Objects go to
paper_conf_icpp_bastemuzas17_b200/_build/. cudart is linked statically;
NCCL is dlopen'ed at run time (comm_nccl.cpp).
"""
import glob
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
OBJ = os.path.join(HERE, "_build")
LIB = os.path.join(HERE, "libtiles.so")
CUDA = os.environ.get("CUDA_HOME", "/usr/local/cuda")
NVCC = os.path.join(CUDA, "bin", "nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
# experiment hook (e.g. TILES_NVCC_DEFS="-DTILES_ARRIVE_PER_THREAD=1"); use --force when changing it
EXTRA = os.environ.get("TILES_NVCC_DEFS", "").split()


def _nccl_include():
    try:
        import nvidia.nccl  # noqa: F401
        import nvidia
        for p in nvidia.__path__:
            inc = os.path.join(p, "nccl", "include")
            if os.path.exists(os.path.join(inc, "nccl.h")):
                return inc
    except Exception:
        pass
    for inc in ("/usr/include", "/usr/local/include", os.path.join(CUDA, "include")):
        if os.path.exists(os.path.join(inc, "nccl.h")):
            return inc
    raise RuntimeError("nccl.h not found")


def _run(cmd):
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        sys.stderr.write(" ".join(cmd) + "\n" + r.stdout + r.stderr)
        raise RuntimeError("build step failed: " + os.path.basename(cmd[-1]))
    return r


def build(force=False, verbose=False):
    os.makedirs(OBJ, exist_ok=True)
    headers = glob.glob(os.path.join(CSRC, "*.h*")) + glob.glob(os.path.join(CSRC, "*.cuh")) + \
        [os.path.join(ROOT, "include", "tiles.h")]
    hdr_mtime = max(os.path.getmtime(h) for h in headers)
    inc = ["-I" + os.path.join(ROOT, "include"), "-I" + CSRC, "-I" + os.path.join(CUDA, "include"),
           "-I" + _nccl_include()]
    objs = []
    changed = force or not os.path.exists(LIB)
    for src in sorted(glob.glob(os.path.join(CSRC, "*.cu")) + glob.glob(os.path.join(CSRC, "*.cpp"))):
        obj = os.path.join(OBJ, os.path.basename(src) + ".o")
        objs.append(obj)
        if not force and os.path.exists(obj) and os.path.getmtime(obj) >= max(os.path.getmtime(src), hdr_mtime):
            continue
        changed = True
        if src.endswith(".cu"):
            cmd = [NVCC, *ARCH, "-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC",
                   "-Xptxas", "-v", *EXTRA, *inc, "-c", src, "-o", obj]
        else:
            cmd = ["g++", "-O2", "-std=c++17", "-fPIC", "-Wall", "-Wno-unused-function", *inc,
                   "-c", src, "-o", obj]
        r = _run(cmd)
        if verbose:
            sys.stdout.write(r.stdout + r.stderr)
    if changed:
        _run([NVCC, *ARCH, "-shared", "-cudart", "static", "-o", LIB, *objs, "-ldl", "-lpthread"])
    return LIB


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv))
