"""Build the in-tree C-ABI library libtri.so (sm_100a) with nvcc.

One object per kernel family (csrc/l_*.cu), compiled in parallel, linked into
one shared library.  The .so is git-ignored but travels to the GPU box with the
gpurun snapshot.
"""
import concurrent.futures as cf
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
INCLUDE = os.path.join(ROOT, "include")
LIB = os.path.join(HERE, "libtri.so")
OBJ = os.path.join(HERE, "build_obj")
SOURCES = ["tri_api.cu", "host_util.cu", "l_scan.cu", "l_split.cu", "l_stream.cu", "l_fused.cu", "l_small.cu",
           "l_strided.cu"]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
FLAGS = ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC,-fvisibility=hidden",
         "--expt-relaxed-constexpr", "-Xptxas", "-warn-spills"]


def _deps():
    files = [os.path.join(CSRC, f) for f in os.listdir(CSRC)]
    files.append(os.path.join(INCLUDE, "tri.h"))
    return files


def stale():
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(f) > t for f in _deps())


def _compile(src, verbose):
    obj = os.path.join(OBJ, os.path.splitext(src)[0] + ".o")
    cmd = [NVCC, *ARCH, *FLAGS, "-I", INCLUDE, "-I", CSRC, "-c", "-o", obj, os.path.join(CSRC, src)]
    if verbose:
        cmd += ["-Xptxas", "-v"]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.stderr:
        sys.stderr.write(r.stderr)
    if r.returncode:
        raise subprocess.CalledProcessError(r.returncode, cmd)
    return obj


def build(force=False, verbose=False, only=None):
    """Compile every source (or only the named ones, reusing the other objects) and link."""
    if not force and not stale() and only is None:
        return LIB
    os.makedirs(OBJ, exist_ok=True)
    srcs = SOURCES if only is None else [s for s in SOURCES if s in only]
    with cf.ThreadPoolExecutor(max_workers=min(len(srcs), os.cpu_count() or 4)) as ex:
        list(ex.map(lambda s: _compile(s, verbose), srcs))
    objs = [os.path.join(OBJ, os.path.splitext(s)[0] + ".o") for s in SOURCES]
    subprocess.check_call([NVCC, *ARCH, "-shared", "-o", LIB, *objs])
    return LIB


if __name__ == "__main__":
    only = [a for a in sys.argv[1:] if a.endswith(".cu")] or None
    build(force=True, verbose="-v" in sys.argv, only=only)
    print(LIB)
