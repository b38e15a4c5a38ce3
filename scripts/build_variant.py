"""Build libtri.so with extra nvcc flags into build_var/NAME/ (A/B experiments;
load it with TRI_LIB_PATH=build_var/NAME/libtri.so).  usage: build_variant.py NAME FLAG..."""
import concurrent.futures as cf
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_icpp_kimwch11_b200 import _build as B  # noqa: E402

name, extra = sys.argv[1], sys.argv[2:]
# TRI_CSRC=dir: build another copy of the sources (e.g. a git revision exported for an A/B)
CSRC = os.environ.get("TRI_CSRC", B.CSRC)
out = os.path.join(ROOT, "build_var", name)
os.makedirs(out, exist_ok=True)


def comp(src):
    obj = os.path.join(out, src.replace(".cu", ".o"))
    subprocess.check_call([B.NVCC, *B.ARCH, *B.FLAGS, *extra, "-I", B.INCLUDE, "-I", CSRC, "-c", "-o", obj,
                           os.path.join(CSRC, src)], stderr=subprocess.DEVNULL)
    return obj


with cf.ThreadPoolExecutor(8) as ex:
    objs = list(ex.map(comp, B.SOURCES))
subprocess.check_call([B.NVCC, *B.ARCH, "-shared", "-o", os.path.join(out, "libtri.so"), *objs])
print(os.path.join(out, "libtri.so"))
