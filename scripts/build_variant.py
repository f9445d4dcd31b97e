"""Build an A/B variant of libwdntt.so with extra nvcc flags (not part of the product build).

usage: python scripts/build_variant.py NAME [-DFLAG ...]
-> paper_conf_hpca_fanzzfzdtksy25_b200/libwdntt_NAME.so (git-ignored); a GPU job swaps it in with
   cp libwdntt_NAME.so libwdntt.so before timing it."""
import concurrent.futures as cf
import os
import subprocess
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_hpca_fanzzfzdtksy25_b200 import build as B  # noqa: E402

name, extra = sys.argv[1], sys.argv[2:]
od = os.path.join(B.HERE, "build_obj", "var_" + name)
os.makedirs(od, exist_ok=True)


def comp(src):
    o = os.path.join(od, os.path.basename(src)[:-3] + ".o")
    cmd = [B.NVCC, *B.NVCC_FLAGS, *extra, "-I", B.INCLUDE, "-I", B.CSRC, "-c", "-o", o, src]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode:
        sys.exit(r.stderr)
    return o


with cf.ThreadPoolExecutor(max_workers=os.cpu_count() or 4) as ex:
    objs = list(ex.map(comp, B.sources()))
lib = os.path.join(B.HERE, "libwdntt_%s.so" % name)
subprocess.run([B.NVCC, *B.ARCH, "-shared", "-Xcompiler", "-fPIC", "-o", lib, *objs, "-lcudart"], check=True)
print(lib)
