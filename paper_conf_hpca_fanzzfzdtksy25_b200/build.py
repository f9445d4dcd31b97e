"""Build libwdntt.so in-tree with nvcc for sm_100a (no JIT, no torch extension).

``python -m paper_conf_hpca_fanzzfzdtksy25_b200.build`` or ``build()``.
Each csrc/*.cu translation unit compiles to its own object (in parallel, rebuilt only when the unit
or a header it includes changed: nvcc -MMD dependency files), then one link step makes the .so.
The shared object lands next to this file so gpurun snapshots carry it.
"""
from __future__ import annotations

import concurrent.futures as cf
import glob
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
INCLUDE = os.path.join(ROOT, "include")
OBJ = os.path.join(HERE, "build_obj")
LIB = os.path.join(HERE, "libwdntt.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")

ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
NVCC_FLAGS = ARCH + [
    "-O3", "-lineinfo", "-std=c++17",
    "-Xcompiler", "-fPIC,-O2",
    "--expt-relaxed-constexpr",
    "-Xptxas", "-v",
]


def sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")))


def _obj(src):
    return os.path.join(OBJ, os.path.basename(src)[:-3] + ".o")


def _deps(src):
    """The unit plus every header nvcc recorded for it (missing .d: everything in csrc/include)."""
    d = _obj(src)[:-2] + ".d"
    if not os.path.exists(d):
        return None
    txt = open(d).read().replace("\\\n", " ")
    parts = txt.split(":", 1)[1].split() if ":" in txt else []
    return [p for p in parts if p.endswith((".cu", ".cuh", ".h"))]


def _stale(src) -> bool:
    o = _obj(src)
    if not os.path.exists(o):
        return True
    deps = _deps(src)
    if deps is None:
        return True
    t = os.path.getmtime(o)
    return any(not os.path.exists(f) or os.path.getmtime(f) > t for f in deps + [src])


def stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    return any(_stale(s) or os.path.getmtime(_obj(s)) > t for s in sources())


def _compile(src):
    o = _obj(src)
    cmd = [NVCC, *NVCC_FLAGS, "-I", INCLUDE, "-I", CSRC, "-MMD", "-MF", o[:-2] + ".d", "-c", "-o", o, src]
    res = subprocess.run(cmd, capture_output=True, text=True)
    return src, cmd, res


def build(force: bool = False, verbose: bool = False) -> str:
    os.makedirs(OBJ, exist_ok=True)
    todo = [s for s in sources() if force or _stale(s)]
    log_lines = []
    if todo:
        with cf.ThreadPoolExecutor(max_workers=min(len(todo), os.cpu_count() or 4)) as ex:
            results = list(ex.map(_compile, todo))
        failed = False
        for src, cmd, res in results:
            log_lines.append(" ".join(cmd) + "\n" + res.stdout + res.stderr)
            if res.returncode != 0:
                failed = True
                sys.stderr.write(res.stdout + res.stderr)
        with open(os.path.join(HERE, "build.log"), "w") as f:
            f.write("\n".join(log_lines))
        if failed:
            raise RuntimeError("nvcc failed (see %s)" % os.path.join(HERE, "build.log"))
        if verbose:
            for _, _, res in results:
                sys.stderr.write(res.stderr)
    if todo or force or not os.path.exists(LIB) or stale():
        tmp = LIB + ".tmp%d" % os.getpid()
        cmd = [NVCC, *ARCH, "-shared", "-Xcompiler", "-fPIC", "-o", tmp, *[_obj(s) for s in sources()], "-lcudart"]
        res = subprocess.run(cmd, capture_output=True, text=True)
        if res.returncode != 0:
            sys.stderr.write(res.stdout + res.stderr)
            raise RuntimeError("link failed: " + " ".join(cmd))
        os.replace(tmp, LIB)
    return LIB


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose="-v" in sys.argv)
    print(LIB)
