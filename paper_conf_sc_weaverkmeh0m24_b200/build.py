"""Build libsched.so in-tree for sm_100a (nvcc cross-compiles; no GPU needed).

Each translation unit is compiled to an object in parallel, then linked:
  python -m paper_conf_sc_weaverkmeh0m24_b200.build [--force]
"""
from __future__ import annotations

import glob
import os
import subprocess
import sys
from concurrent.futures import ThreadPoolExecutor

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
# SCHED_BUILD_TAG=X (A/B measurements): objects in build_obj_X/, library ab/lib_X.so
# (load it with SCHED_SO_PATH=ab/lib_X.so); the product build leaves it unset
_TAG = os.environ.get("SCHED_BUILD_TAG", "")
OBJ = os.path.join(HERE, "build_obj" + ("_" + _TAG if _TAG else ""))
SO = os.path.join(ROOT, "ab", f"lib_{_TAG}.so") if _TAG else os.path.join(HERE, "libsched.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")

ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
CFLAGS = [*ARCH, "-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC,-ffp-contract=off,-fno-fast-math",
          "-Xptxas", "-v", "-Xcompiler", "-iquote," + os.path.join(ROOT, "include"), "-I", CSRC,
          # include/sched.h only as "sched.h" (-iquote): <sched.h> of the system headers (pthread) stays glibc's
          *os.environ.get("SCHED_NVCC_EXTRA", "").split()]


def sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")) + glob.glob(os.path.join(CSRC, "*.cpp")))


def headers():
    return sorted(glob.glob(os.path.join(CSRC, "*.hpp")) + glob.glob(os.path.join(CSRC, "*.cuh")) +
                  [os.path.join(ROOT, "include", "sched.h")])


def _obj(src):
    return os.path.join(OBJ, os.path.basename(src) + ".o")


def _newest_header():
    return max(os.path.getmtime(h) for h in headers())


def _compile(src):
    o = _obj(src)
    cmd = [NVCC, *CFLAGS, "-c", "-o", o, src]
    r = subprocess.run(cmd, capture_output=True, text=True)
    return src, r.returncode, " ".join(cmd) + "\n" + r.stdout + r.stderr


def build(force: bool = False, verbose: bool = False) -> str:
    os.makedirs(OBJ, exist_ok=True)
    os.makedirs(os.path.dirname(SO), exist_ok=True)
    hdr = _newest_header()
    todo = [s for s in sources()
            if force or not os.path.exists(_obj(s))
            or os.path.getmtime(_obj(s)) < max(os.path.getmtime(s), hdr)]
    logs = []
    if todo:
        with ThreadPoolExecutor(max_workers=min(len(todo), os.cpu_count() or 4)) as ex:
            for src, rc, log in ex.map(_compile, todo):
                logs.append(log)
                if rc != 0:
                    sys.stderr.write(log)
                    raise RuntimeError("nvcc failed on " + os.path.basename(src))
    objs = [_obj(s) for s in sources()]
    if todo or not os.path.exists(SO) or os.path.getmtime(SO) < max(os.path.getmtime(o) for o in objs):
        tmp = SO + f".tmp{os.getpid()}"
        cmd = [NVCC, *ARCH, "-shared", "-cudart", "static", "-o", tmp, *objs]
        r = subprocess.run(cmd, capture_output=True, text=True)
        logs.append(" ".join(cmd) + "\n" + r.stdout + r.stderr)
        if r.returncode != 0:
            sys.stderr.write(r.stdout + r.stderr)
            raise RuntimeError("nvcc link failed")
        os.replace(tmp, SO)
    if logs:
        with open(os.path.join(HERE, "build.log"), "w") as f:
            f.write("\n".join(logs))
    if verbose:
        sys.stderr.write("\n".join(logs))
    return SO


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv))
