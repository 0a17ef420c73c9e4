"""Build libfi.so in-tree with nvcc for sm_100a (no GPU needed).

    python -m paper_conf_dsn_0002hsvk21_b200.build [--force]
"""
from __future__ import annotations

import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
ROOT = os.path.dirname(HERE)
LIB = os.path.join(HERE, "libfi.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
FLAGS = ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC,-O2", "--expt-relaxed-constexpr",
         "-Xptxas", "-v,-warn-spills"] + ARCH
SOURCES = ["abi.cpp", "golden.cu", "golden_run.cpp", "scan.cu", "profile.cu", "select.cu", "inject.cu", "propagate.cu", "propagate8.cu",
           "campaign.cpp", "jit.cpp"]
HEADERS = ["common.cuh", "sem.cuh", "emu.cuh", "scan.cuh", "jit_prelude.cuh", "jit_k8.h"]


def _stale(obj: str, deps: list[str]) -> bool:
    return not os.path.exists(obj) or any(os.path.getmtime(d) > os.path.getmtime(obj) for d in deps)


def build(force: bool = False, verbose: bool = False) -> str:
    objdir = os.path.join(HERE, "_obj")
    os.makedirs(objdir, exist_ok=True)
    hdrs = [os.path.join(CSRC, h) for h in HEADERS] + [os.path.join(ROOT, "include", "fi.h")]
    # the JIT prelude is embedded into libfi.so as a string (NVRTC compiles it per program)
    # the JIT prelude is sem.cuh (the §3.2 semantics, shared with emu.cuh) + jit_prelude.cuh
    inc = os.path.join(objdir, "jit_prelude.inc")
    pre = [os.path.join(CSRC, "sem.cuh"), os.path.join(CSRC, "jit_prelude.cuh")]
    if force or _stale(inc, pre):
        with open(inc, "w") as g:
            g.write('R"FIJITPRELUDE(' + "".join(open(x).read() for x in pre) + ')FIJITPRELUDE"\n')
    objs = []
    for src in SOURCES:
        s = os.path.join(CSRC, src)
        o = os.path.join(objdir, src + ".o")
        objs.append(o)
        if force or _stale(o, [s] + hdrs):
            cmd = [NVCC, *FLAGS, "-I", objdir, "-c", s, "-o", o]
            r = subprocess.run(cmd, capture_output=True, text=True)
            if r.returncode:
                sys.stderr.write(r.stdout + r.stderr)
                raise RuntimeError(f"nvcc failed on {src}")
            if verbose:
                sys.stderr.write(r.stderr)
    if force or _stale(LIB, objs):
        cmd = [NVCC, *ARCH, "-shared", "-o", LIB, *objs, "-cudart", "static"]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode:
            sys.stderr.write(r.stdout + r.stderr)
            raise RuntimeError("nvcc link failed")
    return LIB


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv))
