"""In-tree build of the native libraries (sm_100a only; no JIT, no torch extension cache).

  libsh.so      the offload engine (hot path): csrc/{engine,layout,autotune,cpu_adam}.cpp + kernels.cu
  libsh_gpt.so  GPT block compute used by the bench and parity tests (outside the hot path):
                csrc/gpt/*.cu + cuBLASLt

Objects are rebuilt when a source or header is newer.  Run: python -m paper_conf_sc_sunwqyhxw22_b200._build
"""
from __future__ import annotations

import glob
import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
OUT = os.path.join(PKG, "lib")
BUILD = os.path.join(ROOT, "build")
CUDA = os.environ.get("CUDA_HOME", "/usr/local/cuda")
NVCC = os.path.join(CUDA, "bin", "nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def _nccl_include() -> str:
    import importlib.util
    spec = importlib.util.find_spec("nvidia")
    for base in (spec.submodule_search_locations or []) if spec else []:
        inc = os.path.join(base, "nccl", "include")
        if os.path.exists(os.path.join(inc, "nccl.h")):
            return inc
    return "/usr/include"


INCS = ["-I" + os.path.join(ROOT, "include"), "-I" + CSRC, "-I" + os.path.join(CUDA, "include")]
CXXFLAGS = ["-O3", "-fPIC", "-std=c++17", "-ffp-contract=off", "-fno-fast-math", "-g1", "-Wall",
            "-Wno-unused-function", "-Werror=return-type", "-pthread"]
NVFLAGS = ARCH + ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC,-ffp-contract=off,-Werror=return-type",
                  "--fmad=false", "-Xptxas", "-v"]


def _newer(out: str, deps: list[str]) -> bool:
    if not os.path.exists(out):
        return True
    t = os.path.getmtime(out)
    return any(os.path.getmtime(d) > t for d in deps)


def _run(cmd: list[str], log: list[str]):
    r = subprocess.run(cmd, capture_output=True, text=True)
    log.append(" ".join(cmd) + "\n" + r.stdout + r.stderr)
    if r.returncode != 0:
        sys.stderr.write(r.stdout + r.stderr)
        raise RuntimeError("build failed: " + " ".join(cmd[:3]) + " ... " + cmd[-1])


def _compile(src: str, headers: list[str], extra: list[str], log: list[str]) -> str:
    rel = os.path.relpath(src, CSRC).replace(os.sep, "_")
    obj = os.path.join(BUILD, rel + ".o")
    if _newer(obj, [src] + headers):
        if src.endswith(".cu"):
            _run([NVCC] + NVFLAGS + INCS + extra + ["-c", src, "-o", obj], log)
        else:
            _run(["g++"] + CXXFLAGS + INCS + extra + ["-c", src, "-o", obj], log)
    return obj


def build(verbose: bool = False) -> dict:
    os.makedirs(OUT, exist_ok=True)
    os.makedirs(BUILD, exist_ok=True)
    log: list[str] = []
    headers = glob.glob(os.path.join(ROOT, "include", "*.h")) + glob.glob(os.path.join(CSRC, "*.hpp"))
    nccl = ["-I" + _nccl_include()]
    srcs = [os.path.join(CSRC, f) for f in ("engine.cpp", "layout.cpp", "autotune.cpp", "cpu_adam.cpp", "numa.cpp",
                                            "spill_io.cpp", "kernels.cu")]
    objs = [_compile(s, headers, nccl, log) for s in srcs]
    lib = os.path.join(OUT, "libsh.so")
    if _newer(lib, objs):
        _run([NVCC] + ARCH + ["-shared", "-o", lib] + objs + ["-lpthread", "-ldl"], log)
    out = {"libsh": lib}
    gpt_srcs = sorted(glob.glob(os.path.join(CSRC, "gpt", "*.cu")))
    if gpt_srcs:
        gh = headers + glob.glob(os.path.join(CSRC, "gpt", "*.cuh"))
        gobjs = [_compile(s, gh, [], log) for s in gpt_srcs]
        glib = os.path.join(OUT, "libsh_gpt.so")
        if _newer(glib, gobjs):
            _run([NVCC] + ARCH + ["-shared", "-o", glib] + gobjs +
                 ["-L" + os.path.join(CUDA, "lib64"), "-lcublasLt", "-lcublas", "-lpthread"], log)
        out["libsh_gpt"] = glib
    with open(os.path.join(BUILD, "build.log"), "w") as f:
        f.write("\n".join(log))
    if verbose:
        print("\n".join(log))
    return out


if __name__ == "__main__":
    print(build(verbose="-v" in sys.argv))
