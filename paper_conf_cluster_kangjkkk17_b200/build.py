"""Build libconvgpu.so in-tree with nvcc for sm_100a (no JIT cache: the .so
travels with the repo snapshot to the GPU box)."""
from __future__ import annotations

import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
SO = os.path.join(PKG, "libconvgpu.so")
SOURCES = ["replay.cu", "replay_lpt.cu", "replay_lpt16.cu", "generate.cu", "wrap.cu", "pack16.cu",
           "abi.cu"]
HEADERS = ["common.cuh", "internal.h", "lpt_util.cuh", "oem64.cuh"]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
FLAGS = ["-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo", "-std=c++17",
         "-Xcompiler", "-fPIC", "-Xcompiler", "-Wall", "-Xptxas", "-v",
         "-I" + os.path.join(ROOT, "include"), "-I" + CSRC]


def _stale() -> bool:
    if not os.path.exists(SO):
        return True
    t = os.path.getmtime(SO)
    deps = [os.path.join(CSRC, f) for f in SOURCES + HEADERS]
    deps.append(os.path.join(ROOT, "include", "convgpu.h"))
    deps.append(os.path.abspath(__file__))
    return any(os.path.getmtime(d) > t for d in deps)


def build(force: bool = False, verbose: bool = False) -> str:
    """Compile every translation unit to an object in parallel (the units are
    independent: no relocatable device code), then link the shared library."""
    if not force and not _stale():
        return SO
    from concurrent.futures import ThreadPoolExecutor
    objdir = os.path.join(PKG, "build")
    os.makedirs(objdir, exist_ok=True)

    def compile_one(f):
        obj = os.path.join(objdir, f.replace(".cu", ".o"))
        # CONVGPU_NVCC_DEFS: extra -D flags for A/B builds of kernel variants
        extra = os.environ.get("CONVGPU_NVCC_DEFS", "").split()
        cmd = [NVCC, *FLAGS, *extra, "-c", "-o", obj, os.path.join(CSRC, f)]
        r = subprocess.run(cmd, capture_output=True, text=True)
        return obj, cmd, r

    with ThreadPoolExecutor(len(SOURCES)) as ex:
        results = list(ex.map(compile_one, SOURCES))
    tmp = SO + ".tmp"
    link = [NVCC, "-gencode", "arch=compute_100a,code=sm_100a", "-shared", "-o", tmp] + \
        [o for o, _, _ in results]
    log = os.path.join(PKG, "build.log")
    failed = [r for _, _, r in results if r.returncode != 0]
    with open(log, "w") as f:
        for _, cmd, r in results:
            f.write(" ".join(cmd) + "\n" + r.stdout + r.stderr)
    if failed:
        sys.stderr.write("".join(r.stdout + r.stderr for r in failed))
        raise RuntimeError(f"nvcc failed; see {log}")
    r = subprocess.run(link, capture_output=True, text=True)
    with open(log, "a") as f:
        f.write(" ".join(link) + "\n" + r.stdout + r.stderr)
    if r.returncode != 0:
        sys.stderr.write(r.stdout + r.stderr)
        raise RuntimeError(f"nvcc link failed ({r.returncode}); see {log}")
    os.replace(tmp, SO)
    if verbose:
        sys.stderr.write("".join(r.stderr for _, _, r in results))
    return SO


# ---- NEXT-4: the live control plane (native, host side) --------------------
CTL = os.path.join(CSRC, "ctl")
DAEMON = os.path.join(PKG, "convgpud")
SHIM = os.path.join(PKG, "libconvgpu_shim.so")
CXX = os.environ.get("CXX", "g++")
CTL_HDR = [os.path.join(ROOT, "include", "convgpu_ctl.h"), os.path.join(CTL, "sched.hpp")]


def _run(cmd, what):
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        sys.stderr.write(r.stdout + r.stderr)
        raise RuntimeError(f"{what} failed ({r.returncode})")


def _older(out, srcs):
    return not os.path.exists(out) or any(os.path.getmtime(s) > os.path.getmtime(out) for s in srcs)


def build_ctl(force: bool = False) -> tuple:
    """convgpud (scheduler daemon) and libconvgpu_shim.so (LD_PRELOAD wrapper
    module, linked against nothing CUDA: it resolves the real CUDA entry points
    with dlsym(RTLD_NEXT) at run time)."""
    dsrc = [os.path.join(CTL, "convgpud.cpp"), os.path.join(CTL, "sched.cpp")]
    if force or _older(DAEMON, dsrc + CTL_HDR):
        _run([CXX, "-O2", "-std=c++17", "-Wall", "-Wextra", "-I" + os.path.join(ROOT, "include"),
              "-o", DAEMON + ".tmp"] + dsrc,
             "convgpud build")
        os.replace(DAEMON + ".tmp", DAEMON)
    ssrc = [os.path.join(CTL, "shim.cpp")]
    if os.path.exists(ssrc[0]) and (force or _older(SHIM, ssrc + CTL_HDR)):
        # no C++ runtime, hidden by default: only the CUDA entry points are exported
        _run([CXX, "-O2", "-std=c++17", "-Wall", "-Wextra", "-fPIC", "-shared",
              "-fno-exceptions", "-fno-rtti", "-fno-threadsafe-statics", "-nostdlib++",
              "-fvisibility=hidden",
              "-I/usr/local/cuda/include", "-I" + os.path.join(ROOT, "include"),
              "-o", SHIM + ".tmp"] + ssrc + ["-ldl", "-lpthread"],
             "shim build")
        os.replace(SHIM + ".tmp", SHIM)
    return DAEMON, SHIM


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose=True))
    print(build_ctl(force="--force" in sys.argv))
