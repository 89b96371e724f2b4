"""NEXT-4 on a real GPU: the wrapper module (libconvgpu_shim.so, LD_PRELOAD)
in front of the CUDA runtime / driver of a CUDA process, talking to a live
convgpud.  Checks what the process sees (§III-C/D): the context
charge at the first allocation, rejection over the limit (P:78,
P:104), pitched / managed / 3D sizes, frees by address (P:110,
P:133), cudaMemGetInfo from the ledger, and a paused allocation that
resumes when another container exits.  The latency of each
call with and without the wrapper (Fig. 4's experiment on B200) is written
to gpurun_out/ when that directory exists."""
import json
import os
import subprocess
import tempfile
import time

import pytest

from paper_conf_cluster_kangjkkk17_b200 import ctl

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
MiB = 1 << 20


@pytest.fixture(scope="module")
def probe():
    from paper_conf_cluster_kangjkkk17_b200 import build
    build.build_ctl()
    d = tempfile.mkdtemp(prefix="cgprobe")
    exe = os.path.join(d, "shim_probe")
    subprocess.check_call(["/usr/local/cuda/bin/nvcc", "-O2", "-cudart=shared",
                           "-Wno-deprecated-gpu-targets", "-o", exe,
                           os.path.join(ROOT, "tests", "shim_probe.cu"), "-lcuda"])
    return exe


def _env(sock, limit_mib, key):
    e = dict(os.environ)
    e.update(LD_PRELOAD=ctl.SHIM, CONVGPU_SOCKET=sock, CONVGPU_LIMIT_MIB=str(limit_mib),
             CONVGPU_CONTAINER=str(key))
    return e


def _lines(out):
    return [json.loads(x) for x in out.splitlines() if x.startswith("{")]


def test_api_semantics_live(probe):
    sock = os.path.join(tempfile.mkdtemp(prefix="cgd"), "s")
    with ctl.Daemon(sock, 4096 * MiB, "fifo", overhead=66 * MiB):
        r = subprocess.run([probe, "api"], env=_env(sock, 1024, 1), capture_output=True,
                           text=True, timeout=120)
        assert r.returncode == 0, r.stderr
        steps = {d["step"]: d for d in _lines(r.stdout) if "step" in d}
        pitch = [d["pitch"] for d in _lines(r.stdout) if "pitch" in d][0]
    L = 1024 * MiB
    assert steps["start"]["total"] == L and steps["start"]["free"] == L
    assert steps["malloc_100"]["rc"] == 0
    assert steps["malloc_100"]["free"] == L - 100 * MiB - 66 * MiB  # P:135 context
    assert steps["malloc_over"]["rc"] == 2  # cudaErrorMemoryAllocation
    assert steps["malloc_over"]["free"] == steps["malloc_100"]["free"]
    assert pitch == 1024  # the runtime's own pitch for 513 B rows on B200
    assert steps["pitch_513x2048"]["free"] == steps["malloc_100"]["free"] - 1024 * 2048
    assert steps["managed_1"]["free"] == steps["pitch_513x2048"]["free"] - 128 * MiB
    assert steps["malloc3d_1000x7x3"]["free"] == steps["managed_1"]["free"] - 1024 * 7 * 3
    assert steps["free_3d"]["free"] == steps["managed_1"]["free"]  # freed by address
    assert steps["free_100"]["free"] == L - 66 * MiB  # the context stays charged
    assert steps["cuMemAlloc_50"]["free"] == L - 66 * MiB - 50 * MiB  # driver API
    assert steps["cuMemFree_50"]["free"] == L - 66 * MiB


def test_pause_until_another_container_exits(probe):
    """cap 1024 MiB: A (limit 700) holds 600 MiB for 4 s; B (limit 700)
    arrives meanwhile, gets 324 MiB as fill target and asks for 300 MiB
    (+66 context): its cudaMalloc blocks until A exits, then succeeds.  (B's
    own CUDA start-up takes part of A's 4 s; the rest is B's pause.)"""
    sock = os.path.join(tempfile.mkdtemp(prefix="cgd"), "s")
    with ctl.Daemon(sock, 1024 * MiB, "fifo", overhead=66 * MiB):
        a = subprocess.Popen([probe, "hold", "600", "4.0"], env=_env(sock, 700, 1),
                             stdout=subprocess.PIPE, text=True)
        first = json.loads(a.stdout.readline())
        assert first["rc"] == 0 and first["blocked_s"] < 0.5
        t0 = time.time()
        b = subprocess.run([probe, "hold", "300", "0"], env=_env(sock, 700, 2),
                           capture_output=True, text=True, timeout=60)
        a.wait(timeout=60)
        got = _lines(b.stdout)[0]
    assert got["rc"] == 0
    assert got["blocked_s"] > 0.5, got  # paused while A ran
    assert time.time() - t0 < 30


def test_api_latency_with_and_without_wrapper(probe):
    n = 200

    def plain():
        return _lines(subprocess.run([probe, "latency", str(n)], capture_output=True, text=True,
                                     timeout=300).stdout)[0]
    base = plain()
    sock = os.path.join(tempfile.mkdtemp(prefix="cgd"), "s")
    with ctl.Daemon(sock, 180 * 1024 * MiB, "fifo", overhead=66 * MiB):
        wrapped = _lines(subprocess.run([probe, "latency", str(n)], env=_env(sock, 8192, 1),
                                        capture_output=True, text=True, timeout=300).stdout)[0]
    base2 = plain()
    doc = {"what": "median microseconds per CUDA API call (after 20 warm-up rounds), "
                   "shim_probe latency mode, one B200; baseline measured before and after",
           "n": n, "without_wrapper": base, "without_wrapper_after": base2, "with_wrapper": wrapped,
           "paper_fig4": "K20m: allocation APIs 0.035 ms -> 0.082 ms with ConVGPU (P:197)"}
    out = os.path.join(ROOT, "gpurun_out")
    if os.path.isdir(out):
        with open(os.path.join(out, "r01_shim_latency.json"), "w") as f:
            json.dump(doc, f, indent=1)
    # the wrapper adds a socket round trip per allocation; cudaMemGetInfo is
    # answered without the device
    assert wrapped["cudaMalloc_us"] > 0 and base["cudaMalloc_us"] > 0
