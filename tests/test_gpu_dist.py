"""Row a7 (multi-GPU gather) on a real GPU: bench.py's N > 1 flow with two
ranks sharing cuda:0 (gloo; NCCL needs one GPU per rank and gpurun grants
one).  Each rank replays its own shard of global trace ids on the compact
kernel, the per-policy statistics are all-reduced every step, and after the
timed steps the per-range rows (digest, events, waits, selections,
makespans, traces) are all-reduced with dist.reduce_range_digests and rank 0
checks every rank's row against the oracle's golden ranges
(tests/golden/c3_range_digests.json).  The config [3] flow (10^8-id space
sharded [r*N/G, (r+1)*N/G), chunked generate -> replay, range digests
all-reduced) runs the same way on a 4-range prefix."""
import json
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
BENCH = os.path.join(ROOT, "bench.py")


def _torchrun(args, port):
    env = dict(os.environ, CONVGPU_DIST_BACKEND="gloo", OMP_NUM_THREADS="1")
    r = subprocess.run([sys.executable, "-m", "torch.distributed.run", "--nnodes=1",
                        "--nproc-per-node", "2", "--master-addr", "127.0.0.1", "--master-port",
                        str(port), BENCH, "--gpus", "2"] + args,
                       capture_output=True, text=True, timeout=900, cwd=ROOT, env=env)
    lines = [json.loads(l) for l in r.stdout.splitlines() if l.startswith("{")]
    return r, lines


def test_two_rank_bench_gather_checked_against_oracle():
    r, lines = _torchrun(["--steps", "5", "--warmup", "3", "--traces", "65536", "--no-e2e",
                          "--no-cpu-baseline"], 29531)
    assert r.returncode == 0, r.stderr[-3000:]
    assert len(lines) == 1
    d = lines[0]
    assert d["n_gpus"] == 2 and d["config"]["traces_per_gpu"] == 65536
    par = d["parity"]
    assert par["equal"] is True and par["ranges"] == 8, par
    assert par["tail_traces_per_rank"] == (1 << 20) - 65536
    for p, v in d["per_policy"].items():
        assert v["kernel"] == "lane16"


def test_two_rank_config3_prefix_checked_against_oracle():
    r, lines = _torchrun(["--workload", "c3", "--traces", str(4 << 20), "--c3-chunk", str(1 << 20),
                          "--steps", "1", "--warmup", "1"], 29532)
    assert r.returncode == 0, r.stderr[-3000:]
    assert len(lines) == 1
    d = lines[0]
    par = d["parity"]
    assert par["equal"] is True and par["ranges"] == 16, par
    assert d["config"]["traces_total"] == 4 << 20 and d["config"]["traces_per_gpu"] == 2 << 20


def test_rho_sweep_two_ranks_equals_one(tmp_path):
    """Config [4] sharded over ranks: the statistics all-reduced over two
    ranks (each replaying half of every point's trace ids) equal one rank
    replaying all of them, run by run (digest sums, events, flags)."""
    one, two = tmp_path / "one.json", tmp_path / "two.json"
    common = ["--traces", "20000", "--seeds", "2", "--lit-seeds", "1", "--rhos", "2,8"]
    r = subprocess.run([sys.executable, os.path.join(ROOT, "scripts", "rho_sweep.py")] + common +
                       ["--out", str(one)], capture_output=True, text=True, timeout=900, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-3000:]
    env = dict(os.environ, CONVGPU_DIST_BACKEND="gloo", OMP_NUM_THREADS="1")
    r = subprocess.run([sys.executable, "-m", "torch.distributed.run", "--nnodes=1",
                        "--nproc-per-node", "2", "--master-addr", "127.0.0.1", "--master-port",
                        "29533", os.path.join(ROOT, "scripts", "rho_sweep.py")] + common +
                       ["--out", str(two)], capture_output=True, text=True, timeout=900, cwd=ROOT,
                       env=env)
    assert r.returncode == 0, r.stderr[-3000:]
    a, b = json.loads(one.read_text()), json.loads(two.read_text())
    assert b["n_gpus"] == 2
    for part in ("runs",):
        for x, y in zip(a[part], b[part]):
            assert (x["rho"], x["policy"], x["seed"]) == (y["rho"], y["policy"], y["seed"])
            assert x["digest_sum"] == y["digest_sum"] and x["events"] == y["events"]
            assert x["flag_count"] == y["flag_count"]
    for x, y in zip(a["literal"]["runs"], b["literal"]["runs"]):
        assert x["digest_sum"] == y["digest_sum"] and x["deadlock_share"] == y["deadlock_share"]
