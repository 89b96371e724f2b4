#!/usr/bin/env python
"""Attribute an ncu --set full capture to CUDA source lines: executed warp
instructions and stall samples per line of a kernel, via the SASS page of the
report (per-instruction counts) and `nvdisasm -g` of the same build's cubin
(offset -> line).  The .so must be the build that was profiled.

  python scripts/ncu_lines.py gpurun_out/prof.ncu-rep --kernel 'replay_lpt16_kernel<(int)0>' \
      --cubin-src replay_lpt16 [--top 40]
"""
import argparse
import csv
import io
import os
import re
import subprocess
import tempfile
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SO = os.path.join(ROOT, "paper_conf_cluster_kangjkkk17_b200", "libconvgpu.so")


def sass_page(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                         capture_output=True, text=True).stdout
    blocks, kern, hdr = {}, None, None
    for r in csv.reader(io.StringIO(out)):
        if len(r) >= 2 and r[0] == "Kernel Name":
            kern, hdr = r[1], None
            blocks[kern] = []
            continue
        if r and r[0] == "Address":
            hdr = r
            blocks[kern].append(hdr)
            continue
        if kern and hdr:
            blocks[kern].append(r)
    return blocks


def line_map(cubin_src, mangled_pat):
    d = tempfile.mkdtemp()
    subprocess.run(["cuobjdump", "-xelf", "all", SO], cwd=d, capture_output=True)
    cub = os.path.join(d, f"{cubin_src}.sm_100a.cubin")
    dis = subprocess.run(["nvdisasm", "-g", "-c", cub], capture_output=True, text=True).stdout
    m, cur_fun, line = {}, None, None
    for ln in dis.splitlines():
        if ln.startswith(".text.") and ln.endswith(":"):
            cur_fun = ln[len(".text."):-1]
            continue
        mm = re.search(r'File "([^"]+)", line (\d+)', ln) if ln.lstrip().startswith("//##") else None
        if mm:
            line = (os.path.basename(mm.group(1)), int(mm.group(2)))
            continue
        mo = re.match(r"\s+/\*([0-9a-f]+)\*/", ln)
        if mo and cur_fun and re.search(mangled_pat, cur_fun):
            m[int(mo.group(1), 16)] = line
    return m


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("rep")
    ap.add_argument("--kernel", required=True, help="substring of the demangled kernel name")
    ap.add_argument("--mangled", required=True, help="regex on the mangled name")
    ap.add_argument("--cubin-src", default="replay_lpt16")
    ap.add_argument("--src", default=os.path.join(ROOT, "paper_conf_cluster_kangjkkk17_b200", "csrc",
                                                   "replay_lpt16.cu"))
    ap.add_argument("--top", type=int, default=50)
    a = ap.parse_args()
    blocks = sass_page(a.rep)
    kb = [b for k, b in blocks.items() if a.kernel in k]
    assert kb, list(blocks)
    b = kb[0]
    idx = {x: i for i, x in enumerate(b[0])}
    data = b[1:]
    base = int(data[0][0], 16)
    lm = line_map(a.cubin_src, a.mangled)
    S = lambda r, k: float(r[idx[k]] or 0)  # noqa: E731
    inst, stall = defaultdict(float), defaultdict(float)
    stall_kind = defaultdict(lambda: defaultdict(float))
    kinds = [h for h in b[0] if h.startswith("stall_") and "Not Issued" not in h]
    for r in data:
        off = int(r[0], 16) - base
        ln = lm.get(off, ("?", -1))
        inst[ln] += S(r, "Instructions Executed")
        stall[ln] += S(r, "Warp Stall Sampling (All Samples)")
        for k in kinds:
            stall_kind[ln][k] += S(r, k)
    srcs = {}

    def text_of(ln):
        f, n = ln
        if f not in srcs:
            cand = [os.path.join(os.path.dirname(a.src), f)]
            srcs[f] = open(cand[0]).read().splitlines() if os.path.exists(cand[0]) else []
        s_ = srcs[f]
        return s_[n - 1].strip()[:64] if 0 < n <= len(s_) else ""
    ti, ts = sum(inst.values()), sum(stall.values())
    print(f"total warp instructions {ti:.4g}, stall samples {ts:.4g}")
    for ln in sorted(sorted(inst, key=lambda l: -inst[l])[:a.top]):
        top = sorted(stall_kind[ln].items(), key=lambda kv: -kv[1])[:2]
        tops = " ".join(f"{k[6:]}:{v / max(stall[ln], 1):.0%}" for k, v in top)
        print(f"{ln[0][:14]:>14s}:{ln[1]:<5d} {100 * inst[ln] / ti:5.1f}% inst {100 * stall[ln] / ts:5.1f}% stall  {tops:28s} {text_of(ln)}")


if __name__ == "__main__":
    main()
