#!/usr/bin/env python
"""A/B check of a kernel variant against the current build on config [2]:
every per-container output and summary field of 2^16 traces, per policy,
compared with the build at $CONVGPU_SO_REF (fields listed in --ignore may
differ, e.g. while a variant's peak_used is still being built)."""
import argparse
import os
import subprocess
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def run(so, count, out_npz):
    code = f"""
import numpy as np, torch, workloads as W, paper_conf_cluster_kangjkkk17_b200 as cg
w = W.CONFIGS['c2']; tr = cg.generate(w.gen, 0, {count}); res = {{}}
for pol in W.POLICIES:
    out = cg.alloc_out({count}, w.gen.n)
    cg.replay(tr, w.cap, pol, out, rand_seed=w.rand_seed, ovh=w.ovh, kernel='lane16')
    torch.cuda.synchronize()
    s = out.summary_np(); f = out.full_np()
    for k in s.dtype.names: res[pol + ':' + k] = s[k]
    for k in f: res[pol + ':' + k] = f[k]
    st = cg.stats_dict(out.stats_np())
    res[pol + ':events'] = np.array([st['events']])
np.savez('{out_npz}', **res)
"""
    env = dict(os.environ, CONVGPU_SO=so)
    subprocess.run([sys.executable, "-c", code], env=env, check=True, cwd=ROOT)
    return np.load(out_npz)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--ref", default="ab/base.so")
    ap.add_argument("--var", default="ab/skip.so")
    ap.add_argument("--count", type=int, default=65536)
    ap.add_argument("--ignore", default="")
    a = ap.parse_args()
    r = run(a.ref, a.count, "/tmp/ref.npz")
    v = run(a.var, a.count, "/tmp/var.npz")
    ign = set(a.ignore.split(",")) if a.ignore else set()
    bad = 0
    for k in r.files:
        if k.split(":")[1] in ign:
            continue
        if not np.array_equal(r[k], v[k]):
            d = np.nonzero(r[k].ravel() != v[k].ravel())[0]
            print("DIFF", k, len(d), "first", d[:5], r[k].ravel()[d[:3]], v[k].ravel()[d[:3]])
            bad += 1
    print("fields differing:", bad)


if __name__ == "__main__":
    main()
