#!/usr/bin/env python
"""Write csrc/oem64.cuh: Batcher's odd-even merge sort network for 64 keys
(Knuth TAOCP vol. 3, 5.3.4, Algorithm M), one CE(a, b) per comparator, and
check it sorts (random inputs)."""
import os
import random

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def network(n=64):
    ces, p = [], 1
    while p < n:
        k = p
        while k >= 1:
            j = k % p
            while j <= n - 1 - k:
                for x in range(k):
                    if x + j + k < n and (x + j) // (2 * p) == (x + j + k) // (2 * p):
                        ces.append((x + j, x + j + k))
                j += 2 * k
            k >>= 1
        p <<= 1
    return ces


def main():
    ces = network()
    rng = random.Random(1)
    for _ in range(20000):
        v = [rng.randrange(8) for _ in range(64)]
        w = list(v)
        for a, b in ces:
            if w[a] > w[b]:
                w[a], w[b] = w[b], w[a]
        assert w == sorted(v)
    lines = ["// oem64.cuh — Batcher's odd-even merge sort network for 64 keys as a list",
             "// of compare-exchanges (%d; the bitonic network needs 672), written out so" % len(ces),
             "// that every index is a literal and the keys stay in registers.  Generated",
             "// by scripts/gen_oem64.py; CE(a, b) must leave the minimum at a.",
             "#pragma once",
             "#define OEM64_NETWORK(CE) \\"]
    for i in range(0, len(ces), 8):
        lines.append("  " + " ".join("CE(%d,%d)" % c for c in ces[i:i + 8]) + " \\")
    lines.append("  /* end */")
    with open(os.path.join(ROOT, "paper_conf_cluster_kangjkkk17_b200", "csrc", "oem64.cuh"), "w") as f:
        f.write("\n".join(lines) + "\n")


if __name__ == "__main__":
    main()
