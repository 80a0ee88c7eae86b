"""Write tests/golden/c5_rmat26_trees.txt: the ORACLE's results for single
trees of the C5 graph (RMAT scale 26, edge factor 16; BASELINE configs[4]).

Test infrastructure: calls only graphgen (the seeded input generator; C5 is
generated with torch on a CUDA device, graphgen.rmat_gpu) and oracle/ -- never
the CUDA library.  Run on a GPU box (generation) with ~60 GB of host memory
for the oracle's copy of the 1.05 B-edge graph:

    python tools/make_c5_golden.py [t ...]      (default trees 0 7)

Per tree t (seed 1): sum of cycle lengths, cycles, depth, the 64-bit
signature of the switched edge set, and sha256 of the one-tree counters
edge_flip_counts (uint32 LE, m) and vertex_agree (uint32 LE, n).  The first
line pins the graph itself (n, m, sha256 of col and sign), so a different
generator stream fails loudly instead of comparing different graphs.
"""
import hashlib
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import graphgen  # noqa: E402
import oracle  # noqa: E402


def sha(a):
    return hashlib.sha256(np.ascontiguousarray(a).tobytes()).hexdigest()


def main():
    trees = [int(x) for x in sys.argv[1:]] or [0, 7]
    t0 = time.time()
    g, _, _ = graphgen.config("c5")
    print(f"generated n={g.n} m={g.m} in {time.time() - t0:.0f} s", flush=True)
    lines = ["# C5 oracle golden (tools/make_c5_golden.py): graph n m sha256(col) sha256(sign)",
             f"graph {g.n} {g.m} {sha(g.col.astype('<i4'))} {sha(g.sign.astype('i1'))}",
             "# tree t (seed 1): sum_cycle_len cycles depth signature sha256(cnt u32) sha256(agree u32)"]
    t1 = time.time()
    og = oracle.Graph.from_csr(g)
    print(f"oracle graph built in {time.time() - t1:.0f} s (ncomp {og.ncomp})", flush=True)
    for t in trees:
        t2 = time.time()
        cnt, agree, st = og.balance(t + 1, 1, t_begin=t, stride=1, with_stats=True)
        sk, nc, dep, sig = (int(x) for x in st[0])
        lines.append(f"tree {t} {sk} {nc} {dep} {sig:016x} {sha(cnt.astype('<u4'))} {sha(agree.astype('<u4'))}")
        print(lines[-1], f"({time.time() - t2:.0f} s)", flush=True)
    out = os.path.join(ROOT, "tests", "golden", "c5_rmat26_trees.txt")
    if os.environ.get("GOLDEN_OUT"):
        out = os.environ["GOLDEN_OUT"]
    with open(out, "w") as f:
        f.write("\n".join(lines) + "\n")
    print("wrote", out)


if __name__ == "__main__":
    main()
