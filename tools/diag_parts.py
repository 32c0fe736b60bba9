"""Debug helper (GPU): bc parity vs the oracle over SM partitions x engine modes x repeats.

    TBC_VARIANT="-DTBC_BLOCK=512 -DTBC_LANE_ITEMS=8" python tools/diag_parts.py [--directed 1]
Prints one line per (parts, mode) with the number of wrong entries in each repeat.
"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

import graphgen as gg  # noqa: E402
import oracle  # noqa: E402
import paper_conf_icppw_artiless21_b200 as tbc  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--directed", type=int, default=1)
ap.add_argument("--scale", type=int, default=13)
ap.add_argument("--k", type=int, default=37)
ap.add_argument("--reps", type=int, default=3)
ap.add_argument("--parts", default="1,2,3,4,8")
ap.add_argument("--modes", default="0,0,0;0,0,1;0,0,2;1,1,1;2,1,1;2,2,0")
a = ap.parse_args()

g = gg.kronecker(a.scale, 16, seed=4, directed=bool(a.directed), device="cuda")
src = gg.sources(g, a.k, seed=3)
want = oracle.bc(g.col_ptr, g.row_idx, bool(a.directed), src)
zero = want == 0


def nbad(got):
    bad = (zero & (got != 0)) | (~zero & (np.abs(got - want) > 1e-9 * np.abs(np.where(zero, 1, want))))
    return int(bad.sum())


print("variant", os.environ.get("TBC_VARIANT", ""), flush=True)
with tbc.Graph.from_csc(g.col_ptr, g.row_idx, g.directed) as G:
    for parts in [int(x) for x in a.parts.split(",")]:
        for mode in a.modes.split(";"):
            dm, fm, bm = (int(x) for x in mode.split(","))
            G.set_partitions(parts)
            G.set_direction(dm)
            G.set_format(fm)
            G.set_bwd_direction(bm)
            res = [nbad(G.bc(src)) for _ in range(a.reps)]
            # one source at a time: isolates per-source vs cross-source state leaks
            single = 0
            if any(res):
                acc = np.zeros(g.n)
                for s in src:
                    acc += G.bc(np.array([s], dtype=np.int32))
                single = nbad(acc)
            print(f"parts={parts} mode={mode} bad={res} one-by-one bad={single}", flush=True)
