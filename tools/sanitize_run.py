"""compute-sanitizer target: every engine and mode on small graphs, checked against the oracle.

    compute-sanitizer --tool memcheck|racecheck|synccheck python tools/sanitize_run.py
(tools/gpu_sanitize.sh; the library variant -DTBC_WATCHDOG_S=600 keeps the grid-barrier watchdog
from firing under the sanitizer's slowdown)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import numpy as np  # noqa: E402

import graphgen as gg  # noqa: E402
import oracle  # noqa: E402
import paper_conf_icppw_artiless21_b200 as tbc  # noqa: E402
from tbc_testutil import assert_bc, assert_bfs_rows  # noqa: E402

cases = [gg.make_config(1)[0], gg.kronecker(11, 16, seed=3, directed=True), gg.kronecker(11, 16, seed=3, directed=False),
         gg.road_lattice(64, 0.1, seed=2), gg.star(300)]
runs = 0
for g in cases:
    src = gg.sources(g, 70, seed=1)
    want = oracle.bc(g.col_ptr, g.row_idx, g.directed, src)
    modes = [("batched64", dict(batch=1, width=64)), ("batched32_parts3", dict(batch=1, width=32, parts=3)),
             ("narrow", dict(batch=2)), ("narrow_xr", dict(batch=2, sigma=1)), ("per_source", dict(batch=0)),
             ("list1", dict(batch=1, width=64, blist=1))]
    for name, kw in modes:
        with tbc.Graph.from_csc(g.col_ptr, g.row_idx, g.directed) as G:
            G.set_batch(kw["batch"])
            if "width" in kw:
                G.set_batch_width(kw["width"])
            if "parts" in kw:
                G.set_batch_parts(kw["parts"])
            if "sigma" in kw:
                G.set_sigma_mode(kw["sigma"])
            if "blist" in kw:
                G.set_batch_list(kw["blist"])
            assert_bc(G.bc(src), want)
            if kw["batch"] != 0:
                d, s = G.bfs_batch(src[:3])
                assert_bfs_rows(g, src[:3], d, s)
            runs += 1
    if g.directed:
        with tbc.Graph.from_csc(g.col_ptr, g.row_idx, True, one_format=True) as G:
            assert_bc(G.bc(src), want)
            runs += 1
    with tbc.Graph.from_csc(g.col_ptr, g.row_idx, g.directed, engine=tbc.ENGINE_COOT) as G:
        assert_bc(G.bc(src[:8]), oracle.bc(g.col_ptr, g.row_idx, g.directed, src[:8]))
        runs += 1
print(f"SANITIZE_OK {runs} runs")
