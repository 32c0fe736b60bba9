import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import graphgen as gg, oracle
import paper_conf_icppw_artiless21_b200 as tbc
g = gg.path(7, directed=True)
src = np.arange(7, dtype=np.int32)
print("oracle", oracle.bc(g.col_ptr, g.row_idx, True, src))
for of in (False, True):
    G = tbc.Graph.from_csc(g.col_ptr, g.row_idx, True, one_format=of)
    G.set_batch(1); G.set_batch_width(32)
    print("one_format", of, G.bc(src), G.stats())
    d, s = G.bfs_batch(src[:2]); print(d, s)
