"""ncu target: one warm-up k_bcb (or k_bc) launch, then one profiled launch over --sources sources of a config."""
import argparse, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import graphgen as gg
import paper_conf_icppw_artiless21_b200 as tbc
ap = argparse.ArgumentParser()
ap.add_argument("--config", type=int, default=3)
ap.add_argument("--sources", type=int, default=16)
ap.add_argument("--settings", default="")
a = ap.parse_args()
g, _ = gg.make_config(a.config, device="cuda")
src = gg.sources(g, a.sources, seed=gg.CONFIGS[a.config]["src_seed"] or 0)
G = tbc.Graph.from_csc(g.col_ptr, g.row_idx, g.directed)
kv = dict(x.split("=") for x in a.settings.split(",") if x)
G.set_format(int(kv.get("fmt", 0)))
G.set_direction(int(kv.get("dir", 0)))
G.set_bwd_direction(int(kv.get("bwd", 0)))
if "batch" in kv:
    G.set_batch(int(kv["batch"]))
s = torch.from_numpy(src).cuda()
bc = torch.zeros(g.n, dtype=torch.float64, device="cuda")
for _ in range(2):
    G.bc_device(s, bc)
torch.cuda.synchronize()
print("done", flush=True)
