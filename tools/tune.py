"""Tuning helper (GPU): time option settings of the engine on a config and dump per-level traces.

    python tools/tune.py --config 3 --sources 256 --settings "fmt=0;fmt=1;fmt=2" --trace 0,1
Each setting is a comma list of key=value: fmt, dir, list, stream, atomic, vertex (cost model, ps).
Prints one JSON line per setting (ms/source, GTEPS) and TRACE lines for the traced sources.
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import graphgen as gg  # noqa: E402
import paper_conf_icppw_artiless21_b200 as tbc  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", type=int, default=3)
ap.add_argument("--sources", type=int, default=256)
ap.add_argument("--settings", default="fmt=0")
ap.add_argument("--trace", default="")
ap.add_argument("--reps", type=int, default=2)
a = ap.parse_args()

ap2 = None
g, _ = gg.make_config(a.config, device="cuda")
src = gg.sources(g, a.sources, seed=gg.CONFIGS[a.config]["src_seed"] or 0)
if os.environ.get("TUNE_SORT") == "deg":      # group sources of similar out-degree into batches
    src = src[np.argsort(-g.out_degree()[src], kind="stable")]
elif os.environ.get("TUNE_SORT") == "indeg":
    src = src[np.argsort(-g.in_degree()[src], kind="stable")]
elif os.environ.get("TUNE_SORT", "").startswith("hop2"):
    od = g.out_degree().astype(np.float64)
    col = np.repeat(np.arange(g.n), np.diff(g.col_ptr))        # edge row_idx[e] -> col[e]
    hop2 = np.bincount(g.row_idx, weights=od[col], minlength=g.n)  # sum of out-degrees of out-neighbours
    if os.environ["TUNE_SORT"] == "hop2":
        src = src[np.argsort(-hop2[src], kind="stable")]
    elif os.environ["TUNE_SORT"] == "hop3":
        hop3 = np.bincount(g.row_idx, weights=hop2[col], minlength=g.n)
        src = src[np.argsort(-hop3[src], kind="stable")]
    elif os.environ["TUNE_SORT"].startswith("hop2log"):  # classes of log2 volume, degree within
        gran = float(os.environ["TUNE_SORT"][7:] or 4)
        cls = np.floor(np.log2(hop2[src] + 1) * gran)
        src = src[np.lexsort((-od[src], -cls))]
    elif os.environ["TUNE_SORT"].startswith("degloghop"):  # classes of log2 degree, volume within
        gran = float(os.environ["TUNE_SORT"][9:] or 4)
        cls = np.floor(np.log2(od[src] + 1) * gran)
        src = src[np.lexsort((-hop2[src], -cls))]
    else:  # hop2deg: out-degree, ties by 2-hop volume
        src = src[np.lexsort((-hop2[src], -od[src]))]
G = tbc.Graph.from_csc(g.col_ptr, g.row_idx, g.directed, one_format=os.environ.get("TUNE_ONE_FORMAT") == "1")
s_d = torch.from_numpy(src).cuda()
bc = torch.zeros(g.n, dtype=torch.float64, device="cuda")
st = torch.cuda.current_stream()
for setting in a.settings.split(";"):
    kv = dict(x.split("=") for x in setting.split(",") if x)
    G.set_format(int(kv.get("fmt", 0)))
    G.set_direction(int(kv.get("dir", 0)))
    G.set_bwd_direction(int(kv.get("bwd", 0)))
    G.set_partitions(int(kv.get("parts", 8)))
    G.set_batch(int(kv.get("batch", 1)))
    if "slots" in kv:
        G.set_narrow_slots(int(kv["slots"]))
    G.set_batch_width(int(kv.get("width", 0)))
    G.set_batch_pull(float(kv.get("bpull", 8)))
    G.set_batch_parts(int(kv.get("bparts", 0)))
    G.set_batch_order(int(kv.get("order", 1)))
    G.set_cost(**{k: float(v) for k, v in kv.items() if k in ("list", "stream", "atomic", "vertex", "scan", "bpush")})
    G.bc_device(s_d, bc, st)  # warm-up
    torch.cuda.synchronize()
    G.reset_stats()
    prof = "TBC_PROF" in os.environ.get("TBC_VARIANT", "")
    if prof:
        G.profile()  # reset
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(st)
    for _ in range(a.reps):
        G.bc_device(s_d, bc, st)
    e1.record(st)
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / a.reps
    s = G.stats()
    print(json.dumps({"setting": setting, "ms_per_source": ms / a.sources,
                      "gteps": a.sources * g.nnz / (ms / 1e3) / 1e9,
                      "fwd_edges_per_src": s["fwd_edges"] / max(s["sources"], 1),
                      "bwd_edges_per_src": s["bwd_edges"] / max(s["sources"], 1),
                      "pull_levels": s["pull_levels"] / max(s["sources"], 1),
                      "levels": s["levels"], "reached_per_src": s["reached"] / max(s["sources"], 1)}), flush=True)
    if prof:
        pr = G.profile()
        tot = sum(pr.values()) or 1
        if int(kv.get("batch", 1)):
            names = ["barrier", "bphase", "r2", "r3", "r4", "retire", "other", "r7",
                     "tile_window", "tile_index", "tile_append", "tile_owners", "owner_gather", "owner_epilogue"]
            vals = list(pr.values())
            pr = {**{n: v for n, v in zip(names, vals) if not n.startswith("r")},
                  **{k: v for k, v in pr.items() if k.startswith("b_")},
                  "b_owners_push": vals[16], "b_owners_pull": vals[17], "b_owners_bwd": vals[18]}
        reg = {k: v for k, v in pr.items() if not k.startswith("b_")}
        tot = sum(reg.values()) or 1
        print("PROFILE " + setting + " " + " ".join(f"{k}={100 * v / tot:.1f}" for k, v in reg.items() if v), flush=True)
        print("COUNTS " + setting + " " + " ".join(f"{k}={v}" for k, v in pr.items() if k.startswith("b_")), flush=True)
    for t in [int(x) for x in a.trace.split(",") if x]:
        G.set_trace(t)
        G.bc(src[: 32 * (t // 32 + 1)])
        for r in G.trace():
            print("TRACE " + json.dumps({"setting": setting, "src": t, **r}), flush=True)
        G.set_trace(-1)
    G.set_cost(list=12, stream=4, atomic=18, vertex=10, scan=3, bpush=6)
G.close()
