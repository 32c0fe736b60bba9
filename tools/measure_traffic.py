#!/usr/bin/env python
"""Measure the DRAM traffic of bench.py's exact launch with ncu (GPU box) -- tools, no method arithmetic.

    python tools/measure_traffic.py --config 3 [--sources K]

Runs ncu (--metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,
--clock-control none) on this script's --target mode, which builds the bench workload exactly as
bench.py does at N = 1 (same graph, same source list, default engine options), makes one warm-up
call, then one full call (forward + backward) and one forward-only call (TBC_OPT_STAGE = 1).  The
hot kernel's DRAM bytes per launch are written to profiles/traffic_<signature>.json, which
bench.py reports as roofline.traffic / hbm_frac (and the forward / backward split).
"""
import argparse
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def target(args):
    import numpy as np
    import torch
    import bench
    import paper_conf_icppw_artiless21_b200 as tbc
    g, _ = bench.make_graph(args.config, "cuda")
    total = args.sources or bench.SOURCES_TOTAL[args.config]
    src = bench.source_list(g, args.config, total) if args.config not in bench.EXACT else np.arange(g.n, dtype=np.int32)
    G = tbc.Graph.from_csc(g.col_ptr, g.row_idx, g.directed, engine=tbc.ENGINE_COOT if args.engine == "coot" else 0)
    s = torch.from_numpy(np.ascontiguousarray(src)).cuda()
    bc = torch.zeros(g.n, dtype=torch.float64, device="cuda")
    G.bc_device(s, bc)  # warm-up (probe, workspace)
    torch.cuda.synchronize()
    G.bc_device(s, bc)  # full launch
    G.set_stage(1)
    G.bc_device(s, bc)  # forward-only launch
    torch.cuda.synchronize()
    st = G.stats()
    eng = st["engine"] if args.engine == "csc" else 0
    meta = {"config": args.config, "engine": args.engine, "k": len(src), "eng": eng,
            "width": st["batch_width"] if eng == 1 else 1,
            "kernel": {0: "k_bc", 1: "k_bcb", 2: "k_bcs"}[eng]}
    json.dump(meta, open(args.meta, "w"))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", type=int, default=3)
    ap.add_argument("--sources", type=int, default=None)
    ap.add_argument("--engine", default="csc")
    ap.add_argument("--target", action="store_true")
    ap.add_argument("--meta", default="/tmp/traffic_meta.json")
    args = ap.parse_args()
    if args.target:
        target(args)
        return
    cmd = ["ncu", "--metrics", "dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum",
           "--clock-control", "none", "--kernel-name-base", "function", "-k", "regex:^k_bc[bs]?$", "--csv",
           sys.executable, os.path.abspath(__file__), "--target", "--config", str(args.config),
           "--engine", args.engine, "--meta", args.meta]
    if args.sources:
        cmd += ["--sources", str(args.sources)]
    out = subprocess.run(cmd, capture_output=True, text=True)
    rows = [r for r in csv.reader(io.StringIO(out.stdout)) if len(r) > 10]
    if not rows:
        sys.exit("ncu produced no rows:\n" + out.stdout[-2000:] + out.stderr[-2000:])
    hdr = rows[0]
    ii, ik, im, iv, iu = (hdr.index(c) for c in ("ID", "Kernel Name", "Metric Name", "Metric Value", "Metric Unit"))
    launches = {}
    for r in rows[1:]:
        d = launches.setdefault(int(r[ii]), {"kernel": r[ik]})
        val = float(r[iv].replace(",", ""))
        scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12,
                 "B": 1, "KB": 1e3, "MB": 1e6, "GB": 1e9, "TB": 1e12,
                 "nsecond": 1e-6, "usecond": 1e-3, "msecond": 1.0, "second": 1e3,
                 "ns": 1e-6, "us": 1e-3, "ms": 1.0, "s": 1e3}.get(r[iu])
        if scale is None:
            sys.exit(f"unknown ncu unit {r[iu]!r} for {r[im]}")
        d[r[im]] = val * scale
    meta = json.load(open(args.meta))
    import re
    pat = re.compile(r"(^|::|\s)" + meta["kernel"] + r"(<|\(|$)")
    hot = [launches[i] for i in sorted(launches) if pat.search(launches[i]["kernel"])]
    if len(hot) < 2:
        sys.exit("hot kernel launches not found: " + json.dumps(sorted({d["kernel"] for d in launches.values()})))
    full, fwd = hot[-2], hot[-1]

    def rec(d):
        return {"dram_bytes": d["dram__bytes_read.sum"] + d["dram__bytes_write.sum"],
                "dram_read": d["dram__bytes_read.sum"], "dram_write": d["dram__bytes_write.sum"],
                "ms": d["gpu__time_duration.sum"]}
    sig = f"cfg{meta['config']}_{meta['engine']}_k{meta['k']}_e{meta['eng']}_w{meta['width']}"
    res = {"signature": sig, **meta, "full": rec(full), "forward": rec(fwd),
           "how": "ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum "
                  "--clock-control none on bench.py's N=1 launch (tools/measure_traffic.py); ncu times are "
                  "serialised cold-cache replays (context only): bench.py divides the bytes by its own "
                  "event-timed kernel duration"}
    path = os.path.join(ROOT, "profiles", f"traffic_{sig}.json")
    json.dump(res, open(path, "w"), indent=1)
    print(json.dumps(res))


if __name__ == "__main__":
    main()
