#!/usr/bin/env python
"""bench.py -- TurboBC hot path on B200: GTEPS and sec/source, roofline, CPU-oracle baseline.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config 3] [--impl ours|reference]
    (N > 1: torchrun --nproc-per-node N ... bench.py --gpus N ...)

A step = one full pass of the hot path (forward + backward for every source of the rank's
source batch, then the one all-reduce of bc across ranks) -- PAPER.md Algorithm 1 over a
source list.  Workload (BASELINE.json configs[2], the one the metric's 1/2/4/8-GPU figures
are quoted on): Graph500 Kronecker scale 22, edgefactor 16, directed, CSC engine, 4096
sources per GPU (weak scaling: rank r takes sources [r*4096, (r+1)*4096) of one seeded list).
GTEPS = sources * m / t (paper convention: m = stored nnz, every source counted
against all m).  The graph (523 MB of CSC+CSR) is larger than the 126 MB L2.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "BC GTEPS and sec/source at 1/2/4/8 B200; HBM GB/s fraction of peak"
# the configs' source lists (BASELINE.json configs); strong scaling splits them over the ranks
SOURCES_TOTAL = {1: 1024, 2: 1024, 3: 4096, 4: 1024, 5: 8192, 6: None, 7: 1024, 8: 1024}
# the paper's printed figure for the SAME workload (context: Titan Xp), GTEPS
PAPER_GTEPS = {6: (10.257, "Table 5 P:452: exact BC of mycielski16, 159.8 s, 10,257 MTEPs on a Titan Xp"),
               7: (18.470, "Table 3 P:380: one source of mycielski19, 48.9 ms, 18,470 MTEPs on a Titan Xp")}
EXACT = (6,)  # configs whose step is exact BC over all n sources, split across the ranks


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", type=int, default=3)
    ap.add_argument("--sources", type=int, default=None,
                    help="sources per step (strong) or per GPU (weak); default: the config's list")
    ap.add_argument("--scaling", choices=["strong", "weak"], default="strong",
                    help="strong: the config's list split over the ranks; weak: that many per rank")
    ap.add_argument("--assign", choices=["contiguous", "interleaved"], default="contiguous",
                    help="rank r takes a contiguous range of the list, or every world-th source")
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-sample", type=int, default=None, help="sources in the CPU-oracle sample")
    ap.add_argument("--direction", type=int, default=0)
    ap.add_argument("--format", type=int, default=0, help="0 auto, 1 list passes, 2 edge streams")
    ap.add_argument("--engine", choices=["csc", "coot"], default="csc")
    ap.add_argument("--one-format", action="store_true",
                    help="directed graphs keep the CSC alone (TBC_FLAG_ONE_FORMAT; batched engine)")
    ap.add_argument("--batch", type=int, default=-1,
                    help="engine: -1 auto (level-width probe), 0 per source, 1 batched, 2 narrow-level")
    ap.add_argument("--width", type=int, default=0, help="batched engine: sources per sweep (32, 64; 0 auto)")
    ap.add_argument("--inplace", type=int, default=-1,
                    help="batched engine: 1 backward overwrites sigma with delta_u in place, 0 separate rows, -1 auto")
    ap.add_argument("--order", type=int, default=1, help="batched engine: 1 group sources by 2-hop out-volume, 0 as given")
    ap.add_argument("--cost", default="", help="cost model overrides, e.g. list=10,stream=2")
    ap.add_argument("--trace", type=int, default=-1, help="print the per-level timeline of this source to stderr")
    return ap.parse_args()


def peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            p = json.load(f)
        return float(p["hbm_gbs"]), "measured"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md)"


class ClockSampler:
    """nvidia-smi clocks/throttle reasons sampled every 200 ms during the timed region."""

    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index):
        self.idx = gpu_index
        self.rows = []
        self.proc = None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", f"--id={self.idx}", f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "200"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append([x.strip() for x in line.split(",")])

    def __exit__(self, *a):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()

    def summary(self):
        sm = [float(r[1]) for r in self.rows if len(r) >= 9 and r[1].replace(".", "").isdigit()]
        mx = [float(r[2]) for r in self.rows if len(r) >= 9 and r[2].replace(".", "").isdigit()]
        reasons = set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for r in self.rows:
            if len(r) >= 9:
                for nm, val in zip(names, r[5:9]):
                    if val.strip().lower() == "active":
                        reasons.add(nm)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(sm)}


def make_graph(cfg, device):
    import graphgen as gg
    t0 = time.time()
    g, _ = gg.make_config(cfg, device=device)
    return g, time.time() - t0


def source_list(g, cfg, total):
    import graphgen as gg
    if cfg == 1:
        return np.tile(np.arange(g.n, dtype=np.int32), (total + g.n - 1) // g.n)[:total]
    return gg.sources(g, total, seed=gg.CONFIGS[cfg]["src_seed"])


def cpu_model():
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except Exception:
        pass
    return None


def cpu_baseline(g, sources, sample):
    """The oracle as it stands on this host's cores, bounded sample of the same workload: all-core
    throughput (one source per thread) and the single-thread sec/source (the comparator of the
    paper's "(sequential)x")."""
    import oracle
    cores = os.cpu_count() or 1
    k = sample or min(max(cores, 4), 64)
    src = sources[:k]
    _, secs = oracle.bc_timed(g.col_ptr, g.row_idx, g.directed, src, nthreads=min(cores, k))
    k1 = 2 if g.nnz > 2e8 else 4
    _, secs1 = oracle.bc_timed(g.col_ptr, g.row_idx, g.directed, sources[:k1], nthreads=1)
    return {"value": k * g.nnz / secs / 1e9, "unit": "GTEPS", "cores": min(cores, k), "kind": "oracle",
            "sample": f"{k} sources of the same graph (first {k} of the rank-0 source list), "
                      f"{secs:.2f} s of C Brandes oracle, one source per thread, graph build excluded; "
                      f"single-thread: {k1} sources in {secs1:.2f} s",
            "sec_per_source": secs / k, "single_thread_sec_per_source": secs1 / k1,
            "cpu_model": cpu_model(), "host_cores": cores}


def run_reference(args):
    """--impl reference: the oracle (this tier's reference arm) on the bench workload, rank 0 only."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    import oracle
    g, _ = make_graph(args.config, "cpu" if args.config in (1,) else _gen_device())
    if args.config in EXACT:
        srcs = np.arange(g.n, dtype=np.int32)
    else:
        total = args.sources or SOURCES_TOTAL[args.config]
        srcs = source_list(g, args.config, total * (args.gpus if args.scaling == "weak" else 1))
    cores = os.cpu_count() or 1
    k = args.cpu_sample or min(max(cores, 4), 64)
    times = []
    for i in range(args.warmup + args.steps):
        sub = srcs[(i * k) % len(srcs):][:k]
        _, secs = oracle.bc_timed(g.col_ptr, g.row_idx, g.directed, sub, nthreads=min(cores, k))
        if i >= args.warmup:
            times.append(secs / len(sub))
    spp = statistics.mean(times)
    val = g.nnz / spp / 1e9
    line = {"impl": "reference", "metric": METRIC, "value": val, "unit": "GTEPS", "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": spp * k * 1e3,
            "higher_is_better": True, "scaling": args.scaling, "vs_baseline": None, "dtype": "f64",
            "data": "synthetic", "sec_per_source": spp,
            "config": {"workload": _workload_name(args.config), "n": g.n, "m": g.nnz,
                       "sources_per_step": k},
            "cpu_baseline": {"value": val, "unit": "GTEPS", "cores": min(cores, k), "kind": "oracle",
                             "sample": f"{k} sources per step of the same workload"},
            "e2e": {"value": val, "unit": "GTEPS", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def _gen_device():
    import torch
    return "cuda" if torch.cuda.is_available() else "cpu"


def _workload_name(cfg):
    import graphgen as gg
    return gg.CONFIGS[cfg]["name"]


def traffic_signature(cfg, engine, k, eng, width):
    """Key of a measured-traffic file: the exact launch (workload, engine, sources per launch, W)."""
    return f"cfg{cfg}_{engine}_k{k}_e{eng}_w{width}"


def load_traffic(sig):
    """DRAM bytes of the exact launch from tools/measure_traffic.py (an ncu capture of this launch
    configuration, committed under profiles/), or None."""
    path = os.path.join(ROOT, "profiles", f"traffic_{sig}.json")
    if not os.path.exists(path):
        return None, None
    try:
        return json.load(open(path)), os.path.relpath(path, ROOT)
    except Exception:
        return None, None


def main():
    args = parse()
    if args.impl == "reference":
        run_reference(args)
        return
    import torch
    import torch.distributed as dist
    import paper_conf_icppw_artiless21_b200 as tbc
    from paper_conf_icppw_artiless21_b200 import dist as tdist

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world != args.gpus:
        raise SystemExit(f"--gpus {args.gpus} but WORLD_SIZE={world}")
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        os.environ.setdefault("NCCL_DEBUG", "INFO")  # communicator init lines: the rank count is on record
        dist.init_process_group("nccl", device_id=dev)

    g, gen_s = make_graph(args.config, "cuda")
    # the source list and this rank's share: strong scaling splits the config's list
    # over the ranks, weak scaling gives every rank a list of that size
    if args.config in EXACT:  # exact BC: all n sources per step
        all_src = np.arange(g.n, dtype=np.int32)
    else:
        total = args.sources or SOURCES_TOTAL[args.config]
        if args.scaling == "weak":
            total *= world
        all_src = source_list(g, args.config, total)
    n_sources = len(all_src)
    if args.assign == "interleaved":
        my_src = all_src[rank::world]
    else:
        lo, hi = tdist.partition(n_sources, world, rank)
        my_src = all_src[lo:hi]
    per_gpu = len(my_src)
    t0 = time.time()
    engine = tbc.ENGINE_COOT if args.engine == "coot" else tbc.ENGINE_CSC
    G = tbc.Graph.from_csc(g.col_ptr, g.row_idx, g.directed, engine=engine, device=local,
                           one_format=args.one_format)
    create_s = time.time() - t0
    G.set_direction(args.direction)
    G.set_format(args.format)
    G.set_batch(1 if args.one_format and g.directed else args.batch)
    G.set_batch_width(args.width)
    G.set_batch_order(args.order)
    G.set_batch_inplace(args.inplace)
    if args.cost:
        G.set_cost(**{k: float(v) for k, v in (kv.split("=") for kv in args.cost.split(","))})
    src_d = torch.from_numpy(np.ascontiguousarray(my_src)).to(dev)
    bc = torch.zeros(g.n, dtype=torch.float64, device=dev)
    stream = torch.cuda.current_stream(dev)

    def step():
        bc.zero_()
        G.bc_device(src_d, bc, stream)
        if world > 1:
            dist.all_reduce(bc, op=dist.ReduceOp.SUM)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    G.reset_stats()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    kev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    with ClockSampler(local) as clk:
        for i in range(args.steps):
            ev[i][0].record(stream)
            bc.zero_()
            kev[i][0].record(stream)
            G.bc_device(src_d, bc, stream)
            kev[i][1].record(stream)
            if world > 1:
                dist.all_reduce(bc, op=dist.ReduceOp.SUM)
            ev[i][1].record(stream)
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
    step_ms = [a.elapsed_time(b) for a, b in ev]
    kern_ms = [a.elapsed_time(b) for a, b in kev]
    total_ms = sum(step_ms)
    busy_ms = sum(kern_ms)  # this rank's time in the hot path (its source slice)
    busy = [busy_ms]
    if world > 1:
        t = torch.tensor([total_ms], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        total_ms = float(t.item())
        bt = torch.zeros(world, dtype=torch.float64, device=dev)
        bt[rank] = busy_ms
        dist.all_reduce(bt, op=dist.ReduceOp.SUM)
        busy = bt.tolist()
    st = G.stats()
    eng = st["engine"] if args.engine == "csc" else 0
    batched = eng == 1
    kname = {0: "k_bc", 1: "k_bcb", 2: "k_bcs"}[eng]
    sources_total = n_sources * args.steps
    gteps = sources_total * g.nnz / (total_ms / 1e3) / 1e9
    ms_per_step = total_ms / args.steps

    # roofline of the hot-path kernel: SURVEY 8(d) algorithmic bytes B_min = 8 B per
    # out-edge of the reached set (4 B index read once per stage) + 80 B per reached vertex, summed
    # over the launch's sources, / the kernel's event-timed duration on its stream.  The batched
    # engine shares the index stream between the W sources of a sweep, so its own compulsory
    # traffic is 8 B per reached edge / W + 80 B per reached (vertex, source).
    alg_bytes_per_launch = (8.0 * st["reached_edges"] + 80.0 * st["reached"]) / args.steps
    wdt = st["batch_width"] if batched else 1
    alg_bytes_batched = (8.0 * st["reached_edges"] / wdt + 80.0 * st["reached"]) / args.steps
    k_avg_s = statistics.mean(kern_ms) / 1e3
    peak, peak_kind = peaks()
    achieved = alg_bytes_per_launch / k_avg_s / 1e9
    # measured DRAM bytes of this exact launch (ncu, profiles/traffic_<signature>.json)
    sig = traffic_signature(args.config, args.engine, per_gpu, eng, wdt)
    tj, tpath = load_traffic(sig)
    traffic = hbm = None
    stages = None
    if tj:
        traffic = tj["full"]["dram_bytes"]
        hbm = traffic / k_avg_s / 1e9 / peak
        if tj.get("forward"):
            fw, fu = tj["forward"], tj["full"]
            stages = {"forward_bytes": fw["dram_bytes"], "forward_ms": fw["ms"],
                      "backward_bytes": fu["dram_bytes"] - fw["dram_bytes"], "backward_ms": fu["ms"] - fw["ms"],
                      "forward_hbm_frac": fw["dram_bytes"] / (fw["ms"] / 1e3) / 1e9 / peak,
                      "backward_hbm_frac": (fu["dram_bytes"] - fw["dram_bytes"]) / ((fu["ms"] - fw["ms"]) / 1e3)
                      / 1e9 / peak if fu["ms"] > fw["ms"] else None}

    # end to end through the public host API: H2D sources, run, all-reduce, D2H bc
    e2e_times = []
    for i in range(max(2, min(args.steps, 3))):
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        t1 = time.perf_counter()
        out = tdist.bc(G, all_src, None) if world > 1 else G.bc(my_src)
        t2 = time.perf_counter()
        e2e_times.append(t2 - t1)
    e2e_s = statistics.median(e2e_times)
    if world > 1:
        t = torch.tensor([e2e_s], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        e2e_s = float(t.item())
    e2e_gteps = n_sources * g.nnz / e2e_s / 1e9

    if rank == 0:
        cpu = None
        if not args.no_cpu_baseline and world == 1:
            cpu = cpu_baseline(g, my_src, args.cpu_sample)
        clocks = clk.summary()
        line = {
            "metric": METRIC, "value": gteps, "unit": "GTEPS", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True,
            "scaling": "strong" if (args.config in EXACT or args.scaling == "strong") else "weak",
            "vs_baseline": gteps / PAPER_GTEPS[args.config][0] if args.config in PAPER_GTEPS else None,
            "dtype": "f64", "data": "synthetic",
            "sec_per_source": total_ms / 1e3 / sources_total,
            "config": {"workload": _workload_name(args.config), "n": g.n, "m": g.nnz,
                       "directed": g.directed, "engine": args.engine, "sources_per_step": n_sources,
                       "sources_per_gpu": per_gpu, "assign": args.assign,
                       "parallelism": f"source-partitioned x{world}, graph replicated, 1 NCCL all-reduce/step",
                       "l2": "inputs larger than L2 (CSC+CSR %.0f MB vs 126 MB L2); no flush" %
                             ((8 * (g.n + 1) + 4 * g.nnz) * (2 if g.directed else 1) / 1e6)
                             if (8 * (g.n + 1) + 4 * g.nnz) * (2 if g.directed else 1) > 126e6 else
                             "graph fits in L2 (small config); no flush",
                       "direction": args.direction, "format": args.format, "engine_kind": args.engine,
                       "one_format": bool(args.one_format and g.directed), "inplace_opt": args.inplace,
                       "engine_mode": (f"batched, {wdt} sources per sweep, {st['batch_parts']} SM partition(s)"
                                       + (", sources grouped by 2-hop out-volume" if args.order
                                          else ", sources in the given order")) if eng == 1
                       else "narrow-level: one source per CTA, CTA barriers between levels" if eng == 2
                       else "per source, SM partitions",
                       "engine_choice": "auto (level-width probe: %d vertices per level)" % st["probe_width"]
                       if args.batch == -1 else f"forced {args.batch}",
                       "paper": PAPER_GTEPS[args.config][1] if args.config in PAPER_GTEPS else None,
                       "cost": args.cost},
            "clocks": clocks,
            "gpu_launches": args.steps * (2 if eng == 2 else 1),
            "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                         "frac": achieved / peak, "traffic": traffic, "peak_kind": peak_kind,
                         "kernel": kname, "alg_bytes_per_launch": alg_bytes_per_launch,
                         "model": "SURVEY 8(d) B_min = 8 B per reached edge + 80 B per reached vertex, per "
                                  "source (B_min-equivalent throughput); a batch shares the index stream, so "
                                  "frac may exceed 1",
                         "b_min_equiv_frac": achieved / peak,
                         "hbm_frac": hbm,
                         "hbm_frac_def": "ncu dram__bytes_read+write of this exact launch / its event-timed "
                                         "duration / peak" if hbm is not None else
                                         f"no measured traffic for launch {sig} (tools/measure_traffic.py)",
                         "traffic_file": tpath, "stages": stages,
                         "achieved_batched_model": alg_bytes_batched / k_avg_s / 1e9,
                         "frac_batched_model": alg_bytes_batched / k_avg_s / 1e9 / peak,
                         "kernel_ms": statistics.mean(kern_ms)},
            "e2e": {"value": e2e_gteps, "unit": "GTEPS", "h2d_bytes_per_step": 4 * len(my_src),
                    "d2h_bytes_per_step": 8 * g.n},
            "cpu_baseline": cpu,
            "ranks": {"busy_ms_max": max(busy), "busy_ms_mean": statistics.mean(busy),
                      "imbalance": max(busy) / statistics.mean(busy) - 1.0 if statistics.mean(busy) > 0 else 0.0,
                      "busy_ms": busy},
            "traversal": {"reached_per_source": st["reached"] / max(st["sources"], 1),
                          "reached_edges_per_source": st["reached_edges"] / max(st["sources"], 1),
                          "fwd_edges_per_source": st["fwd_edges"] / max(st["sources"], 1),
                          "bwd_edges_per_source": st["bwd_edges"] / max(st["sources"], 1),
                          "levels_per_source": st["levels"] / max(st["sources"], 1),
                          "pull_levels_per_source": st["pull_levels"] / max(st["sources"], 1),
                          "list_peak": st["list_peak"], "list_overflows": st["list_overflows"],
                          "traversed_gteps": (st["reached_edges"] / args.steps) * world * args.steps
                          / (total_ms / 1e3) / 1e9},
            "setup": {"generate_s": gen_s, "create_s": create_s, "graph_bytes": G.device_bytes,
                      "device_bytes": G.info()["device_bytes"], "workspace_bytes": st["workspace_bytes"],
                      "paper_word_model_bytes": 4 * (7 * g.n + g.nnz)},
        }
        print(json.dumps(line), flush=True)
    if args.trace >= 0 and rank == 0:
        G.set_trace(args.trace)
        G.bc(my_src[: args.trace + 1])
        for r in G.trace():
            print("TRACE " + json.dumps(r), file=sys.stderr)
        G.set_trace(-1)
    G.close()
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
