#!/usr/bin/env python
"""Write the full-source-list oracle fixtures tests/golden/oracle_cfg<N>.npz -- TEST INFRASTRUCTURE.

    python tools/make_oracle_cache.py --config 3 [--threads 8] [--sources K] [--chunk 256]

Calls only graphgen (seeded inputs) and oracle/ (the CPU Brandes oracle): no value here ever
comes from the CUDA path.  The graph is generated on the HOST; graphgen's Kronecker generator is
counter-based, so the GPU tests regenerate the same graph on the device and check it against the
fingerprint stored here before comparing.

The fixture holds, for bc = oracle.bc(graph, the config's source list[:K]) (Eq. 3; halved
per source if undirected):
  * the graph fingerprint (n, nnz, sha256 of col_ptr / row_idx) and the source-list sha256
  * sha256 of the packed exact-zero mask of bc (zeros are exact on both sides, R17),
    the number of zeros, and fsum(bc)
  * bc at a seeded uniform sample of vertices plus at the 1024 largest entries -- or the whole
    vector when it is small (n <= 2^20)
Long runs checkpoint the partial sum per chunk of sources under .oracle_work/ (git/gpurun
ignored), so an interrupted run resumes.
"""
from __future__ import annotations

import argparse
import hashlib
import json
import math
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import graphgen as gg  # noqa: E402
import oracle  # noqa: E402

WORK = os.path.join(ROOT, ".oracle_work")
FULL_MAX_N = 1 << 20
SAMPLE = 1 << 16
TOP = 1024


def sha(a: np.ndarray) -> str:
    return hashlib.sha256(np.ascontiguousarray(a).tobytes()).hexdigest()


def fingerprint(g) -> dict:
    return {"n": int(g.n), "nnz": int(g.nnz), "directed": bool(g.directed),
            "col_ptr_sha": sha(g.col_ptr.astype(np.int64)), "row_idx_sha": sha(g.row_idx.astype(np.int32))}


def summary_of(bc: np.ndarray, seed: int) -> dict:
    """Everything a test compares, computed from a full bc vector (used by the tests too)."""
    zero = bc == 0.0
    return {"zero_sha": sha(np.packbits(zero)), "nzero": int(zero.sum()), "fsum": math.fsum(bc.tolist())}


def sample_index(n: int, seed: int) -> np.ndarray:
    rng = np.random.default_rng(seed)
    return np.sort(rng.choice(n, size=min(SAMPLE, n), replace=False)).astype(np.int64)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", type=int, required=True)
    ap.add_argument("--threads", type=int, default=os.cpu_count() or 1)
    ap.add_argument("--sources", type=int, default=None, help="first K of the config's list (default all)")
    ap.add_argument("--chunk", type=int, default=256)
    args = ap.parse_args()
    t0 = time.time()
    g, src = gg.make_config(args.config, device="cpu")
    if args.sources:
        src = src[: args.sources]
    src = np.ascontiguousarray(src, dtype=np.int32)
    fp = fingerprint(g)
    print(f"cfg{args.config}: n={g.n} nnz={g.nnz} k={src.size} generated in {time.time() - t0:.0f} s", flush=True)
    os.makedirs(WORK, exist_ok=True)
    tag = f"cfg{args.config}_{fp['row_idx_sha'][:12]}_{sha(src)[:12]}"
    ck = os.path.join(WORK, tag + ".npz")
    bc = np.zeros(g.n, dtype=np.float64)
    done = 0
    if os.path.exists(ck):
        z = np.load(ck)
        bc, done = z["bc"].copy(), int(z["done"])
        print(f"resuming at {done}/{src.size}", flush=True)
    while done < src.size:
        t1 = time.time()
        part = src[done:done + args.chunk]
        bc += oracle.bc(g.col_ptr, g.row_idx, g.directed, part, nthreads=args.threads)
        done += part.size
        np.savez(ck + ".tmp.npz", bc=bc, done=done)
        os.replace(ck + ".tmp.npz", ck)
        print(f"  {done}/{src.size} sources, chunk {time.time() - t1:.1f} s", flush=True)
    out = {"config": args.config, "k": int(src.size), "src_sha": sha(src), **fp, **summary_of(bc, args.config)}
    arrays = {}
    if g.n <= FULL_MAX_N:
        arrays["full"] = bc
    else:
        idx = sample_index(g.n, 1000 + args.config)
        top = np.argsort(-bc, kind="stable")[:TOP].astype(np.int64)
        arrays.update(sample_idx=idx, sample_val=bc[idx], top_idx=top, top_val=bc[top])
    name = f"oracle_cfg{args.config}" + (f"_k{src.size}" if args.sources else "")
    path = os.path.join(ROOT, "tests", "golden", name + ".npz")
    np.savez_compressed(path, meta=np.array(json.dumps(out)), **arrays)
    print(f"wrote {path} ({os.path.getsize(path) / 1e6:.2f} MB) in {time.time() - t0:.0f} s: "
          + json.dumps({k: out[k] for k in ("n", "nnz", "k", "nzero", "fsum")}), flush=True)


if __name__ == "__main__":
    main()
