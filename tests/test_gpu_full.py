"""Full-size parity of the engine the bench times, per-source depth/sigma of the batched engine,
and the multi-GPU entry points with the real kernel.  Needs a B200.

* Full source lists (configs 2-4, and the cached config-5 slice): the GPU runs tbc_bc over the
  config's WHOLE list in the bench's launch configuration (default options: auto width, auto
  partitions, sources grouped into batches); the result is compared with a fixture written by
  tools/make_oracle_cache.py, which calls only graphgen and oracle/ on a HOST-generated graph.
  The device regenerates the graph and must match the fixture's fingerprint first (graphgen's
  counter-based generator).  Compared: bc at 2^16 seeded vertices + the 1024 largest (or every
  vertex for n <= 2^20) to 1e-9 relative, the exact-zero mask (sha256), the zero count and fsum(bc).
  PAPER.md P:332 (Sec. 4): only results verified against the sequential code are accepted.
* tbc_bfs_batch: depth bit-exact, sigma bit-exact below 2^53 (relative 1e-12 above) for every
  source of a sweep of the batched engine k_bcb (sigma is an output, Alg.1 l.2; depth S is
  set at l.24).
* dist.bc / dist.bc_device (north star (d)): world-1 NCCL group, and gloo world 2 with both ranks
  on cuda:0, against the oracle.
"""
import hashlib
import json
import math
import os
import socket

import numpy as np
import pytest

import graphgen as gg
import oracle
import paper_conf_icppw_artiless21_b200 as tbc
from tbc_testutil import ROOT, assert_bc, assert_bfs_rows

pytestmark = pytest.mark.gpu


def _sha(a):
    return hashlib.sha256(np.ascontiguousarray(a).tobytes()).hexdigest()


def _fixture(name):
    path = os.path.join(ROOT, "tests", "golden", name + ".npz")
    if not os.path.exists(path):
        pytest.skip(f"{name}.npz not generated (tools/make_oracle_cache.py)")
    z = np.load(path)
    return json.loads(str(z["meta"])), z


# ------------------------------------------------------------------ generator determinism

@pytest.mark.parametrize("directed", [False, True])
def test_kronecker_generator_identical_on_host_and_device(directed):
    a = gg.kronecker(14, 16, seed=7, directed=directed, device="cpu")
    b = gg.kronecker(14, 16, seed=7, directed=directed, device="cuda")
    np.testing.assert_array_equal(a.col_ptr, b.col_ptr)
    np.testing.assert_array_equal(a.row_idx, b.row_idx)


# ------------------------------------------------------------------ full source lists vs cached oracle

def _check_full_list(cfg, name=None, k=None, setup=None):
    meta, z = _fixture(name or f"oracle_cfg{cfg}")
    g, src = gg.make_config(cfg, device="cpu" if gg.CONFIGS[cfg]["kind"] != "kron" else "cuda")
    src = src[: meta["k"]]
    assert (g.n, g.nnz) == (meta["n"], meta["nnz"])
    assert _sha(g.col_ptr.astype(np.int64)) == meta["col_ptr_sha"]
    assert _sha(g.row_idx.astype(np.int32)) == meta["row_idx_sha"]
    assert _sha(np.ascontiguousarray(src, dtype=np.int32)) == meta["src_sha"]
    with tbc.Graph.from_csc(g.col_ptr, g.row_idx, g.directed) as G:  # bench launch configuration
        if setup:
            setup(G)
        got = G.bc(src)
        st = G.stats()
    assert st["sources"] == meta["k"] and st["bad_sources"] == 0
    zero = got == 0.0
    assert _sha(np.packbits(zero)) == meta["zero_sha"], (int(zero.sum()), meta["nzero"])
    assert abs(math.fsum(got.tolist()) - meta["fsum"]) <= 1e-9 * abs(meta["fsum"])
    if "full" in z.files:
        assert_bc(got, z["full"])
    else:
        assert_bc(got[z["sample_idx"]], z["sample_val"])
        assert_bc(got[z["top_idx"]], z["top_val"])
    return st


def test_cfg2_full_source_list_cached_oracle():
    _check_full_list(2)


def test_cfg3_full_source_list_cached_oracle():
    """The bench workload exactly: Kronecker 22 directed, all 4096 sources, 64 grouped sources per sweep."""
    st = _check_full_list(3)
    assert st["batch_width"] == 64


def test_cfg4_full_source_list_cached_oracle():
    _check_full_list(4)


def test_cfg5_rank0_slice_cached_oracle():
    """Config 5 (Kronecker 25, 1.05e9 entries): the first 1024 sources of its list -- the slice rank 0
    runs when 8 GPUs share 8192 sources -- against the cached oracle."""
    _check_full_list(5, name="oracle_cfg5_k1024")


# ------------------------------------------------------------------ per-source depth / sigma of k_bcb

SMALL = [gg.star(7), gg.path(7, directed=True), gg.cycle(9), gg.complete_bipartite(3, 5), gg.grid(6, 7),
         gg.random_tree(50, 1), gg.mycielski(6), gg.from_edges("iso", 4, [(1, 2), (2, 3)], False)]


@pytest.mark.parametrize("direction", [tbc.DIR_AUTO, tbc.DIR_PUSH, tbc.DIR_PULL])
@pytest.mark.parametrize("width", [32, 64, "narrow"])
@pytest.mark.parametrize("g", SMALL, ids=lambda g: g.name)
def test_bfs_batch_small_all_sources(g, width, direction):
    src = np.arange(g.n, dtype=np.int32)
    src = np.concatenate([src, src[:3]]).astype(np.int32)  # repeats inside a sweep
    with tbc.Graph.from_csc(g.col_ptr, g.row_idx, g.directed) as G:
        if width == "narrow":
            G.set_batch(tbc.ENGINE_NARROW)
        else:
            G.set_batch(tbc.ENGINE_BATCHED)
            G.set_batch_width(width)
        G.set_direction(direction)
        depth, sigma = G.bfs_batch(src)
    assert_bfs_rows(g, src, depth, sigma)


@pytest.mark.parametrize("width", [0, 32, 64, "narrow"])
@pytest.mark.parametrize("scale,directed", [(14, False), (15, True)])
def test_bfs_batch_kronecker(scale, directed, width):
    g = gg.kronecker(scale, 16, seed=2, directed=directed, device="cuda")
    src = gg.sources(g, 70, seed=12)  # a full sweep of 64 and a ragged one (or 3 of 32)
    with tbc.Graph.from_csc(g.col_ptr, g.row_idx, g.directed) as G:
        if width == "narrow":
            G.set_batch(tbc.ENGINE_NARROW)
        else:
            G.set_batch(tbc.ENGINE_BATCHED)
            G.set_batch_width(width)
            G.set_batch_parts(2)
        depth, sigma = G.bfs_batch(src)
        st = G.stats()
        assert st["engine"] == (2 if width == "narrow" else 1)
        if width != "narrow":
            assert st["batch_parts"] == 2
    assert_bfs_rows(g, src, depth, sigma)


def test_bfs_batch_grid_sigma_crosses_2_53():
    g = gg.grid(40, 40)
    src = np.array([0, 820, 39, 1599], dtype=np.int32)
    with tbc.Graph.from_csc(g.col_ptr, g.row_idx, g.directed) as G:
        for direction in (tbc.DIR_AUTO, tbc.DIR_PUSH, tbc.DIR_PULL):
            G.set_direction(direction)
            depth, sigma = G.bfs_batch(src)
            assert sigma[0].max() > 2.0 ** 53
            assert_bfs_rows(g, src, depth, sigma)


@pytest.mark.parametrize("cfg", [2, 3])
def test_bfs_batch_full_size_kronecker_sweep(cfg):
    """One full sweep (64 sources, the auto width) of configs 2 and 3 at full size: every row of
    config 2, and 16 rows spread over the sweep's two source words for config 3 (the oracle BFS of a
    4 M-vertex graph per row is the cost)."""
    g, src = gg.make_config(cfg, device="cuda")
    src = src[:64]
    with tbc.Graph.from_csc(g.col_ptr, g.row_idx, g.directed) as G:
        depth, sigma = G.bfs_batch(src)
        assert G.stats()["batch_width"] == 64
    rows = np.arange(64) if cfg == 2 else np.arange(0, 64, 4)
    assert_bfs_rows(g, src[rows], depth[rows], sigma[rows])


@pytest.mark.parametrize("engine", [tbc.ENGINE_AUTO, tbc.ENGINE_BATCHED])
def test_bfs_batch_full_size_road_lattice(engine):
    g, src = gg.make_config(4)
    src = src[:6]
    with tbc.Graph.from_csc(g.col_ptr, g.row_idx, g.directed) as G:
        G.set_batch(engine)
        depth, sigma = G.bfs_batch(src)
        assert G.stats()["engine"] == (2 if engine == tbc.ENGINE_AUTO else 1)
    assert depth.max() > 1000
    assert_bfs_rows(g, src, depth, sigma)


def test_auto_engine_choice():
    """The level-width probe sends deep narrow graphs (lattice, ER 1024) to the narrow-level engine
    and scale-free graphs to the batched engine."""
    cases = [(gg.road_lattice(512, 0.10, seed=4), 2), (gg.make_config(1)[0], 2),
             (gg.kronecker(16, 16, seed=2, directed=False, device="cuda"), 1)]
    for g, want in cases:
        src = gg.sources(g, 40, seed=5)
        with tbc.Graph.from_csc(g.col_ptr, g.row_idx, g.directed) as G:
            assert_bc(G.bc(src), oracle.bc(g.col_ptr, g.row_idx, g.directed, src))
            st = G.stats()
            assert st["engine"] == want, (g.name, st["probe_width"])


@pytest.mark.parametrize("directed", [False, True])
def test_narrow_engine_kronecker_and_hubs(directed):
    """The narrow-level engine on a scale-free graph (hubs: the warp-per-vertex queue of both stages,
    queue overflow to single threads) and with out-of-range device sources."""
    import torch
    g = gg.kronecker(15, 16, seed=9, directed=directed, device="cuda")
    src = gg.sources(g, 300, seed=4)
    want = oracle.bc(g.col_ptr, g.row_idx, directed, src)
    with tbc.Graph.from_csc(g.col_ptr, g.row_idx, g.directed) as G:
        G.set_batch(tbc.ENGINE_NARROW)
        assert_bc(G.bc(src), want)
        bad = np.concatenate([src[:7], [-3, g.n], src[7:]]).astype(np.int32)
        acc = torch.zeros(g.n, dtype=torch.float64, device="cuda")
        G.reset_stats()
        G.bc_device(torch.from_numpy(bad).cuda(), acc)
        torch.cuda.synchronize()
        assert_bc(acc.cpu().numpy(), want)
        st = G.stats()
        assert st["bad_sources"] == 2 and st["sources"] == len(src)


# ------------------------------------------------------------------ multi-GPU entry points, real kernel

def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _dist_graph():
    g = gg.kronecker(12, 16, seed=21, directed=True)
    return g, gg.sources(g, 101, seed=3)


def _dist_worker(rank, world, backend, port, out_dir):
    import torch
    import torch.distributed as dist
    from paper_conf_icppw_artiless21_b200 import dist as tdist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    torch.cuda.set_device(0)
    dist.init_process_group(backend, rank=rank, world_size=world)
    g, src = _dist_graph()
    with tbc.Graph.from_csc(g.col_ptr, g.row_idx, g.directed, device=0) as G:
        host = tdist.bc(G, src)                                          # host API
        dev = tdist.bc_device(G, torch.from_numpy(src).cuda())          # device API
        torch.cuda.synchronize()
        st = G.stats()
    np.save(os.path.join(out_dir, f"host_{rank}.npy"), host)
    np.save(os.path.join(out_dir, f"dev_{rank}.npy"), dev.cpu().numpy())
    np.save(os.path.join(out_dir, f"srcs_{rank}.npy"), np.array([st["sources"]]))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("backend,world", [("nccl", 1), ("gloo", 2)])
def test_dist_bc_real_kernel(tmp_path, backend, world):
    import torch.multiprocessing as mp
    mp.spawn(_dist_worker, args=(world, backend, _free_port(), str(tmp_path)), nprocs=world, join=True)
    g, src = _dist_graph()
    want = oracle.bc(g.col_ptr, g.row_idx, True, src)
    per_rank = []
    for r in range(world):
        assert_bc(np.load(tmp_path / f"host_{r}.npy"), want)
        assert_bc(np.load(tmp_path / f"dev_{r}.npy"), want)
        per_rank.append(int(np.load(tmp_path / f"srcs_{r}.npy")[0]))
    # each rank ran only its contiguous slice, twice (host and device API)
    from paper_conf_icppw_artiless21_b200 import dist as tdist
    assert per_rank == [2 * (hi - lo) for lo, hi in (tdist.partition(len(src), world, r) for r in range(world))]


@pytest.mark.parametrize("width", [32, 64])
def test_batched_list_overflow_reruns_halves(width):
    """Level lists sized below a sweep's need (TBC_OPT_BATCH_LIST = 1 on a deep lattice, where the W
    sources of a sweep sit on different levels): k_bcb re-runs overflowing sweeps as halves, bc stays
    exact, the overflow is reported, and the next call grows the lists."""
    g = gg.road_lattice(128, 0.10, seed=4)
    src = gg.sources(g, 70, seed=2)
    want = oracle.bc(g.col_ptr, g.row_idx, False, src)
    with tbc.Graph.from_csc(g.col_ptr, g.row_idx, g.directed) as G:
        G.set_batch(tbc.ENGINE_BATCHED)
        G.set_batch_width(width)
        G.set_batch_parts(1)
        G.set_batch_list(1)
        assert_bc(G.bc(src), want)
        st = G.stats()
        assert st["list_overflows"] > 0 and st["sources"] == len(src)
        depth, sigma = G.bfs_batch(src[:9])
        assert_bfs_rows(g, src[:9], depth, sigma)
        for _ in range(8):  # the lists grow call by call until a sweep fits
            G.reset_stats()
            assert_bc(G.bc(src), want)
        assert G.stats()["list_overflows"] == 0


# ------------------------------------------------------------------ in-place backward (TBC_OPT_BATCH_INPLACE)

INPLACE_CASES = [gg.star(9), gg.path(9, directed=True), gg.cycle(11), gg.complete(7), gg.grid(9, 8),
                 gg.mycielski(7), gg.random_tree(300, 3)]


@pytest.mark.parametrize("width", [32, 64])
@pytest.mark.parametrize("g", INPLACE_CASES, ids=lambda g: g.name)
def test_inplace_backward_small(g, width):
    """sigma rows overwritten by delta_u, split owners through the split accumulator: the oracle's bc
    on closed-form graphs, over two calls (the first may re-run sweeps whose accumulator is short,
    the second runs with the accumulator sized from the first)."""
    src = np.concatenate([np.arange(g.n), np.arange(min(g.n, 40))]).astype(np.int32)  # repeats (R18)
    want = oracle.bc(g.col_ptr, g.row_idx, g.directed, src)
    with tbc.Graph.from_csc(g.col_ptr, g.row_idx, g.directed) as G:
        G.set_batch(tbc.ENGINE_BATCHED)
        G.set_batch_width(width)
        G.set_batch_inplace(1)
        for _ in range(2):
            assert_bc(G.bc(src), want)


@pytest.mark.parametrize("directed", [False, True])
@pytest.mark.parametrize("parts", [1, 3])
def test_inplace_backward_kronecker(directed, parts):
    """Kronecker 14 (hubs: owners spanning hundreds of tiles, most tiles holding a split owner), W = 64,
    1 or 3 SM partitions; and the workspace is smaller than with separate delta_u rows."""
    g = gg.kronecker(14, 16, seed=21, directed=directed, device="cuda")
    src = gg.sources(g, 200, seed=5)
    want = oracle.bc(g.col_ptr, g.row_idx, directed, src)
    ws = {}
    for mode in (1, 0):
        with tbc.Graph.from_csc(g.col_ptr, g.row_idx, g.directed) as G:
            G.set_batch(tbc.ENGINE_BATCHED)
            G.set_batch_width(64)
            G.set_batch_parts(parts)
            G.set_batch_inplace(mode)
            for _ in range(2):
                G.reset_stats()
                assert_bc(G.bc(src), want)
            ws[mode] = G.stats()["workspace_bytes"]
    assert ws[1] < ws[0]


def test_inplace_cfg3_full_source_list_cached_oracle():
    """The bench workload (Kronecker 22 directed, all 4096 sources) with the in-place backward."""
    _check_full_list(3, setup=lambda G: G.set_batch_inplace(1))


# ------------------------------------------------------------------ strict single format (NEXT-4)

def _one_format_cases():
    rng = np.random.default_rng(8)
    out = [gg.path(7, directed=True), gg.star(9, directed_both=True),
           gg.from_edges("dstar_d", 3000, [(0, 1)] + [(0, i) for i in range(2, 1500)] + [(1, i) for i in range(1500, 3000)]
                         + [(i, 1) for i in range(2, 1500)], True)]
    for t in range(6):
        n = int(rng.integers(5, 80))
        A = rng.random((n, n)) < float(rng.choice([0.03, 0.1, 0.3]))
        np.fill_diagonal(A, False)
        u, v = np.nonzero(A)
        out.append(gg.from_edges(f"rd{t}", n, np.stack([u, v], 1), True))
    out.append(gg.kronecker(14, 16, seed=6, directed=True, device="cuda"))
    return out


@pytest.mark.parametrize("width", [32, 64])
def test_one_format_directed_parity(width):
    """TBC_FLAG_ONE_FORMAT: CSC only; pull-only forward, backward push over in-edges (fp64 atomics)."""
    for g in _one_format_cases():
        src = gg.sources(g, min(3 * g.n, 150), seed=1) if g.n > 5 else np.arange(g.n, dtype=np.int32)
        want = oracle.bc(g.col_ptr, g.row_idx, True, src)
        with tbc.Graph.from_csc(g.col_ptr, g.row_idx, True, one_format=True) as G:
            G.set_batch_width(width)
            assert_bc(G.bc(src), want)
            depth, sigma = G.bfs_batch(src[:5])
            assert_bfs_rows(g, src[:5], depth, sigma)
            d1, s1 = G.bfs(int(src[0]))  # tbc_bfs routes to the batched forward stage
            np.testing.assert_array_equal(d1, depth[0])
            with pytest.raises(tbc.TBCError):
                G.set_batch(0)


def test_one_format_footprint_and_cfg3_full_list():
    """Config 3 in strict single-format mode: graph bytes against the paper's 7n+m word model
    (7n + m words with 4-byte words; here 24 n + 4 m bytes) and the two-format graph, and
    the full 4096-source list against the cached oracle."""
    meta, z = _fixture("oracle_cfg3")
    g, src = gg.make_config(3, device="cuda")
    n, m = g.n, g.nnz
    with tbc.Graph.from_csc(g.col_ptr, g.row_idx, True) as G2:
        two = G2.info()["device_bytes"]
    with tbc.Graph.from_csc(g.col_ptr, g.row_idx, True, one_format=True) as G:
        one = G.info()["device_bytes"]
        # col_ptr 8 B + degrees 8 B + label maps 8 B per vertex, row_idx 4 B per entry, counters/trace
        assert one <= 24 * n + 4 * m + (16 << 20), (one, 24 * n + 4 * m)
        assert one < 0.5 * two, (one, two)
        got = G.bc(src)
        assert G.stats()["sources"] == len(src)
    zero = got == 0.0
    assert _sha(np.packbits(zero)) == meta["zero_sha"]
    assert_bc(got[z["sample_idx"]], z["sample_val"])
    assert_bc(got[z["top_idx"]], z["top_val"])


# ------------------------------------------------------------------ extended-range sigma (NEXT-2)

def _assert_sigma_ext(mant, expo, m_ora, e_ora):
    """sigma as (mantissa, exponent): exact below 2^53, relative 1e-12 above (any range)."""
    zero = m_ora == 0
    assert np.all(mant[zero] == 0)
    small = ~zero & (e_ora <= 53)
    np.testing.assert_array_equal(np.ldexp(mant[small], expo[small]), np.ldexp(m_ora[small], e_ora[small]))
    big = ~zero & ~small
    rel = np.abs(mant[big] / m_ora[big] * np.exp2((expo[big] - e_ora[big]).astype(np.float64)) - 1.0)
    assert rel.size == 0 or rel.max() <= 1e-12, rel.max()


def test_xr_mesh_sigma_beyond_fp64():
    """700^2 mesh: sigma up to ~2^1393 from a corner, exported as mantissa + exponent, against the long
    double oracle; auto mode re-runs the overflowing sources in extended range."""
    g = gg.grid(700, 700)
    src = np.array([0, 699, 700 * 350 + 350, 700 * 700 - 1, 12345], dtype=np.int32)
    with tbc.Graph.from_csc(g.col_ptr, g.row_idx, False) as G:
        G.set_batch(tbc.ENGINE_NARROW)
        depth, mant, expo = G.bfs_batch_ext(src)
        assert G.stats()["xr_sources"] >= 3  # the corners overflow fp64
    assert expo.max() > 1300
    for i, s in enumerate(src):
        d_o, m_o, e_o = oracle.bfs_ld(g.col_ptr, g.row_idx, int(s))
        np.testing.assert_array_equal(depth[i], d_o)
        _assert_sigma_ext(mant[i], expo[i], m_o, e_o)


def test_xr_mesh_bc_vs_long_double_oracle():
    """bc on a 560^2 mesh (sigma ~2^1113 from a corner) with sources that overflow fp64 and others that
    do not, against the long double oracle (1e-9), in auto and forced extended mode."""
    g = gg.grid(560, 560)
    src = np.concatenate([[0, 559, 560 * 559, 560 * 560 - 1], gg.sources(g, 20, seed=3)]).astype(np.int32)
    want = oracle.bc_ld(g.col_ptr, g.row_idx, False, src)
    with tbc.Graph.from_csc(g.col_ptr, g.row_idx, False) as G:
        G.set_batch(tbc.ENGINE_NARROW)
        assert_bc(G.bc(src), want)
        assert G.stats()["xr_sources"] >= 4
        G.set_sigma_mode(1)
        G.reset_stats()
        assert_bc(G.bc(src), want)
        assert G.stats()["xr_sources"] == len(src)


@pytest.mark.parametrize("directed", [False, True])
def test_xr_forced_matches_fp64_oracle(directed):
    """Extended-range arithmetic everywhere (TBC_OPT_SIGMA = 1) on graphs fp64 handles: scale-free
    (hubs: warp paths of the sigma pull and the backward), small closed forms, random digraphs."""
    cases = [gg.kronecker(14, 16, seed=11, directed=directed, device="cuda"), gg.grid(40, 40)]
    if not directed:
        cases += [gg.star(9), gg.cycle(9), gg.complete_bipartite(3, 5), gg.mycielski(7)]
    for g in cases:
        src = gg.sources(g, min(g.n, 120), seed=4)
        with tbc.Graph.from_csc(g.col_ptr, g.row_idx, g.directed) as G:
            G.set_batch(tbc.ENGINE_NARROW)
            G.set_sigma_mode(1)
            assert_bc(G.bc(src), oracle.bc(g.col_ptr, g.row_idx, g.directed, src))
            depth, sigma = G.bfs_batch(src[:4])
            assert_bfs_rows(g, src[:4], depth, sigma)


def test_cfg8_literal_mesh_4096():
    """BASELINE configs[3] taken literally: the 4096^2 average-degree-4 mesh (sigma ~2^8190 from a
    corner).  One corner source's depth and sigma against the long double oracle, and the delta-sum
    invariant sum_v bc_s(v) = 1/2 sum_t (depth_s(t) - 1) for three sources, in the auto engine."""
    g, src = gg.make_config(8)
    corner = 0
    with tbc.Graph.from_csc(g.col_ptr, g.row_idx, False) as G:
        depth, mant, expo = G.bfs_batch_ext([corner])
        d_o, m_o, e_o = oracle.bfs_ld(g.col_ptr, g.row_idx, corner)
        np.testing.assert_array_equal(depth[0], d_o)
        _assert_sigma_ext(mant[0], expo[0], m_o, e_o)
        assert expo.max() > 8000
        for s in (corner, int(src[0]), int(src[1])):
            d = depth[0] if s == corner else G.bfs_batch([s])[0][0]
            want = 0.5 * float(np.sum(d[d > 0] - 1))
            got = G.bc([s]).sum()
            assert abs(got - want) <= 1e-9 * want
        assert G.stats()["engine"] == 2 and G.stats()["xr_sources"] >= 1
