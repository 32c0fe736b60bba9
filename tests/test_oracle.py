"""Pins for the CPU oracle (oracle/), independent of the CUDA path.  CPU only.

Each test pins the oracle to something other than itself (SURVEY.md 8(c) pin table):
  c-1 depth  : BFS certificate, brute-force distances, grid corner depth i+j
  c-2 sigma  : sigma certificate, walk counts (brute force), grid C(i+j,i), trees = 1
  c-3 delta  : sum_v delta_s(v) = sum_t (depth(t)-1); tree descendants
  c-4 bc     : brute-force Eq. 1 with rationals (all small graphs), closed forms,
               networkx betweenness_centrality_subset, label-permutation equivariance
  c-5 paper  : Table 3 mycielski n, m, and d = BFS height + 1 = 3
"""
import itertools
import math
import random

import networkx as nx
import numpy as np
import pytest

import graphgen as gg
from oracle import brute
from tbc_testutil import golden


def csc_from_A(A, directed=True):
    n = len(A)
    e = [(u, v) for u in range(n) for v in range(n) if A[u][v]]
    return gg.from_edges("A", n, e, directed)


def assert_bc_close(got, exact, rel=1e-12):
    exact = np.asarray([float(x) for x in exact])
    got = np.asarray(got)
    zero = exact == 0
    assert np.all(got[zero] == 0.0), (got, exact)
    np.testing.assert_allclose(got[~zero], exact[~zero], rtol=rel, atol=0)


# ------------------------------------------------------------------ c-4 brute force, exhaustive

def _undirected_graphs(n):
    pairs = list(itertools.combinations(range(n), 2))
    for mask in range(1 << len(pairs)):
        yield [p for i, p in enumerate(pairs) if mask >> i & 1]


@pytest.mark.parametrize("n", [2, 3, 4, 5, 6])
def test_bc_vs_bruteforce_all_undirected(oracle_lib, n):
    """Every undirected graph on n <= 6 vertices (2^15 at n=6): Eq. 1 exactly / 2."""
    for edges in _undirected_graphs(n):
        g = gg.from_edges("u", n, edges, directed=False)
        A = brute.adjacency_from_csc(g.col_ptr, g.row_idx)
        exact = brute.bc_exact(A, directed=False)
        got = oracle_lib.bc(g.col_ptr, g.row_idx, False, np.arange(n), nthreads=1)
        assert_bc_close(got, exact)


@pytest.mark.parametrize("n", [2, 3, 4])
def test_bc_vs_bruteforce_all_digraphs(oracle_lib, n):
    """Every digraph on n <= 4 vertices (2^12 at n=4), no halving for directed graphs."""
    arcs = [(u, v) for u in range(n) for v in range(n) if u != v]
    for mask in range(1 << len(arcs)):
        edges = [a for i, a in enumerate(arcs) if mask >> i & 1]
        g = gg.from_edges("d", n, edges, directed=True)
        A = brute.adjacency_from_csc(g.col_ptr, g.row_idx)
        exact = brute.bc_exact(A, directed=True)
        got = oracle_lib.bc(g.col_ptr, g.row_idx, True, np.arange(n), nthreads=1)
        assert_bc_close(got, exact)


def test_bc_vs_bruteforce_random_upto12_with_source_lists(oracle_lib):
    """Random graphs n <= 12, directed and undirected, partial source lists with repeats."""
    rng = random.Random(12)
    for trial in range(120):
        n = rng.randint(1, 12)
        directed = trial % 2 == 0
        p = rng.choice([0.1, 0.25, 0.5])
        if directed:
            edges = [(u, v) for u in range(n) for v in range(n) if u != v and rng.random() < p]
        else:
            edges = [(u, v) for u, v in itertools.combinations(range(n), 2) if rng.random() < p]
        g = gg.from_edges("r", n, edges, directed)
        A = brute.adjacency_from_csc(g.col_ptr, g.row_idx)
        k = rng.randint(0, 2 * n)
        src = [rng.randrange(n) for _ in range(k)]
        exact = brute.bc_exact(A, directed, sources=src)
        got = oracle_lib.bc(g.col_ptr, g.row_idx, directed, np.asarray(src, dtype=np.int32),
                            nthreads=rng.randint(1, 4))
        assert_bc_close(got, exact)


# ------------------------------------------------------------------ c-4 closed forms (golden)

def test_closed_forms(oracle_lib):
    for c in golden("closed_forms.json")["cases"]:
        if c["graph"] == "star":
            g = gg.star(c["n"], directed_both=c["directed_flag"])
            got = oracle_lib.bc(g.col_ptr, g.row_idx, g.directed, np.arange(g.n))
            np.testing.assert_allclose(got, c["bc"], rtol=1e-14)
        elif c["graph"] == "path":
            g = gg.path(c["n"], directed=c["directed"])
            got = oracle_lib.bc(g.col_ptr, g.row_idx, c["directed"], np.arange(g.n))
            np.testing.assert_allclose(got, c["bc"], rtol=1e-14)
        elif c["graph"] == "cycle":
            g = gg.cycle(c["n"])
            got = oracle_lib.bc(g.col_ptr, g.row_idx, False, np.arange(g.n))
            np.testing.assert_allclose(got, c["bc_each"], rtol=1e-14)
        elif c["graph"] == "complete":
            g = gg.complete(c["n"])
            got = oracle_lib.bc(g.col_ptr, g.row_idx, False, np.arange(g.n))
            assert np.all(got == 0.0)
        elif c["graph"] == "complete_bipartite":
            a, b = c["a"], c["b"]
            g = gg.complete_bipartite(a, b)
            got = oracle_lib.bc(g.col_ptr, g.row_idx, False, np.arange(g.n))
            np.testing.assert_allclose(got[:a], c["bc_a"], rtol=1e-14)
            np.testing.assert_allclose(got[a:], c["bc_b"], rtol=1e-14)


@pytest.mark.parametrize("n", [3, 10, 101])
def test_closed_form_families_scaled(oracle_lib, n):
    """The same formulas at other sizes (n-dependence is where dropped terms show)."""
    g = gg.star(n)
    got = oracle_lib.bc(g.col_ptr, g.row_idx, False, np.arange(n))
    assert got[0] == (n - 1) * (n - 2) / 2 and np.all(got[1:] == 0)
    g = gg.path(n)
    got = oracle_lib.bc(g.col_ptr, g.row_idx, False, np.arange(n))
    np.testing.assert_allclose(got, [i * (n - 1 - i) for i in range(n)], rtol=1e-13)
    g = gg.path(n, directed=True)
    got = oracle_lib.bc(g.col_ptr, g.row_idx, True, np.arange(n))
    np.testing.assert_allclose(got, [i * (n - 1 - i) for i in range(n)], rtol=1e-13)
    g = gg.cycle(n)
    want = (n - 2) ** 2 / 8 if n % 2 == 0 else (n - 1) * (n - 3) / 8
    np.testing.assert_allclose(oracle_lib.bc(g.col_ptr, g.row_idx, False, np.arange(n)), want, rtol=1e-12)


@pytest.mark.parametrize("seed", range(5))
def test_trees_components_formula(oracle_lib, seed):
    """Trees: BC(v) = sum over unordered pairs of components of T - v of |Ci||Cj| (one path per pair)."""
    g = gg.random_tree(60, seed)
    src, dst = g.edges()
    T = nx.Graph()
    T.add_nodes_from(range(g.n))
    T.add_edges_from(zip(src.tolist(), dst.tolist()))
    want = []
    for v in range(g.n):
        H = T.copy()
        H.remove_node(v)
        sizes = [len(c) for c in nx.connected_components(H)]
        tot = sum(sizes)
        want.append((tot * tot - sum(s * s for s in sizes)) / 2)
    got = oracle_lib.bc(g.col_ptr, g.row_idx, False, np.arange(g.n))
    np.testing.assert_allclose(got, want, rtol=1e-13)
    # sigma == 1 on trees, delta_s(v) = number of descendants of v rooted at s
    for s in (0, 17, 59):
        depth, sigma = oracle_lib.bfs(g.col_ptr, g.row_idx, s)
        assert np.all(sigma == 1.0)
        delta = oracle_lib.delta(g.col_ptr, g.row_idx, s)
        for v in range(g.n):
            if v == s:
                assert delta[v] == 0.0
                continue
            H = T.copy()
            H.remove_edge(v, next(u for u in T.neighbors(v) if depth[u] == depth[v] - 1))
            sub = nx.node_connected_component(H, v)
            assert delta[v] == len(sub) - 1


# ------------------------------------------------------------------ c-1, c-2 depth and sigma

def test_grid_sigma_binomial_and_depth(oracle_lib):
    """P_a x P_b grid from the corner: depth(i,j) = i+j and sigma(i,j) = C(i+j, i); crosses 2^53."""
    a = b = 32
    g = gg.grid(a, b)
    depth, sigma = oracle_lib.bfs(g.col_ptr, g.row_idx, 0)
    for i in range(a):
        for j in range(b):
            assert depth[i * b + j] == i + j
            exact = math.comb(i + j, i)
            if exact < 2 ** 53:
                assert sigma[i * b + j] == float(exact)
            else:
                assert abs(sigma[i * b + j] - exact) <= 1e-12 * exact


def _certify_bfs(g, s, depth, sigma):
    """Graph500-style certificate for depth, plus the sigma recurrence, checked edge by edge."""
    src, dst = g.edges()
    assert depth[s] == 0 and sigma[s] == 1.0
    du, dv = depth[src], depth[dst]
    reached_u = du >= 0
    assert np.all(dv[reached_u] >= 0)
    assert np.all(dv[reached_u] <= du[reached_u] + 1)
    # every reached v != s has a parent at depth(v)-1; sigma(v) = sum of parents' sigma
    parent = (du >= 0) & (dv == du + 1)
    acc = np.zeros(g.n)
    np.add.at(acc, dst[parent], sigma[src[parent]])
    reached = depth >= 0
    nz = reached.copy()
    nz[s] = False
    assert np.all(acc[nz] > 0)
    np.testing.assert_allclose(sigma[nz], acc[nz], rtol=1e-15)
    assert np.all(sigma[~reached] == 0)


@pytest.mark.parametrize("directed", [False, True])
def test_bfs_certificate_random(oracle_lib, directed):
    g = gg.kronecker(11, 8, seed=7, directed=directed)
    for s in gg.sources(g, 6, seed=1):
        depth, sigma = oracle_lib.bfs(g.col_ptr, g.row_idx, int(s))
        _certify_bfs(g, int(s), depth, sigma)


def test_bfs_vs_bruteforce_small(oracle_lib):
    rng = random.Random(3)
    for _ in range(60):
        n = rng.randint(1, 10)
        edges = [(u, v) for u in range(n) for v in range(n) if u != v and rng.random() < 0.25]
        g = gg.from_edges("b", n, edges, True)
        A = brute.adjacency_from_csc(g.col_ptr, g.row_idx)
        dist, sig = brute.all_pairs(A)
        for s in range(n):
            depth, sigma = oracle_lib.bfs(g.col_ptr, g.row_idx, s)
            assert list(depth) == dist[s]
            assert list(sigma) == [float(x) for x in sig[s]]


# ------------------------------------------------------------------ c-3 delta invariant

@pytest.mark.parametrize("directed", [False, True])
def test_delta_sum_invariant(oracle_lib, directed):
    """sum_{v != s} delta_s(v) = sum_{t reached, t != s} (depth_s(t) - 1): each shortest s-t path
    has depth(t)-1 interior vertices, and delta_s(v) sums the fractions through v (Eq. 2)."""
    g = gg.kronecker(10, 8, seed=9, directed=directed)
    for s in gg.sources(g, 5, seed=2):
        s = int(s)
        depth, _ = oracle_lib.bfs(g.col_ptr, g.row_idx, s)
        delta = oracle_lib.delta(g.col_ptr, g.row_idx, s)
        want = float(np.sum(depth[depth > 0] - 1))
        assert abs(delta.sum() - want) <= 1e-9 * max(want, 1.0)
        # and bc from the single source equals delta (halved when undirected)
        bc1 = oracle_lib.bc(g.col_ptr, g.row_idx, directed, [s])
        np.testing.assert_allclose(bc1, delta * (1.0 if directed else 0.5), rtol=1e-15, atol=0)


# ------------------------------------------------------------------ c-4 library special case

@pytest.mark.parametrize("directed", [False, True])
def test_vs_networkx_subset(oracle_lib, directed):
    """networkx.betweenness_centrality_subset(normalized=False) applies the same per-source 1/2 for
    undirected graphs; sources with repeats are not supported there, so use a set."""
    g = gg.kronecker(9, 6, seed=11, directed=directed)
    src, dst = g.edges()
    G = nx.DiGraph() if directed else nx.Graph()
    G.add_nodes_from(range(g.n))
    G.add_edges_from(zip(src.tolist(), dst.tolist()))
    S = sorted(set(gg.sources(g, 40, seed=4).tolist()))
    want = nx.betweenness_centrality_subset(G, S, list(range(g.n)), normalized=False)
    got = oracle_lib.bc(g.col_ptr, g.row_idx, directed, np.asarray(S, dtype=np.int32))
    np.testing.assert_allclose(got, [want[v] for v in range(g.n)], rtol=1e-10, atol=1e-12)


def test_permutation_equivariance(oracle_lib):
    g = gg.kronecker(9, 8, seed=5, directed=True)
    rng = np.random.default_rng(0)
    perm = rng.permutation(g.n)
    src, dst = g.edges()
    h = gg.from_edges("p", g.n, np.stack([perm[src], perm[dst]], 1), True)
    S = gg.sources(g, 30, seed=1)
    a = oracle_lib.bc(g.col_ptr, g.row_idx, True, S)
    b = oracle_lib.bc(h.col_ptr, h.row_idx, True, perm[S].astype(np.int32))
    np.testing.assert_allclose(b[perm], a, rtol=1e-12, atol=1e-12)


# ------------------------------------------------------------------ c-5 paper-printed values

def test_paper_table3_mycielski_shape_and_depth(oracle_lib):
    """Table 3: n, m (stored nnz) of mycielski15..19 and d = 3 (= height + 1).
    n and m follow from the recurrence, so check all rows; BFS heights on mycielski15."""
    for row in golden("paper_table3_mycielski.json")["rows"]:
        k = row["k"]
        n = 3 * 2 ** (k - 2) - 1
        e = 1
        nn = 2
        for _ in range(k - 2):
            e, nn = 3 * e + nn, 2 * nn + 1
        assert round(n / 1000) == row["n_thousands"]
        # mycielski16 prints 33383 for 2e = 33,382,480 -- every other row is 2e rounded to
        # thousands, so the table's last digit is taken as +-1 (reading R16)
        assert abs(round(2 * e / 1000) - row["m_thousands"]) <= 1
    g = gg.mycielski(15)
    assert g.n == 24575 and round(g.nnz / 1000) == 11111
    for s in (0, 1, 12345, g.n - 1):
        depth, _ = oracle_lib.bfs(g.col_ptr, g.row_idx, s)
        assert depth.max() + 1 == 3          # printed d = height + 1 (reading 15)
    for k in range(4, 9):
        h = gg.mycielski(k)
        for s in range(h.n):
            depth, _ = oracle_lib.bfs(h.col_ptr, h.row_idx, s)
            assert depth.min() >= 0 and depth.max() == 2


# ------------------------------------------------------------------ edge cases

def test_edge_cases(oracle_lib):
    g = gg.from_edges("one", 1, [], False)
    assert list(oracle_lib.bc(g.col_ptr, g.row_idx, False, [0])) == [0.0]
    g = gg.path(5)
    assert np.all(oracle_lib.bc(g.col_ptr, g.row_idx, False, []) == 0)
    # repeated sources count each occurrence
    one = oracle_lib.bc(g.col_ptr, g.row_idx, False, [1])
    three = oracle_lib.bc(g.col_ptr, g.row_idx, False, [1, 1, 1])
    np.testing.assert_array_equal(three, 3 * one)
    # duplicates and self-loops in the input CSC change nothing (A is boolean)
    cp = np.array([0, 3, 6, 8], dtype=np.int64)
    ri = np.array([1, 1, 0, 0, 2, 2, 1, 1], dtype=np.int32)   # path 0-1-2 with dups + self-loop at 0
    clean = gg.path(3)
    np.testing.assert_array_equal(oracle_lib.bc(cp, ri, False, [0, 1, 2]),
                                  oracle_lib.bc(clean.col_ptr, clean.row_idx, False, [0, 1, 2]))
    # isolated source: nothing reached
    g = gg.from_edges("iso", 4, [(1, 2), (2, 3)], False)
    assert np.all(oracle_lib.bc(g.col_ptr, g.row_idx, False, [0]) == 0)
    depth, sigma = oracle_lib.bfs(g.col_ptr, g.row_idx, 0)
    assert list(depth) == [0, -1, -1, -1] and list(sigma) == [1, 0, 0, 0]
    with pytest.raises(ValueError):
        oracle_lib.bc(g.col_ptr, g.row_idx, False, [7])


# ------------------------------------------------------------------ extended-range oracle (NEXT-2)

def _ld_value_vs_int(mant, expo, exact: int, rel: float):
    """|mant * 2^expo - exact| <= rel * exact, in exact integer arithmetic (values beyond fp64)."""
    M = int(float(mant) * 2 ** 53)  # the double mantissa times 2^53 is an integer
    e = int(expo) - 53
    approx_num, approx_den = (M << e, 1) if e >= 0 else (M, 1 << -e)
    diff = abs(approx_num - exact * approx_den)
    return diff * (10 ** 15) <= int(rel * 1e15) * exact * approx_den


def test_ld_grid_sigma_binomial_beyond_fp64(oracle_lib):
    """700 x 700 mesh from the corner: sigma(i,j) = C(i+j, i) up to ~2^1393 (> DBL_MAX ~ 2^1024),
    depth(i,j) = i+j.  Exact below 2^64, relative 1e-15 above (64-bit long double mantissa)."""
    a = b = 700
    g = gg.grid(a, b)
    depth, mant, expo = oracle_lib.bfs_ld(g.col_ptr, g.row_idx, 0)
    assert expo.max() > 1300
    rng = np.random.default_rng(3)
    cells = [(i, j) for i in range(0, a, 37) for j in range(0, b, 41)] + [(a - 1, b - 1), (a - 1, 0), (0, b - 1)]
    cells += [tuple(x) for x in rng.integers(0, a, size=(200, 2))]
    for i, j in cells:
        v = i * b + j
        assert depth[v] == i + j
        assert _ld_value_vs_int(mant[v], expo[v], math.comb(i + j, i), 1e-15), (i, j)


def test_ld_matches_fp64_and_bruteforce_small(oracle_lib):
    """Where fp64 does not overflow, the long double oracle equals the fp64 oracle and Eq. 1."""
    rng = random.Random(5)
    for trial in range(40):
        n = rng.randint(1, 11)
        directed = trial % 2 == 1
        edges = [(u, v) for u in range(n) for v in range(n) if u != v and rng.random() < 0.3]
        if not directed:
            edges = [(u, v) for u, v in edges if u < v]
        g = gg.from_edges("r", n, edges, directed)
        src = np.asarray([rng.randrange(n) for _ in range(rng.randint(0, 2 * n))], dtype=np.int32)
        exact = brute.bc_exact(brute.adjacency_from_csc(g.col_ptr, g.row_idx), directed, sources=list(src))
        got = oracle_lib.bc_ld(g.col_ptr, g.row_idx, directed, src)
        assert_bc_close(got, exact)
        np.testing.assert_allclose(got, oracle_lib.bc(g.col_ptr, g.row_idx, directed, src), rtol=1e-13, atol=0)
        if n:
            d1, s1 = oracle_lib.bfs(g.col_ptr, g.row_idx, 0)
            d2, m2, e2 = oracle_lib.bfs_ld(g.col_ptr, g.row_idx, 0)
            np.testing.assert_array_equal(d1, d2)
            np.testing.assert_array_equal(np.ldexp(m2, e2), s1)


def test_ld_delta_sum_invariant_on_overflowing_mesh(oracle_lib):
    """Backward stage in extended range: on a 600 x 600 mesh (sigma ~2^1195 from a corner), one source's
    sum_v delta_s(v) = sum_t (depth_s(t) - 1) (each shortest path's interior vertices), halved if
    undirected -- exact integer, checked to 1e-12 relative; and delta is finite everywhere."""
    g = gg.grid(600, 600)
    for s in (0, 600 * 300 + 300, 600 * 599 + 17):
        depth, _, expo = oracle_lib.bfs_ld(g.col_ptr, g.row_idx, s)
        bc = oracle_lib.bc_ld(g.col_ptr, g.row_idx, False, [s])
        want = 0.5 * float(np.sum(depth[depth > 0] - 1))
        assert np.all(np.isfinite(bc))
        assert abs(bc.sum() - want) <= 1e-12 * want
        if s == 0:
            assert expo.max() > 1100
