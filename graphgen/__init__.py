"""Seeded synthetic graph generators shared by the oracle side and the CUDA side.

This module holds NONE of the method's arithmetic (no BFS, no path counting, no
dependency accumulation).  It only produces inputs: edge lists and their CSC form
(the input format of PAPER.md P:95-97: column v lists the rows u with A(u,v) = 1,
i.e. the edges u -> v), plus seeded source lists.

Workload recipes (restated in DESIGN.md "Inputs"):
  cfg1  Erdos-Renyi G(n=1024, M=4096) undirected, seed 1, all sources
  cfg2  RMAT/Kronecker scale 18, edgefactor 16, undirected, seed 2, 1024 sources
  cfg3  Graph500 Kronecker scale 22, edgefactor 16, DIRECTED, seed 3, 4096 sources
  cfg4  road-like 4096x4096 lattice: MST under iid U(0,1) weights + 10% of the other
        lattice edges, undirected, seed 4, 1024 sources
  cfg5  Graph500 Kronecker scale 25, edgefactor 16, undirected, seed 5, 8192 sources
Kronecker: A,B,C,D = 0.57,0.19,0.19,0.05 (Graph500), seeded label permutation,
self-loops and duplicates removed, undirected = symmetrised.
Sources: the first k of a seeded permutation of the vertices with out-degree >= 1.

Kronecker generation runs in torch on whatever device is given (CUDA for the big configs)
with a counter-based generator, so the host and the GPU produce the same graph bit for bit
(the oracle caches of tests/golden/ are computed from host-generated graphs).
"""
from __future__ import annotations

import dataclasses
import math

import numpy as np

try:  # torch is only needed for the large generators
    import torch
except Exception:  # pragma: no cover
    torch = None


@dataclasses.dataclass
class Graph:
    """A generated graph in CSC form (0-based, int64 col_ptr, int32 row_idx, sorted, deduplicated)."""
    name: str
    n: int
    col_ptr: np.ndarray
    row_idx: np.ndarray
    directed: bool

    @property
    def nnz(self) -> int:
        return int(self.col_ptr[-1])

    def out_degree(self) -> np.ndarray:
        return np.bincount(self.row_idx, minlength=self.n).astype(np.int64)

    def in_degree(self) -> np.ndarray:
        return np.diff(self.col_ptr)

    def edges(self):
        """(src, dst) int32 arrays of the stored edges src -> dst."""
        dst = np.repeat(np.arange(self.n, dtype=np.int32), np.diff(self.col_ptr))
        return self.row_idx.copy(), dst


# ----------------------------------------------------------------------------- CSC build

def csc_from_edges(n: int, src, dst, directed: bool):
    """Edge list src->dst -> canonical CSC (sorted, dedup, self-loops removed; symmetrised if undirected)."""
    src = np.asarray(src, dtype=np.int64)
    dst = np.asarray(dst, dtype=np.int64)
    keep = src != dst
    src, dst = src[keep], dst[keep]
    if not directed:
        src, dst = np.concatenate([src, dst]), np.concatenate([dst, src])
    key = np.unique(dst * n + src)           # column-major order: by dst, then src
    col = key // n
    row = (key - col * n).astype(np.int32)
    col_ptr = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(np.bincount(col, minlength=n), out=col_ptr[1:])
    return col_ptr, row


def csc_from_edges_torch(n: int, src, dst, directed: bool):
    """Same as :func:`csc_from_edges` but sorts on the tensors' device (for ~1e9-edge graphs)."""
    src = src.to(torch.int64)
    dst = dst.to(torch.int64)
    keep = src != dst
    src, dst = src[keep], dst[keep]
    if not directed:
        src, dst = torch.cat([src, dst]), torch.cat([dst, src])
    key = dst * n + src
    del src, dst
    key = torch.unique(key, sorted=True)
    col = key // n
    row = (key - col * n).to(torch.int32)
    counts = torch.bincount(col, minlength=n)
    del col, key
    col_ptr = torch.zeros(n + 1, dtype=torch.int64, device=row.device)
    col_ptr[1:] = torch.cumsum(counts, 0)
    return col_ptr.cpu().numpy(), row.cpu().numpy()


# ----------------------------------------------------------------------------- generators

def erdos_renyi(n: int, m_edges: int, seed: int, directed: bool = False) -> Graph:
    """G(n, M): M distinct uniformly random (unordered if undirected) pairs, no self-loops."""
    rng = np.random.default_rng(seed)
    chosen = set()
    pairs = []
    while len(pairs) < m_edges:
        u, v = (int(x) for x in rng.integers(0, n, size=2))
        if u == v:
            continue
        key = (u, v) if directed else (min(u, v), max(u, v))
        if key in chosen:
            continue
        chosen.add(key)
        pairs.append(key)
    p = np.asarray(pairs, dtype=np.int64).reshape(-1, 2)
    cp, ri = csc_from_edges(n, p[:, 0], p[:, 1], directed)
    return Graph(f"er_n{n}_M{m_edges}_s{seed}", n, cp, ri, directed)


def _s64(c: int) -> int:
    """An unsigned 64-bit constant as the signed int64 torch stores."""
    return c - (1 << 64) if c >= (1 << 63) else c


_GOLDEN = _s64(0x9E3779B97F4A7C15)
_MIX1 = _s64(0xBF58476D1CE4E5B9)
_MIX2 = _s64(0x94D049BB133111EB)


def _lsr(x, k: int):
    """Logical right shift of an int64 tensor (torch's >> is arithmetic)."""
    return (x >> k) & ((1 << (64 - k)) - 1)


def mix64(x):
    """splitmix64 finaliser of an int64 tensor, arithmetic mod 2^64 (two's complement wrap),
    computed in place (x is consumed).  A counter-based generator: the same counters give the
    same bits on CPU and CUDA, so a graph generated on the GPU is bit-identical to the one
    generated on the host."""
    y = x >> 30
    y &= (1 << 34) - 1
    x ^= y
    x *= _MIX1
    y = x >> 27
    y &= (1 << 37) - 1
    x ^= y
    x *= _MIX2
    y = x >> 31
    y &= (1 << 33) - 1
    x ^= y
    return x


def _stream_key(seed: int, stream: int) -> int:
    """Key of an independent counter stream (a pure-Python splitmix64 of (seed, stream))."""
    z = (seed * 0x9E3779B97F4A7C15 + stream * 0xD1B54A32D192ED03 + 0x632BE59BD9B4E019) % (1 << 64)
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) % (1 << 64)
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) % (1 << 64)
    return _s64(z ^ (z >> 31))


def kronecker(scale: int, edgefactor: int, seed: int, directed: bool, device: str = "cpu",
              abc=(0.57, 0.19, 0.19)) -> Graph:
    """Graph500 Kronecker/RMAT generator: edgefactor * 2^scale tuples, each bit of (src,dst)
    drawn from the 2x2 initiator (A,B;C,D), then a seeded vertex-label permutation.

    Randomness is counter-based (mix64 of (stream key + counter)): tuple t, bit b draws one
    64-bit word whose high / low 32 bits are the two uniforms of that bit, and the label
    permutation sorts the vertices by mix64 of (key + v).  Every step is integer or exact
    fp64 arithmetic, so device="cpu" and device="cuda" give the same graph bit for bit."""
    if torch is None:
        raise RuntimeError("torch required for kronecker()")
    n = 1 << scale
    m_t = edgefactor * n
    a, b, c = abc
    src = torch.zeros(m_t, dtype=torch.int64, device=device)
    dst = torch.zeros(m_t, dtype=torch.int64, device=device)
    ab = a + b
    c_norm = c / (1.0 - ab)
    a_norm = a / ab
    key_bits = _stream_key(seed, 1)
    key_perm = _stream_key(seed, 2)
    # integer thresholds: bit i of the source is 1 iff the high 32-bit draw exceeds
    # floor((A+B) 2^32), i.e. with probability C+D; bit j of the destination is 1 iff the low
    # draw exceeds floor(C/(C+D) 2^32) when i = 1, floor(A/(A+B) 2^32) when i = 0
    t_ab = int(ab * 4294967296.0)
    t_c = int(c_norm * 4294967296.0)
    t_a = int(a_norm * 4294967296.0)
    chunk = 1 << 24
    for lo in range(0, m_t, chunk):
        hi = min(m_t, lo + chunk)
        s = src[lo:hi]
        d = dst[lo:hi]
        ctr = torch.arange(lo, hi, dtype=torch.int64, device=device) * scale + key_bits
        for bit in range(scale):
            h = mix64(ctr + bit)
            ii = _lsr(h, 32) > t_ab
            h &= 0xFFFFFFFF
            jj = h > torch.where(ii, t_c, t_a)
            s |= ii.to(torch.int64) << bit
            d |= jj.to(torch.int64) << bit
        del ctr
    perm = torch.sort(mix64(torch.arange(n, dtype=torch.int64, device=device) + key_perm), stable=True).indices
    src = perm[src]
    dst = perm[dst]
    del perm
    if device == "cpu":
        cp, ri = _csc_lean_host(n, src, dst, directed)
    else:
        cp, ri = csc_from_edges_torch(n, src, dst, directed)
    kind = "dir" if directed else "undir"
    return Graph(f"kron_s{scale}_ef{edgefactor}_{kind}_seed{seed}", n, cp, ri, directed)


def _csc_lean_host(n: int, src, dst, directed: bool):
    """csc_from_edges for large host tensors with a small memory peak: keys (column-major) built
    in place, sorted in place, duplicates compressed out.  Same result as csc_from_edges_torch."""
    s = src.numpy()
    d = dst.numpy()
    keep = s != d
    m = int(keep.sum())
    key = np.empty(m if directed else 2 * m, dtype=np.int64)
    np.multiply(d[keep], n, out=key[:m])
    key[:m] += s[keep]
    if not directed:
        np.multiply(s[keep], n, out=key[m:])
        key[m:] += d[keep]
    del s, d, keep, src, dst
    key.sort()  # introsort, in place (no second copy of the keys)
    uniq = np.empty(key.size, dtype=bool)
    uniq[:1] = True
    np.not_equal(key[1:], key[:-1], out=uniq[1:])
    key = key[uniq]
    del uniq
    col = key // n
    row = (key - col * n).astype(np.int32)
    del key
    col_ptr = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(np.bincount(col, minlength=n), out=col_ptr[1:])
    return col_ptr, row


def road_lattice(side: int, q: float, seed: int) -> Graph:
    """Road-like lattice: the minimum spanning tree of the side x side 4-neighbour grid under iid
    U(0,1) edge weights, plus each remaining grid edge independently with probability q."""
    from scipy.sparse import coo_matrix
    from scipy.sparse.csgraph import minimum_spanning_tree
    rng = np.random.default_rng(seed)
    n = side * side
    idx = np.arange(n, dtype=np.int64).reshape(side, side)
    h_u, h_v = idx[:, :-1].ravel(), idx[:, 1:].ravel()
    v_u, v_v = idx[:-1, :].ravel(), idx[1:, :].ravel()
    eu = np.concatenate([h_u, v_u])
    ev = np.concatenate([h_v, v_v])
    w = rng.random(eu.size) + 1e-12  # strictly positive so scipy keeps every edge
    mst = minimum_spanning_tree(coo_matrix((w, (eu, ev)), shape=(n, n)).tocsr()).tocoo()
    in_tree = np.zeros(eu.size, dtype=bool)
    # identify tree edges by key
    tkey = np.minimum(mst.row, mst.col).astype(np.int64) * n + np.maximum(mst.row, mst.col)
    ekey = np.minimum(eu, ev) * n + np.maximum(eu, ev)
    in_tree[np.isin(ekey, tkey)] = True
    extra = (~in_tree) & (rng.random(eu.size) < q)
    keep = in_tree | extra
    cp, ri = csc_from_edges(n, eu[keep], ev[keep], directed=False)
    return Graph(f"road_{side}x{side}_q{q}_s{seed}", n, cp, ri, False)


def grid(a: int, b: int) -> Graph:
    """P_a x P_b grid graph (undirected); vertex (i, j) has id i*b + j."""
    idx = np.arange(a * b).reshape(a, b)
    eu = np.concatenate([idx[:, :-1].ravel(), idx[:-1, :].ravel()])
    ev = np.concatenate([idx[:, 1:].ravel(), idx[1:, :].ravel()])
    cp, ri = csc_from_edges(a * b, eu, ev, directed=False)
    return Graph(f"grid_{a}x{b}", a * b, cp, ri, False)


def from_edges(name: str, n: int, edges, directed: bool) -> Graph:
    e = np.asarray(list(edges), dtype=np.int64).reshape(-1, 2)
    cp, ri = csc_from_edges(n, e[:, 0], e[:, 1], directed)
    return Graph(name, n, cp, ri, directed)


def star(n: int, directed_both: bool = False) -> Graph:
    """K_{1,n-1} with centre 0. directed_both: the same symmetric pattern flagged directed."""
    e = [(0, i) for i in range(1, n)]
    g = from_edges(f"star{n}", n, e, directed=False)
    g.directed = directed_both
    return g


def path(n: int, directed: bool = False) -> Graph:
    return from_edges(f"path{n}", n, [(i, i + 1) for i in range(n - 1)], directed)


def cycle(n: int) -> Graph:
    return from_edges(f"cycle{n}", n, [(i, (i + 1) % n) for i in range(n)], False)


def complete(n: int) -> Graph:
    return from_edges(f"K{n}", n, [(i, j) for i in range(n) for j in range(i + 1, n)], False)


def complete_bipartite(a: int, b: int) -> Graph:
    return from_edges(f"K{a},{b}", a + b, [(i, a + j) for i in range(a) for j in range(b)], False)


def random_tree(n: int, seed: int) -> Graph:
    rng = np.random.default_rng(seed)
    e = [(int(rng.integers(0, i)), i) for i in range(1, n)]
    return from_edges(f"tree{n}_s{seed}", n, e, False)


def mycielski(k: int, device: str = "cpu") -> Graph:
    """Mycielski graph M_k (networkx convention: M_1 = K_1, M_2 = K_2); the paper's
    'mycielski15..19' (Table 3) are M_15..M_19 of SuiteSparse.  device="cuda" builds
    the edge list and the CSC with torch on the GPU (M_19 has 903 M stored entries)."""
    if k == 1:
        return from_edges("mycielski1", 1, [], False)
    xp_cat = np.concatenate if device == "cpu" else torch.cat
    if device == "cpu":
        arange = lambda a, b: np.arange(a, b, dtype=np.int64)  # noqa: E731
        full = lambda c, v: np.full(c, v, dtype=np.int64)  # noqa: E731
        eu, ev = np.array([0], dtype=np.int64), np.array([1], dtype=np.int64)
    else:
        arange = lambda a, b: torch.arange(a, b, dtype=torch.int64, device=device)  # noqa: E731
        full = lambda c, v: torch.full((c,), v, dtype=torch.int64, device=device)  # noqa: E731
        eu = torch.tensor([0], dtype=torch.int64, device=device)
        ev = torch.tensor([1], dtype=torch.int64, device=device)
    n = 2
    for _ in range(k - 2):
        # Mycielskian: copies u_i = i + n adjacent to N(v_i), hub w = 2n adjacent to all u_i
        ui = arange(n, 2 * n)
        eu, ev = (xp_cat([eu, eu, eu + n, ui]), xp_cat([ev, ev + n, ev, full(n, 2 * n)]))
        n = 2 * n + 1
    if device == "cpu":
        cp, ri = csc_from_edges(n, eu, ev, directed=False)
    else:
        cp, ri = csc_from_edges_torch(n, eu, ev, directed=False)
    return Graph(f"mycielski{k}", n, cp, ri, False)


# ----------------------------------------------------------------------------- sources

def sources(g: Graph, k: int, seed: int) -> np.ndarray:
    """First k of a seeded permutation of the vertices with out-degree >= 1."""
    cand = np.nonzero(g.out_degree() > 0)[0].astype(np.int32)
    rng = np.random.default_rng(seed)
    perm = rng.permutation(cand.size)
    if k > cand.size:
        reps = math.ceil(k / max(cand.size, 1))
        perm = np.concatenate([rng.permutation(cand.size) for _ in range(reps)])
    return cand[perm[:k]].astype(np.int32)


# ----------------------------------------------------------------------------- configs

CONFIGS = {
    1: dict(name="cfg1_er1024", kind="er", n=1024, M=4096, seed=1, directed=False, k=1024, src_seed=None),
    2: dict(name="cfg2_rmat18_undir", kind="kron", scale=18, ef=16, seed=2, directed=False, k=1024, src_seed=12),
    3: dict(name="cfg3_kron22_dir", kind="kron", scale=22, ef=16, seed=3, directed=True, k=4096, src_seed=13),
    4: dict(name="cfg4_road4096", kind="road", side=4096, q=0.10, seed=4, directed=False, k=1024, src_seed=14),
    5: dict(name="cfg5_kron25_undir", kind="kron", scale=25, ef=16, seed=5, directed=False, k=8192, src_seed=15),
    # the paper's own best-case inputs, reproduced exactly up to vertex labels:
    # exact BC of mycielski16 (Table 5) and single sources of mycielski19 (Table 3)
    6: dict(name="cfg6_mycielski16_exact", kind="myc", myc=16, directed=False, k=None, src_seed=None),
    7: dict(name="cfg7_mycielski19_sources", kind="myc", myc=19, directed=False, k=1024, src_seed=17),
    # the literal average-degree-4 mesh of BASELINE configs[3] (4096 x 4096 grid): sigma overflows
    # fp64 (C(i+j, i) ~ 2^8190 from a corner), runnable with extended-range sigma
    8: dict(name="cfg8_mesh4096_literal", kind="mesh", side=4096, directed=False, k=1024, src_seed=18),
}


def make_config(cfg: int, device: str = "cpu", scale_override: int | None = None,
                side_override: int | None = None):
    """(Graph, sources) for config 1..7; overrides shrink the graph for fast tests."""
    c = CONFIGS[cfg]
    if c["kind"] == "er":
        g = erdos_renyi(c["n"], c["M"], c["seed"], c["directed"])
        src = np.arange(g.n, dtype=np.int32)            # exact BC: all sources (Alg.1 l.6)
    elif c["kind"] == "kron":
        g = kronecker(scale_override or c["scale"], c["ef"], c["seed"], c["directed"], device=device)
        src = sources(g, c["k"], c["src_seed"])
    elif c["kind"] == "myc":
        g = mycielski(c["myc"], device=device)
        src = np.arange(g.n, dtype=np.int32) if c["k"] is None else sources(g, c["k"], c["src_seed"])
    elif c["kind"] == "mesh":
        side = side_override or c["side"]
        g = grid(side, side)
        src = sources(g, c["k"], c["src_seed"])
    else:
        g = road_lattice(side_override or c["side"], c["q"], c["seed"])
        src = sources(g, c["k"], c["src_seed"])
    return g, src
