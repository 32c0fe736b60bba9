"""Exact brute force of Freeman's definition -- TEST INFRASTRUCTURE ONLY (see oracle/__init__).

Eq. 1:  BC(v) = sum_{s != v != t} sigma_st(v) / sigma_st,
with sigma_st(v)/sigma_st := 0 when sigma_st = 0, computed the "straightforward" way
P:76 describes: all-pairs shortest-path lengths and counts first, then, for every v,
every pair (s, t).

  * d(s, t): all-pairs BFS distances.
  * sigma_st = (A^{d(s,t)})[s, t] -- walks of length d(s,t) from s to t are exactly the
    shortest paths, so integer matrix powers count them.
  * sigma_st(v) = sigma_sv * sigma_vt  if d(s,v) + d(v,t) = d(s,t), else 0.
  * undirected graphs: the ordered-pair sum counts each pair twice, halved per P:180.

Exact rationals (fractions.Fraction) throughout; for n <= 12 only.
The ``sources`` argument restricts s to a list (Alg.1 l.6 generalised).
"""
from __future__ import annotations

from fractions import Fraction


def adjacency_from_csc(col_ptr, row_idx):
    """Boolean A with A[u][v] = 1 iff row u is stored in column v (edge u->v)."""
    n = len(col_ptr) - 1
    A = [[0] * n for _ in range(n)]
    for v in range(n):
        for k in range(int(col_ptr[v]), int(col_ptr[v + 1])):
            A[int(row_idx[k])][v] = 1
    return A


def _matmul(X, Y):
    n = len(X)
    return [[sum(X[i][k] * Y[k][j] for k in range(n)) for j in range(n)] for i in range(n)]


def all_pairs(A):
    """(dist, sigma): dist[s][t] BFS distance (-1 unreachable), sigma[s][t] shortest-path count."""
    n = len(A)
    dist = [[-1] * n for _ in range(n)]
    for s in range(n):
        dist[s][s] = 0
        frontier = [s]
        d = 0
        while frontier:
            d += 1
            nxt = []
            for u in frontier:
                for v in range(n):
                    if A[u][v] and dist[s][v] < 0:
                        dist[s][v] = d
                        nxt.append(v)
            frontier = nxt
    # walk counts by matrix powers: P[k] = A^k
    maxd = max(max(r) for r in dist)
    powers = [[[int(i == j) for j in range(n)] for i in range(n)]]
    for _ in range(max(maxd, 0)):
        powers.append(_matmul(powers[-1], A))
    sigma = [[0] * n for _ in range(n)]
    for s in range(n):
        for t in range(n):
            if dist[s][t] >= 0:
                sigma[s][t] = powers[dist[s][t]][s][t]
    return dist, sigma


def bc_exact(A, directed: bool, sources=None):
    """Eq. 1 summed literally over s in sources (default all), t in V; list of Fractions."""
    n = len(A)
    dist, sigma = all_pairs(A)
    srcs = range(n) if sources is None else sources
    bc = [Fraction(0)] * n
    for s in srcs:
        for t in range(n):
            if t == s or sigma[s][t] == 0:
                continue
            for v in range(n):
                if v == s or v == t:
                    continue
                if dist[s][v] >= 0 and dist[v][t] >= 0 and dist[s][v] + dist[v][t] == dist[s][t]:
                    bc[v] += Fraction(sigma[s][v] * sigma[v][t], sigma[s][t])
    if not directed:
        bc = [x / 2 for x in bc]
    return bc
