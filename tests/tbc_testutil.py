"""Shared helpers for the test-suite: fixture loading and the parity bars (no method arithmetic).

Bars (BASELINE.json north star):
  depth  bit-exact;  sigma bit-exact while < 2^53 (relative 1e-12 above);
  bc     |gpu - ora| <= 1e-9 |ora|, and ora == 0  =>  gpu == 0 exactly.
"""
import json
import os

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def golden(name):
    """Load a fixture from tests/golden/ (each one states its citation)."""
    with open(os.path.join(ROOT, "tests", "golden", name)) as f:
        return json.load(f)


def assert_bc(got, want, rel=1e-9):
    got = np.asarray(got)
    want = np.asarray(want)
    zero = want == 0
    assert np.all(got[zero] == 0.0), np.nonzero(got[zero])[0][:10]
    err = np.abs(got[~zero] - want[~zero]) / np.abs(want[~zero])
    assert err.size == 0 or err.max() <= rel, (err.max(), np.argmax(err))


def assert_sigma(got, want):
    exact = want < 2.0 ** 53
    np.testing.assert_array_equal(got[exact], want[exact])
    if (~exact).any():
        np.testing.assert_allclose(got[~exact], want[~exact], rtol=1e-12)


def assert_bfs_rows(g, sources, depth, sigma):
    """Row i of (depth, sigma) against the oracle's BFS from sources[i]."""
    import oracle
    assert depth.shape == sigma.shape == (len(sources), g.n)
    for i, s in enumerate(sources):
        d_ora, s_ora = oracle.bfs(g.col_ptr, g.row_idx, int(s))
        np.testing.assert_array_equal(depth[i], d_ora, err_msg=f"source {i} ({s})")
        assert_sigma(sigma[i], s_ora)
