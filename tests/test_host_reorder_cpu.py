"""The host nm_reorder (libnm, C ABI, no GPU needed) vs the CPU oracle on small graphs, in the
CPU suite: Stage-2's parallel gain tables and lazy priority-list walk must leave the
permutation bit-identical (DESIGN.md §3 readings 12-18).  The full reorder parity suite is
tests/test_parity_reorder.py."""
import numpy as np
import pytest

import oracle
from paper_conf_ppopp_chensz0s25_b200 import api, graphs

_KEYS = ("omega_init", "omega_final", "mb_init", "mb_final", "outer_iters", "stage1_iters",
         "stage2_passes", "max_pairs_per_primary")


def _check(ip, ic, V, N, M, **kw):
    p_or, s_or = oracle.reorder(ip, ic, V, N, M, **kw)
    p_h, s_h = api.reorder(ip, ic, V, N, M, **kw)
    assert np.array_equal(p_or, p_h)
    for k in _KEYS:
        assert s_or[k] == s_h[k], k


@pytest.mark.parametrize("seed", range(24))
def test_host_reorder_tiny(seed):
    rng = np.random.default_rng(5000 + seed)
    n = int(rng.integers(8, 80))
    m = int(rng.integers(n, n * 4))
    ip, ic = graphs.er_graph(n, min(m, n * (n - 1) // 2), 5000 + seed, self_loops=bool(seed % 3 == 0))
    V, N, M = [(1, 2, 4), (1, 2, 8), (4, 2, 8), (2, 1, 4), (8, 2, 16), (1, 2, 16)][seed % 6]
    _check(ip, ic, V, N, M, gain_rule=seed % 2, keep_best=int(seed % 5 != 0))


def test_host_reorder_many_violating_segments():
    # a power-law graph with many violating segments: long priority lists, batched tables
    ip, ic = graphs.lmcl_graph(1200, 9000, 2.1, 1, 0.0, 17, scramble=True)
    _check(ip, ic, 1, 2, 8, max_outer=2)
