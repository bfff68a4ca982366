"""Pins for the oracle's reordering (Alg. 1-3).

The greedy heuristic's exact permutation has no closed form ("parity unpinned" beyond these
pins): it is pinned by the Figure-1 fixture's unique answer, by a brute-force
optimum bound on tiny graphs, and by invariants (bijection, keep-best never worse, at most M
recorded pairs per primary -- the paper's complexity argument L562-569).
"""
import itertools
import os

import numpy as np
import pytest

import oracle
from paper_conf_ppopp_chensz0s25_b200 import graphs

from test_oracle_counts import brute_counts, dense_B

GOLD = os.path.join(os.path.dirname(__file__), "golden", "f1_figure1.txt")


def _f1_golden():
    d = {"rows": {}}
    for line in open(GOLD):
        if line.startswith("#") or not line.strip():
            continue
        parts = line.split()
        if parts[0] == "row":
            d["rows"][int(parts[1])] = parts[2:]
        else:
            d[parts[0]] = parts[1:]
    return d


def test_f1_fixture_matches_figure1():
    g = _f1_golden()
    indptr, indices = graphs.fixture_f1()
    edges = sorted(tuple(map(int, e.split("-"))) for e in g["edges"])
    got = sorted((i, int(j)) for i in range(8) for j in indices[indptr[i]:indptr[i + 1]] if i < j)
    assert got == edges
    w, mb, _ = oracle.counts(indptr, indices, np.arange(8), 1, 2, 4)
    assert w == int(g["omega_init"][0]) and mb == 0
    # row 6 is the only violating segment vector (Figure 1 caption, L38)
    B = dense_B(indptr, indices, np.arange(8))
    assert [i for i in range(8) if B[i, 0:4].sum() > 2 or B[i, 4:8].sum() > 2] == [6]


def test_f1_swap_3_4_is_the_unique_fixing_cross_swap():
    indptr, indices = graphs.fixture_f1()
    fixing = []
    for u in range(4):
        for v in range(4, 8):
            perm = np.arange(8)
            perm[u], perm[v] = perm[v], perm[u]
            w, _, _ = brute_counts(dense_B(indptr, indices, perm), 1, 2, 4)
            if w == 0:
                fixing.append((u, v))
    assert fixing == [(3, 4)]


@pytest.mark.parametrize("gain_rule", [0, 1])
def test_f1_reorder(gain_rule):
    g = _f1_golden()
    indptr, indices = graphs.fixture_f1()
    perm, st = oracle.reorder(indptr, indices, 1, 2, 4, gain_rule=gain_rule)
    assert list(perm) == [int(x) for x in g["perm_after"]]
    assert st["omega_init"] == 1 and st["omega_final"] == int(g["omega_final"][0])


def _partitions(items, size):
    """All partitions of items into consecutive blocks of `size` (unordered blocks)."""
    if not items:
        yield []
        return
    first, rest = items[0], items[1:]
    for comb in itertools.combinations(rest, min(size, len(items)) - 1):
        block = (first,) + comb
        remaining = [x for x in rest if x not in comb]
        for tail in _partitions(remaining, size):
            yield [block] + tail


def _brute_min_omega(indptr, indices, M, N):
    n = len(indptr) - 1
    best = None
    for part in _partitions(list(range(n)), M):
        perm = np.array([v for blk in part for v in blk])
        w, _, _ = brute_counts(dense_B(indptr, indices, perm), 1, N, M)
        best = w if best is None else min(best, w)
    return best


@pytest.mark.parametrize("n,m,seed", [(8, 14, 1), (8, 18, 2), (12, 30, 3), (12, 40, 4)])
@pytest.mark.parametrize("gain_rule", [0, 1])
def test_brute_force_optimum_bounds_the_heuristic(n, m, seed, gain_rule):
    indptr, indices = graphs.er_graph(n, m, seed)
    opt = _brute_min_omega(indptr, indices, 4, 2)
    perm, st = oracle.reorder(indptr, indices, 1, 2, 4, gain_rule=gain_rule)
    w, _, _ = brute_counts(dense_B(indptr, indices, perm), 1, 2, 4)
    assert w == st["omega_final"]
    assert opt <= w <= st["omega_init"]


def _cases():
    return [
        ("er", graphs.er_graph(256, 2048, 11)),
        ("pl", graphs.lmcl_graph(300, 2400, 2.1, 1, 0.0, 12, scramble=True)),
        ("band", graphs.banded_graph(256, 8, 13)),
        ("loops", graphs.er_graph(128, 900, 14, self_loops=True)),
    ]


@pytest.mark.parametrize("ci", range(4))
@pytest.mark.parametrize("V,N,M", [(1, 2, 4), (1, 2, 8), (8, 2, 8), (16, 2, 16)])
@pytest.mark.parametrize("gain_rule", [0, 1])
def test_reorder_invariants(ci, V, N, M, gain_rule):
    _, (indptr, indices) = _cases()[ci]
    n = len(indptr) - 1
    perm, st = oracle.reorder(indptr, indices, V, N, M, gain_rule=gain_rule)
    assert sorted(perm.tolist()) == list(range(n))                     # bijection
    w0, mb0, _ = oracle.counts(indptr, indices, np.arange(n), V, N, M)
    w1, mb1, _ = oracle.counts(indptr, indices, perm, V, N, M)
    assert (st["omega_init"], st["mb_init"]) == (w0, mb0)
    assert (st["omega_final"], st["mb_final"]) == (w1, mb1)
    assert w1 + mb1 <= w0 + mb0                                         # keep-best
    assert st["max_pairs_per_primary"] <= M                             # L562-569
    assert st["outer_iters"] <= 11
    # P A P^T keeps the pattern symmetric with the same nnz (L128-142)
    B = dense_B(indptr, indices, perm)
    assert (B == B.T).all() and B.sum() == indptr[-1]


def test_stage1_is_noop_at_v1_m4():
    """k = 4 makes the vertical constraint vacuous for 1x4 meta-blocks (reading #4)."""
    indptr, indices = graphs.er_graph(200, 1500, 21)
    perm, st = oracle.reorder(indptr, indices, 1, 2, 4)
    assert st["mb_init"] == 0 and st["stage1_iters"] == 0


def test_banded_violations_fixed_substantially():
    """Natural-order banded graphs: paper mode removes most 2:4 violations (Table 7 trend)."""
    indptr, indices = graphs.banded_graph(1024, 8, 31)
    perm, st = oracle.reorder(indptr, indices, 1, 2, 4, gain_rule=0)
    assert st["omega_init"] > 0
    assert st["omega_final"] < st["omega_init"]


def test_select_pattern_closed_forms():
    """PAPER.md:L496 search.  Self-loops only: every row has one nonzero (any M conforms) but a
    diagonal V x M block has min(V, M) distinct columns and no permutation moves the diagonal,
    so V stops at 4 (k = 4): expected (V, M) = (4, 32).  No edges at all: (32, 32)."""
    n = 256
    ip = np.arange(n + 1, dtype=np.int64)
    ic = np.arange(n, dtype=np.int32)
    V, M, perm, st = oracle.select_pattern(ip, ic, max_M=32, max_V=32)
    assert (V, M) == (4, 32) and st["omega_final"] == 0 and st["mb_final"] == 0
    ip0 = np.zeros(n + 1, dtype=np.int64)
    V, M, perm, st = oracle.select_pattern(ip0, np.zeros(0, np.int32), max_M=32, max_V=32)
    assert (V, M) == (32, 32)


def test_select_pattern_returns_conforming_or_fallback():
    for seed in range(4):
        ip, ic = graphs.banded_graph(300, 4, 40 + seed)
        V, M, perm, st = oracle.select_pattern(ip, ic, max_M=16, max_V=8)
        w, mb, _ = oracle.counts(ip, ic, perm, V, 2, M)
        assert (w, mb) == (st["omega_final"], st["mb_final"])
        if (V, M) != (1, 4):
            assert w == 0 and mb == 0
