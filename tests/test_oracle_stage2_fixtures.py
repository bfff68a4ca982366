"""Hand-derived pins for the oracle's Stage-2 (Alg. 3 lines 8-22, PAPER.md file
lines 442-480; details (i)-(v) at lines 398-413).

Each fixture under tests/golden/s2_fixture_*.txt writes out, step by step, one Stage-2 pass
on a 12-vertex graph: the PScore list, the priority order, the gain tables consulted and the
pairs recorded.  The test checks
  * the fixture's own arithmetic against brute force that shares nothing with the oracle
    (PScore by counting dense segment vectors; every listed gain by actually swapping the two
    positions, rebuilding P A P^T and recounting the two segments' violations);
  * that the oracle records exactly the hand-derived pairs, in order (``stage2_trace``), and
    lands on the hand-derived order after applying them together (lines 24-27).
Fixtures A and B exercise the |I| > 1 branch, C and D the single-entry branch (line 6).
Together they kill the plausible misreadings of Alg. 3: an ascending priority list, a
wrong-signed or missing target estimate update / removal (lines 17-19), a missing primary
break on est <= 0 (lines 20-22), freshtop ties resolved to the last pair, the densest instead
of the sparsest target, no stop on est <= 0 and non-beneficial swaps in the single-entry
branch.
"""
import os

import numpy as np
import pytest

import oracle
from paper_conf_ppopp_chensz0s25_b200 import graphs

GOLD = os.path.join(os.path.dirname(__file__), "golden")
FIXTURES = ["s2_fixture_a.txt", "s2_fixture_b.txt", "s2_fixture_c.txt", "s2_fixture_d.txt"]


def _load(name):
    d = {"gain": [], "trace": []}
    for line in open(os.path.join(GOLD, name)):
        if line.startswith("#") or not line.strip():
            continue
        k, *v = line.split()
        if k in ("gain", "trace"):
            d[k].append(tuple(int(x) for x in v))
        elif k == "edges":
            d[k] = [tuple(int(x) for x in e.split("-")) for e in v]
        else:
            d[k] = [int(x) for x in v]
    return d


def _graph(d):
    n = d["n"][0]
    a = np.array([e[0] for e in d["edges"]], np.int64)
    b = np.array([e[1] for e in d["edges"]], np.int64)
    return n, graphs._symmetric_csr(n, a, b)


def _dense(n, edges, perm):
    A = np.zeros((n, n), np.int64)
    for x, y in edges:
        A[x, y] = A[y, x] = 1
    return A[np.ix_(perm, perm)]


def _pscore_brute(B, N, M):
    n = B.shape[0]
    return [int(sum(B[i, s * M:(s + 1) * M].sum() > N for i in range(n))) for s in range(n // M)]


@pytest.mark.parametrize("name", FIXTURES)
def test_fixture_arithmetic_by_brute_force(name):
    d = _load(name)
    n, M, N = d["n"][0], d["M"][0], d["N"][0]
    ident = np.arange(n)
    ps = _pscore_brute(_dense(n, d["edges"], ident), N, M)
    assert ps == d["pscore"]
    order = sorted((s for s in range(len(ps)) if ps[s] > 0), key=lambda s: (-ps[s], s))
    assert order == d["priority"]
    if "sparsest" in d:  # single-entry branch: the target is the sparsest other segment
        A = _dense(n, d["edges"], ident)
        nnz = [int(A[:, s * M:(s + 1) * M].sum()) for s in range(len(ps))]
        others = [s for s in range(len(ps)) if s != order[0]]
        assert min(others, key=lambda s: (nnz[s], s)) == d["sparsest"][0]
    for p, t, u, v, gp, gt in d["gain"]:
        perm = ident.copy()
        perm[u], perm[v] = v, u
        q = _pscore_brute(_dense(n, d["edges"], perm), N, M)
        assert (ps[p] - q[p], ps[t] - q[t]) == (gp, gt), (p, t, u, v)


@pytest.mark.parametrize("name", FIXTURES)
def test_oracle_stage2_pass_matches_hand_derivation(name):
    d = _load(name)
    n, (ip, ic) = _graph(d)
    for rule in d["rules"]:
        got = oracle.stage2_trace(ip, ic, np.arange(n), d["N"][0], d["M"][0], gain_rule=rule)
        assert got == d["trace"], (rule, got)


@pytest.mark.parametrize("name", FIXTURES)
def test_oracle_applies_the_recorded_pairs_together(name):
    d = _load(name)
    n, (ip, ic) = _graph(d)
    expect = np.arange(n)
    for _, _, u, v in d["trace"]:
        expect[u], expect[v] = expect[v], expect[u]
    if "perm_after_pass" in d:
        assert expect.tolist() == d["perm_after_pass"]
    # Alg. 1 with one outer iteration, one Stage-2 pass, no keep-best: exactly this pass
    perm, st = oracle.reorder(ip, ic, 1, d["N"][0], d["M"][0], max_outer=0, max_stage2=0, keep_best=0)
    assert perm.tolist() == expect.tolist()
    assert st["stage2_passes"] == 1
