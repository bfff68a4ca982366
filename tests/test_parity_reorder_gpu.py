"""nm_reorder_gpu (Stage-1 codes + stable lexicographic sort and the omega / MBscore counts on
the device, Stage-2 on the host) vs the CPU oracle: the permutation and
every statistic must match bit-exactly (DESIGN.md §3 readings).  The shapes are chosen so that
Stage-1 actually runs (MBscore > 0 needs V > 1 or M > 4: with M = 4 no meta-block can hold more
than four distinct columns)."""
import numpy as np
import pytest

import oracle
from paper_conf_ppopp_chensz0s25_b200 import api, graphs

pytestmark = pytest.mark.gpu

_KEYS = ("omega_init", "omega_final", "mb_init", "mb_final", "outer_iters", "stage1_iters",
         "stage2_passes", "max_pairs_per_primary")


def _check(indptr, indices, V, N, M, **kw):
    p_or, s_or = oracle.reorder(indptr, indices, V, N, M, **kw)
    p_gpu, s_gpu = api.reorder(indptr, indices, V, N, M, device=True, **kw)
    assert np.array_equal(p_or, p_gpu)
    for k in _KEYS:
        assert s_or[k] == s_gpu[k], k
    return s_gpu


def test_f1():
    ip, ic = graphs.fixture_f1()
    assert _check(ip, ic, 1, 2, 4)["omega_final"] == 0


@pytest.mark.parametrize("seed", range(60))
def test_tiny_random_graphs(seed):
    rng = np.random.default_rng(1000 + seed)
    n = int(rng.integers(5, 60))
    m = int(rng.integers(n, n * 4))
    ip, ic = graphs.er_graph(n, min(m, n * (n - 1) // 2), 1000 + seed, self_loops=bool(seed % 3 == 0))
    V, N, M = [(4, 2, 8), (2, 1, 4), (8, 2, 16), (1, 2, 8), (16, 2, 32), (3, 2, 8)][seed % 6]
    _check(ip, ic, V, N, M, gain_rule=seed % 2, keep_best=int(seed % 7 != 0))


def test_isolated_vertices_and_empty_rows():
    # a path on the first 10 vertices, 30 isolated vertices: empty keys sort first-class
    n = 40
    rows = [[] for _ in range(n)]
    for i in range(9):
        rows[i].append(i + 1)
        rows[i + 1].append(i)
    ip = np.zeros(n + 1, np.int64)
    ip[1:] = np.cumsum([len(r) for r in rows])
    ic = np.array([c for r in rows for c in sorted(r)], np.int32)
    _check(ip, ic, 8, 2, 8)


@pytest.mark.parametrize("kind,V,M", [("band", 64, 8), ("pl", 128, 16), ("band", 8, 16), ("pl", 4, 8)])
def test_stage1_shapes(kind, V, M):
    if kind == "pl":
        ip, ic = graphs.lmcl_graph(1500, 12000, 2.1, 1, 0.0, 11, scramble=True)
    else:
        ip, ic = graphs.banded_graph(12000, 8, 12)
    st = _check(ip, ic, V, 2, M, max_outer=2)
    assert st["stage1_iters"] > 0


def test_config1_er_2048_v128():
    ip, ic = graphs.er_graph(2048, 16384, 1)
    st = _check(ip, ic, 128, 2, 16, max_outer=1)
    assert st["stage1_iters"] > 0


def test_errors():
    ip, ic = graphs.er_graph(64, 128, 3)
    with pytest.raises(Exception):
        api.reorder(ip, ic, 1, 2, 64, device=True)   # M > 32
    with pytest.raises(Exception):
        api.reorder(ip, ic, 0, 2, 4, device=True)    # V < 1


def test_larger_banded_many_panels():
    # 512 panels of 64 rows, 22 Stage-1 sorts over 0.5M stored entries
    ip, ic = graphs.banded_graph(32768, 16, 23)
    st = _check(ip, ic, 64, 2, 8, max_outer=1)
    assert st["stage1_iters"] > 0 and st["mb_final"] < st["mb_init"]
