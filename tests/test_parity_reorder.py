"""nm_reorder (libnm, through the C ABI) vs the CPU oracle: the permutation, omega and
MBscore must match bit-exactly.  nm_reorder itself runs on the host, so these
tests also run without a GPU; they are the reorder parity suite."""
import numpy as np
import pytest

import oracle
from paper_conf_ppopp_chensz0s25_b200 import api, graphs

pytestmark = pytest.mark.gpu


def _check(indptr, indices, V, N, M, gain_rule=0, keep_best=1, **kw):
    p_or, s_or = oracle.reorder(indptr, indices, V, N, M, gain_rule=gain_rule, keep_best=keep_best, **kw)
    p_gpu, s_gpu = api.reorder(indptr, indices, V, N, M, gain_rule=gain_rule, keep_best=keep_best, **kw)
    assert np.array_equal(p_or, p_gpu)
    for k in ("omega_init", "omega_final", "mb_init", "mb_final", "outer_iters", "stage1_iters",
              "stage2_passes", "max_pairs_per_primary"):
        assert s_or[k] == s_gpu[k], k
    return s_gpu


def test_f1():
    ip, ic = graphs.fixture_f1()
    st = _check(ip, ic, 1, 2, 4)
    assert st["omega_final"] == 0


@pytest.mark.parametrize("seed", range(200))
def test_tiny_random_graphs(seed):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(5, 40))
    m = int(rng.integers(n, n * 4))
    ip, ic = graphs.er_graph(n, min(m, n * (n - 1) // 2), seed, self_loops=bool(seed % 3 == 0))
    V, N, M = [(1, 2, 4), (1, 2, 8), (4, 2, 8), (2, 1, 4), (8, 2, 16)][seed % 5]
    _check(ip, ic, V, N, M, gain_rule=seed % 2, keep_best=int(seed % 7 != 0))


@pytest.mark.parametrize("gain_rule", [0, 1])
def test_config1_er_2048(gain_rule):
    ip, ic = graphs.er_graph(2048, 16384, 1)
    _check(ip, ic, 1, 2, 4, gain_rule=gain_rule)


@pytest.mark.parametrize("kind,V,M", [("pl", 1, 4), ("band", 1, 4), ("band", 64, 8), ("pl", 128, 16),
                                      ("band", 8, 8)])
def test_sweep_shapes_small(kind, V, M):
    if kind == "pl":
        ip, ic = graphs.lmcl_graph(1500, 12000, 2.1, 1, 0.0, 3, scramble=True)
    else:
        ip, ic = graphs.banded_graph(2000, 8, 4)
    _check(ip, ic, V, 2, M)


def test_literal_mode_and_caps():
    ip, ic = graphs.banded_graph(700, 12, 5)
    _check(ip, ic, 4, 2, 8, keep_best=0, max_outer=2, max_stage1=1, max_stage2=3)


@pytest.mark.parametrize("seed", range(6))
def test_select_pattern_parity(seed):
    if seed % 2:
        ip, ic = graphs.banded_graph(400, 4, 60 + seed)
    else:
        ip, ic = graphs.er_graph(300, 500, 60 + seed)
    Vo, Mo, po, so = oracle.select_pattern(ip, ic, max_M=16, max_V=16)
    Vg, Mg, pg, sg = api.select_pattern(ip, ic, max_M=16, max_V=16)
    assert (Vo, Mo) == (Vg, Mg)
    assert np.array_equal(po, pg)
    assert so["omega_final"] == sg["omega_final"] and so["mb_final"] == sg["mb_final"]


def test_select_pattern_self_loops():
    n = 256
    ip = np.arange(n + 1, dtype=np.int64)
    ic = np.arange(n, dtype=np.int32)
    assert api.select_pattern(ip, ic)[:2] == (4, 32)
