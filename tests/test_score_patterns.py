"""nm_score_patterns: per candidate V:2:M the score, chunk count and
residual size equal those of an explicit nm_reorder_gpu + nm_pack_auto for F,
the best index is the lowest score (ties: earlier), and its permutation is returned."""
import numpy as np
import pytest

from paper_conf_ppopp_chensz0s25_b200 import api, graphs

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")


@pytest.mark.parametrize("kind", ["band", "pl"])
def test_scores_match_explicit_packs(kind):
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    if kind == "band":
        ip, ic = graphs.banded_graph(3000, 12, 3)
    else:
        ip, ic = graphs.lmcl_graph(3000, 24000, 2.1, 1, 0.0, 4, scramble=True)
    vals = graphs.symmetric_values(ip, ic, 5)
    F = 128
    cands = [(1, 4), (64, 8), (128, 16), (1, 8)]
    best, perm, rows = api.score_patterns(ip, ic, cands, F, dtype="bf16", val=vals, max_outer=2)
    scores = []
    for (V, M), r in zip(cands, rows):
        p, _ = api.reorder(ip, ic, V, 2, M, device=True, max_outer=2)
        P = api.pack(ip, ic, p, V, 2, M, dtype="bf16", val=vals, tau="auto", F=F)
        st = P.stats()
        assert r["n_chunks"] == st["n_chunks"] and r["residual_nnz"] == st["residual_nnz"], (V, M)
        sc = st["n_chunks"] * (0.28 + 0.0075 * F) + st["residual_nnz"] * 0.00016 * F + \
            st["residual_items"] * 0.0024 * F
        assert abs(sc - r["score_ns"]) <= 1e-9 * max(1.0, sc)
        scores.append(sc)
        if (V, M) == cands[best]:
            assert np.array_equal(p, perm)
    assert best == int(np.argmin(scores))


def test_pack_auto_picks_the_model_minimum():
    """nm_pack_auto returns the pack whose tau minimises the time model over its candidates:
    no candidate tau packs to a lower model time (ties: the smaller tau)."""
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    F = 128
    for ip, ic in (graphs.banded_graph(4000, 16, 3), graphs.lmcl_graph(4000, 40000, 2.3, 4, 0.6, 9)):
        perm = np.arange(len(ip) - 1, dtype=np.int32)
        P = api.pack(ip, ic, perm, 1, 2, 4, tau="auto", F=F)

        def model(st):
            return st["n_chunks"] * (0.28 + 0.0075 * F) + st["residual_nnz"] * 0.00016 * F + \
                st["residual_items"] * 0.0024 * F

        best = model(P.stats())
        tm = api.hybrid_tau(F)
        for tau in sorted({0, 2, 4, tm // 2, tm, tm + tm // 2, 2 * tm}):
            Q = api.pack(ip, ic, perm, 1, 2, 4, tau=tau)
            m = model(Q.stats())
            assert best <= m + 1e-9 * max(1.0, m), (tau, best, m)
            if tau < P.tau:
                assert m > best
