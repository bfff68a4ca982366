"""nm_score_patterns: per candidate V:2:M the score, chunk count and
residual size equal those of an explicit nm_reorder_gpu + nm_pack_hybrid at nm_hybrid_tau(F),
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
    tau = api.hybrid_tau(F)
    scores = []
    for (V, M), r in zip(cands, rows):
        p, _ = api.reorder(ip, ic, V, 2, M, device=True, max_outer=2)
        P = api.pack(ip, ic, p, V, 2, M, dtype="bf16", val=vals, tau=tau)
        st = P.stats()
        assert r["n_chunks"] == st["n_chunks"] and r["residual_nnz"] == st["residual_nnz"], (V, M)
        sc = st["n_chunks"] * (0.28 + 0.0075 * F) + st["residual_nnz"] * 0.00016 * F
        assert abs(sc - r["score_ns"]) <= 1e-9 * max(1.0, sc)
        scores.append(sc)
        if (V, M) == cands[best]:
            assert np.array_equal(p, perm)
    assert best == int(np.argmin(scores))
