"""Seeded synthetic inputs shared by the CUDA path's tests/bench and the oracle's tests.

This module holds NO arithmetic of the method (no codes, counts, packing or SpMM): it only
draws graphs, values and features with numpy ``default_rng`` so that both sides consume the
same bits.  Shapes follow the paper's workloads (Tables 1-2) as recorded
in DESIGN.md §Inputs:

* ``er_graph``     -- Erdős–Rényi G(n, m), config C1 (n=2048, m=16,384).
* ``lmcl_graph``   -- locality-mixed Chung–Lu (power-law degrees, contiguous communities),
                      C2 power-law (C=1, rho=0, scrambled) and the Reddit / ogbn shapes C3-C5.
* ``banded_graph`` -- banded SuiteSparse-like matrices, C2 banded.
* ``fixture_f1``   -- the Figure-1 reconstruction used as a pin.

All graphs are returned as a symmetric CSR (indptr int64, indices int32 sorted, no
duplicates); self-loops only when asked for.
"""
from __future__ import annotations

import hashlib

import numpy as np


def _csr_from_pairs(n: int, u: np.ndarray, v: np.ndarray):
    """Directed pairs (already both directions, unique) -> CSR with sorted columns."""
    key = np.sort(u.astype(np.int64) * n + v.astype(np.int64))
    u = key // n
    v = key - u * n
    indptr = np.zeros(n + 1, np.int64)
    np.cumsum(np.bincount(u, minlength=n), out=indptr[1:])
    return indptr, v.astype(np.int32)


def _symmetric_csr(n: int, a: np.ndarray, b: np.ndarray, self_loops: bool = False):
    """Undirected unique pairs a<b -> symmetric CSR (optionally + identity)."""
    u = np.concatenate([a, b]).astype(np.int64)
    v = np.concatenate([b, a]).astype(np.int64)
    if self_loops:
        d = np.arange(n, dtype=np.int64)
        u = np.concatenate([u, d])
        v = np.concatenate([v, d])
    return _csr_from_pairs(n, u, v)


def _sorted_unique(x: np.ndarray) -> np.ndarray:
    """np.unique(x) for 1-D int64 (sorted distinct values) via sort + mask: numpy 2.x's
    np.unique/union1d take minutes at the C3-C5 sizes (~10^8 keys), np.sort seconds."""
    s = np.sort(x)
    if s.size == 0:
        return s
    keep = np.empty(s.size, bool)
    keep[0] = True
    np.not_equal(s[1:], s[:-1], out=keep[1:])
    return s[keep]


def _union(a: np.ndarray, b: np.ndarray) -> np.ndarray:
    return _sorted_unique(np.concatenate([a, b]))


def _searchsorted_right(cum: np.ndarray, q: np.ndarray) -> np.ndarray:
    """np.searchsorted(cum, q, side='right') (exact float64 comparisons, identical result);
    torch's CPU kernel is ~10x faster on 10^8 unsorted queries."""
    import torch
    return torch.searchsorted(torch.from_numpy(np.ascontiguousarray(cum)),
                              torch.from_numpy(np.ascontiguousarray(q)), right=True).numpy()


def _unique_pairs(a: np.ndarray, b: np.ndarray, n: int):
    lo = np.minimum(a, b).astype(np.int64)
    hi = np.maximum(a, b).astype(np.int64)
    keep = lo != hi
    key = _sorted_unique(lo[keep] * n + hi[keep])
    return key


def er_graph(n: int, m: int, seed: int, self_loops: bool = False):
    """G(n, m): m distinct undirected edges drawn uniformly, no self-loops (C1)."""
    rng = np.random.default_rng(seed)
    key = np.empty(0, np.int64)
    while key.size < m:
        k = int((m - key.size) * 1.2) + 16
        a = rng.integers(0, n, k)
        b = rng.integers(0, n, k)
        key = _union(key, _unique_pairs(a, b, n))
    key = key[np.sort(rng.permutation(key.size)[:m])]
    return _symmetric_csr(n, key // n, key % n, self_loops)


def lmcl_graph(n: int, m: int, gamma: float, C: int, rho: float, seed: int,
               dcap_frac: float = 0.1, scramble: bool = False, self_loops: bool = False):
    """Locality-mixed Chung–Lu (SURVEY §8(d) generator spec).

    Weights w_i = (1 + rank_i)^(-1/(gamma-1)) with a random rank (hubs spread over the
    communities), capped at dcap_frac*n expected degree; community(i) = floor(i*C/n)
    (contiguous, i.e. natural order has locality).  Each draw picks u ~ w and, with
    probability rho, v ~ w restricted to u's community, else v ~ w globally.  Self-pairs and
    duplicates are dropped; exactly m undirected edges are kept.
    """
    rng = np.random.default_rng(seed)
    rank = rng.permutation(n)
    w = (1.0 + rank) ** (-1.0 / (gamma - 1.0))
    w *= 2.0 * m / w.sum()
    cap = dcap_frac * n
    for _ in range(50):
        over = w > cap
        if not over.any():
            break
        w[over] = cap
        w *= 2.0 * m / w.sum()
    cum = np.concatenate([[0.0], np.cumsum(w)])
    total = cum[-1]
    bounds = (np.arange(C + 1, dtype=np.int64) * n) // C
    comm_of = (np.arange(n, dtype=np.int64) * C) // n
    key = np.empty(0, np.int64)
    while key.size < m:
        k = int((m - key.size) * 1.3) + 1024
        u = _searchsorted_right(cum, rng.random(k) * total) - 1
        u = np.clip(u, 0, n - 1)
        local = rng.random(k) < rho
        cu = comm_of[u]
        lo = cum[bounds[cu]]
        hi = cum[bounds[cu + 1]]
        r = rng.random(k)
        tgt = np.where(local, lo + r * (hi - lo), r * total)
        v = np.clip(_searchsorted_right(cum, tgt) - 1, 0, n - 1)
        key = _union(key, _unique_pairs(u, v, n))
    key = key[np.sort(rng.permutation(key.size)[:m])]
    a, b = key // n, key % n
    if scramble:
        sp = rng.permutation(n)
        a, b = sp[a], sp[b]
        lo_, hi_ = np.minimum(a, b), np.maximum(a, b)
        a, b = lo_, hi_
    return _symmetric_csr(n, a, b, self_loops)


def banded_graph(n: int, d: int, seed: int, self_loops: bool = False):
    """Banded SuiteSparse-like matrix: every vertex i draws d/2 partners i + U{1..4d}
    (natural order), topped up to n*d/2 distinct undirected edges."""
    rng = np.random.default_rng(seed)
    m = n * d // 2
    key = np.empty(0, np.int64)
    while key.size < m:
        k = int((m - key.size) * 1.2) + 1024
        i = rng.integers(0, n, k)
        j = i + rng.integers(1, 4 * d + 1, k)
        ok = j < n
        key = _union(key, _unique_pairs(i[ok], j[ok], n))
    key = key[np.sort(rng.permutation(key.size)[:m])]
    return _symmetric_csr(n, key // n, key % n, self_loops)


def fixture_f1():
    """Figure-1 reconstruction: n = 8, row 6 = {1,2,3,7} is the only 2:4
    violation; swapping vertices 3 and 4 is the unique cross-segment swap reaching omega = 0."""
    edges = [(0, 2), (0, 4), (1, 3), (1, 4), (1, 6), (2, 3), (2, 6), (3, 6), (3, 7), (4, 5),
             (6, 7)]
    a = np.array([e[0] for e in edges], np.int64)
    b = np.array([e[1] for e in edges], np.int64)
    return _symmetric_csr(8, a, b)


def seed_of(*parts) -> int:
    """Stable seed from a tuple of config parts (e.g. ('banded', n, d))."""
    h = hashlib.sha256(repr(parts).encode()).digest()
    return int.from_bytes(h[:4], "little")


# ---------------------------------------------------------------- values and features

def f32_to_bf16_bits(x: np.ndarray) -> np.ndarray:
    """Round-to-nearest-even float32 -> bfloat16 bit pattern (uint16)."""
    b = np.ascontiguousarray(x, np.float32).view(np.uint32).astype(np.uint64)
    lsb = (b >> 16) & 1
    r = ((b + 0x7FFF + lsb) >> 16).astype(np.uint16)
    nan = np.isnan(np.asarray(x, np.float32))
    if nan.any():
        r[nan] = 0x7FC0
    return r


def bf16_bits_to_f64(b: np.ndarray) -> np.ndarray:
    return (np.asarray(b, np.uint16).astype(np.uint32) << 16).view(np.float32).astype(np.float64)


def round16(x: np.ndarray, dtype: str):
    """Round to the 16-bit dtype; returns (bits uint16, value as float64)."""
    if dtype == "f16":
        h = np.asarray(x, np.float32).astype(np.float16)
        return h.view(np.uint16), h.astype(np.float64)
    if dtype == "bf16":
        bits = f32_to_bf16_bits(np.asarray(x, np.float32))
        return bits, bf16_bits_to_f64(bits)
    raise ValueError(dtype)


def symmetric_values(indptr, indices, seed: int, lo: float = 0.25, hi: float = 1.0):
    """One value per undirected edge, |v| in [lo, hi) with a random sign (never +-0), stored
    on both (i,j) and (j,i) -- A stays symmetric in value, not only in pattern."""
    n = len(indptr) - 1
    rows = np.repeat(np.arange(n, dtype=np.uint64), np.diff(indptr))
    cols = indices.astype(np.uint64)
    key = np.minimum(rows, cols) * np.uint64(n) + np.maximum(rows, cols)
    # counter-based: splitmix64(seed, edge key) -> 53-bit uniform + sign bit
    with np.errstate(over="ignore"):
        z = key + np.uint64(seed) * np.uint64(0x9E3779B97F4A7C15) + np.uint64(0x632BE59BD9B4E019)
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        z = z ^ (z >> np.uint64(31))
    u = (z >> np.uint64(11)).astype(np.float64) * (1.0 / (1 << 53))
    sgn = np.where((z & np.uint64(1)) == 1, -1.0, 1.0)
    return ((lo + (hi - lo) * u) * sgn).astype(np.float32)


def uniform_values(nnz: int, seed: int):
    """A values U[-1, 1) per stored entry (C1 recipe)."""
    rng = np.random.default_rng(seed)
    return (rng.random(nnz) * 2.0 - 1.0).astype(np.float32)


def features(n: int, F: int, seed: int, dist: str = "uniform"):
    """Dense node features X [n x F] float32: U[-1,1) or N(0,1)."""
    rng = np.random.default_rng(seed)
    if dist == "uniform":
        return (rng.random((n, F), dtype=np.float32) * 2.0 - 1.0)
    return rng.standard_normal((n, F), dtype=np.float32)


# ---------------------------------------------------------------- GNN-shaped graphs (C3-C5)
# Shapes from the paper's Table 2: n and directed edge counts are the
# datasets'; gamma, community count and rho are assumptions, natural order
# (contiguous communities), self-loops added as GCN's A + I (Eq. 1; reading #22).

GNN_SHAPES = {
    # name: (n, undirected edges m, gamma, communities, rho)
    "reddit": (232_965, 57_400_000, 2.3, 41, 0.6),        # C3: ~114.8M directed (L520)
    "proteins": (132_534, 39_561_252, 3.0, 8, 0.8),       # C4: 79.12M directed (L521)
    "products": (2_449_029, 61_859_140, 2.5, 47, 0.7),    # C5: 123.72M directed (L522)
}


def gnn_graph(name: str, scale: int = 1):
    """Reddit / ogbn-proteins / ogbn-products-shaped graph (C3 / C4 / C5) as a symmetric CSR
    with self-loops.  scale > 1 divides n and m by that factor (test-sized replicas with the
    same average degree, degree-distribution family and community structure)."""
    n, m, gamma, C, rho = GNN_SHAPES[name]
    n, m = n // scale, m // scale
    return lmcl_graph(n, m, gamma, C, rho, seed_of(name, n, m), self_loops=True)


def gcn_norm_values(indptr, indices):
    """Values of Ahat = D^-1/2 (A + I) D^-1/2 (GCN, Eq. 1) for a CSR that
    already holds the self-loops: v_ij = 1/sqrt(d_i d_j), d = row lengths.  float32."""
    n = len(indptr) - 1
    deg = np.diff(indptr).astype(np.float64)
    dinv = np.where(deg > 0, 1.0 / np.sqrt(np.maximum(deg, 1.0)), 0.0)
    rows = np.repeat(np.arange(n), np.diff(indptr))
    return (dinv[rows] * dinv[indices]).astype(np.float32)
