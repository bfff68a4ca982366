"""Host-side logic of the row-partitioned multi-GPU path: shard boundaries and
the all-gather assembly of paper_conf_ppopp_chensz0s25_b200.dist.gcn_forward, run with the
gloo backend on CPU, world_size 2 (the per-rank SpMM is stood in by the oracle here, so the
collective/sharding logic is what is tested)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_ppopp_chensz0s25_b200 import dist as nmdist
from paper_conf_ppopp_chensz0s25_b200 import graphs


@pytest.mark.parametrize("n", [1, 127, 128, 129, 1000, 2048, 5000])
@pytest.mark.parametrize("world", [1, 2, 3, 4, 8])
def test_shard_rows_partition(n, world):
    cuts = [nmdist.shard_rows(n, world, r) for r in range(world)]
    assert cuts[0][0] == 0 and cuts[-1][1] == n
    for (a, b), (c, d) in zip(cuts[:-1], cuts[1:]):
        assert b == c
    for a, b in cuts:
        assert (a % 128 == 0 or a == n) and a <= b  # empty trailing shards start at n
        assert b - a <= nmdist.padded_rows(n, world)


@pytest.mark.parametrize("world", [1, 2, 3, 4, 8])
@pytest.mark.parametrize("seed", [0, 1])
def test_balanced_bounds_partition_and_balance(world, seed):
    """Cost-balanced shards: a contiguous panel-aligned partition of all rows,
    and no rank exceeds the ideal share by more than one panel's cost -- on a power-law graph
    where equal-row shards are clearly unbalanced."""
    n = 5000
    ip, ic = graphs.lmcl_graph(n, 30000, 2.1, 1, 0.0, seed, scramble=False)
    perm = np.arange(n, dtype=np.int32)
    costs = nmdist.panel_costs(ip, perm)
    assert costs.shape[0] == (n + 127) // 128
    assert costs.sum() == pytest.approx(ip[-1] + 8.0 * n)
    bounds = nmdist.balanced_bounds(costs, n, world)
    assert bounds[0][0] == 0 and bounds[-1][1] == n
    for (a, b), (c, d) in zip(bounds[:-1], bounds[1:]):
        assert b == c
    for a, b in bounds:
        assert a <= b and (a % 128 == 0 or a == n)
    share = [costs[a // 128:(b + 127) // 128].sum() for a, b in bounds]
    assert max(share) <= costs.sum() / world + costs.max() + 1e-9
    if world > 1:
        eq = [costs[a // 128:(b + 127) // 128].sum() for a, b in (nmdist.shard_rows(n, world, r) for r in range(world))]
        assert max(share) <= max(eq) + 1e-9


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _problem():
    n, f0, f1, f2 = 700, 16, 12, 8
    ip, ic = graphs.er_graph(n, 3000, 5, self_loops=True)
    vals = graphs.symmetric_values(ip, ic, 6).astype(np.float64)
    rng = np.random.default_rng(0)
    H = rng.standard_normal((n, f0))
    Ws = [rng.standard_normal((f0, f1)), rng.standard_normal((f1, f2))]
    bs = [rng.standard_normal(f1), rng.standard_normal(f2)]
    return ip, ic, vals, H, Ws, bs


def _local_layer_factory(ip, ic, vals):
    import oracle

    def local_layer(l, Hf, W, b, relu, rb, re):
        XW = Hf.numpy() @ W
        sub_ip = ip[rb:re + 1] - ip[rb]
        Y, _, _ = oracle.spmm(sub_ip, ic[ip[rb]:ip[re]], vals[ip[rb]:ip[re]], XW)
        Y = Y + b
        if relu:
            Y = np.maximum(Y, 0.0)
        return torch.from_numpy(Y)

    return local_layer


def _bounds(ip, world, balanced):
    if not balanced:
        return None
    n = len(ip) - 1
    return nmdist.balanced_bounds(nmdist.panel_costs(ip, np.arange(n)), n, world)


def _worker(rank, world, port, q, balanced=False):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    ip, ic, vals, H, Ws, bs = _problem()
    layers = [(Ws[0], bs[0], True), (Ws[1], bs[1], False)]
    out = nmdist.gcn_forward(torch.from_numpy(H), layers, _local_layer_factory(ip, ic, vals),
                             bounds=_bounds(ip, world, balanced))
    q.put((rank, out.numpy()))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("balanced", [False, True])
def test_gcn_forward_gloo_world2_matches_single_process(balanced):
    ip, ic, vals, H, Ws, bs = _problem()
    layers = [(Ws[0], bs[0], True), (Ws[1], bs[1], False)]
    ref = nmdist.gcn_forward(torch.from_numpy(H), layers, _local_layer_factory(ip, ic, vals)).numpy()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q, balanced)) for r in range(2)]
    for p in procs:
        p.start()
    got = dict(q.get(timeout=120) for _ in range(2))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for r in range(2):
        assert got[r].shape == ref.shape
        np.testing.assert_allclose(got[r], ref, rtol=1e-12, atol=1e-12)


class _EmulatedPeerBuffers:
    """gloo stand-in for dist.SymmetricBuffers: each rank's buffer is local; the destination
    'pointers' are labels, and the fused kernel's stores into every rank's copy are emulated by
    an all-gather of the rows in local_layer_bcast."""

    def __init__(self):
        self.t = {}
        self.barriers = 0

    def alloc(self, key, shape, dtype, device):
        t = torch.full(shape, float("nan"), dtype=dtype, device=device)
        self.t[key] = t
        world = dist.get_world_size() if dist.is_initialized() else 1
        return t, [(key, r) for r in range(world)]

    def barrier(self, key):
        self.barriers += 1
        if dist.is_initialized():
            dist.barrier()


def _local_layer_bcast_factory(ip, ic, vals, bufs):
    layer = _local_layer_factory(ip, ic, vals)

    def local_layer_bcast(l, Hf, W, b, relu, rb, re, dst_ptrs, dst_row0):
        rows = layer(l, Hf, W, b, relu, rb, re)
        key = dst_ptrs[0][0]
        assert [p[1] for p in dst_ptrs] == list(range(len(dst_ptrs)))  # one destination per rank
        full = bufs.t[key]
        world = len(dst_ptrs)
        rows_pad = full.shape[0] // world
        mine = torch.zeros((rows_pad, full.shape[1]), dtype=full.dtype)
        mine[: re - rb] = rows
        parts = [torch.empty_like(mine) for _ in range(world)]
        if world > 1:
            dist.all_gather(parts, mine)
            offs = [None] * world
            dist.all_gather_object(offs, (dst_row0, re - rb))
        else:
            parts, offs = [mine], [(dst_row0, re - rb)]
        for p, (o, k) in zip(parts, offs):
            full[o: o + k] = p[:k]

    return local_layer_bcast


def _worker_fused(rank, world, port, q, balanced=False):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    ip, ic, vals, H, Ws, bs = _problem()
    layers = [(Ws[0], bs[0], True), (Ws[1], bs[1], False), (Ws[1].T @ Ws[1][:, :8] * 0 + np.eye(8), bs[1], True)]
    bufs = _EmulatedPeerBuffers()
    out = nmdist.gcn_forward_fused(torch.from_numpy(H), layers, _local_layer_bcast_factory(ip, ic, vals, bufs),
                                   bufs, bounds=_bounds(ip, world, balanced))
    q.put((rank, out.numpy(), bufs.barriers, sorted(bufs.t)))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("balanced", [False, True])
def test_gcn_forward_fused_gloo_world2_matches_single_process(balanced):
    """gcn_forward_fused (all-gather fused into each layer's last kernel): world 2 = world 1 =
    the collective-based gcn_forward; one barrier per layer; two alternating buffers."""
    ip, ic, vals, H, Ws, bs = _problem()
    layers = [(Ws[0], bs[0], True), (Ws[1], bs[1], False), (Ws[1].T @ Ws[1][:, :8] * 0 + np.eye(8), bs[1], True)]
    ref = nmdist.gcn_forward(torch.from_numpy(H), layers, _local_layer_factory(ip, ic, vals)).numpy()
    b1 = _EmulatedPeerBuffers()
    one = nmdist.gcn_forward_fused(torch.from_numpy(H), layers, _local_layer_bcast_factory(ip, ic, vals, b1), b1)
    np.testing.assert_allclose(one.numpy(), ref, rtol=1e-12, atol=1e-12)
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker_fused, args=(r, 2, port, q, balanced)) for r in range(2)]
    for p in procs:
        p.start()
    got = {}
    for _ in range(2):
        r, out, nbar, keys = q.get(timeout=120)
        got[r] = out
        assert nbar == len(layers)
        assert keys == [(0, 8), (0, 12), (1, 8)]  # layers 0 and 2 share parity 0 only per width
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for r in range(2):
        np.testing.assert_allclose(got[r], ref, rtol=1e-12, atol=1e-12)
