"""The row-partitioned multi-GPU path with the REAL per-rank compute (libnm), two ranks
sharing cuda:0 over the gloo backend (this environment has one GPU; the product collective
is NCCL, one rank per GPU):

* dist.gcn_forward with nm_pack_rows + nm_gcn_layer per rank: the world-2 output equals the
  world-1 output BITWISE (row shards change no arithmetic), for equal and
  cost-balanced shards, and matches the oracle's fp64 GCN within the GCN bound;
* bench.py under torch.distributed.run with NM_DIST_BACKEND=gloo, 2 ranks: one JSON line with
  n_gpus = 2 and a positive value.
"""
import json
import os
import socket
import subprocess
import sys

import numpy as np
import pytest

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _problem():
    from paper_conf_ppopp_chensz0s25_b200 import graphs
    n = 3000  # 24 panels, ragged tail (3000 % 128 = 56)
    ip, ic = graphs.lmcl_graph(n, 40000, 2.3, 4, 0.6, 17, self_loops=True)
    vals = graphs.gcn_norm_values(ip, ic)
    rng = np.random.default_rng(1)
    H = rng.standard_normal((n, 64)).astype(np.float32)
    Ws = [(rng.standard_normal((64, 64)) / 8).astype(np.float32), (rng.standard_normal((64, 32)) / 8).astype(np.float32)]
    bs = [(rng.standard_normal(64) * 0.1).astype(np.float32), (rng.standard_normal(32) * 0.1).astype(np.float32)]
    return ip, ic, vals, H, Ws, bs


def _run(world, rank, balanced):
    """GCN forward (2 layers, bf16, 1:2:4) for this rank; returns the full output (bf16 bits)."""
    from paper_conf_ppopp_chensz0s25_b200 import api, graphs
    from paper_conf_ppopp_chensz0s25_b200 import dist as nmdist
    dev = torch.device("cuda:0")
    ip, ic, vals, H, Ws, bs = _problem()
    n = len(ip) - 1
    perm = np.random.default_rng(3).permutation(n).astype(np.int32)
    bounds = (nmdist.balanced_bounds(nmdist.panel_costs(ip, perm), n, world) if balanced
              else [nmdist.shard_rows(n, world, r) for r in range(world)])
    rb, re = bounds[rank]
    P = api.pack(ip, ic, perm, 1, 2, 4, dtype="bf16", val=vals, row_begin=rb, row_end=re)

    def bf(a):
        b, _ = graphs.round16(np.asarray(a, np.float32), "bf16")
        return torch.from_numpy(b.view(np.int16)).to(dev).view(torch.bfloat16)

    layers = [(bf(W), torch.from_numpy(b).to(dev), relu) for W, b, relu in ((Ws[0], bs[0], True), (Ws[1], bs[1], False))]

    def local_layer(li, Hf, W, b, relu, a, z):
        Hd = Hf.view(torch.int16).to(dev).view(torch.bfloat16)
        out = torch.empty((z - a, W.shape[1]), dtype=torch.bfloat16, device=dev)
        ws = torch.empty(api.gcn_workspace_bytes(n, W.shape[0], W.shape[1]), dtype=torch.uint8, device=dev)
        api.gcn_layer(P, Hd, W, b, out, ws, relu=relu, order="linear")
        torch.cuda.synchronize()
        # gloo collectives run on host tensors and have no 16-bit types: ship the bf16 bits as
        # int32 pairs (F is even), bit-exact
        return out.view(torch.int16).cpu().view(torch.int32)

    Hp = bf(H[perm]).view(torch.int16).cpu().view(torch.int32)
    out = nmdist.gcn_forward(Hp, layers, local_layer, bounds=bounds)
    return out.view(torch.int16).numpy().copy(), perm


def _worker(rank, world, port, balanced, q):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    out, _ = _run(world, rank, balanced)
    q.put((rank, out))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("balanced", [False, True])
def test_gcn_forward_world2_bitwise_equals_world1(balanced):
    import torch.multiprocessing as mp

    import oracle
    from paper_conf_ppopp_chensz0s25_b200 import graphs
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    ref, perm = _run(1, 0, balanced)
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, balanced, q)) for r in range(2)]
    for p in procs:
        p.start()
    got = dict(q.get(timeout=300) for _ in range(2))
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    for r in range(2):
        assert np.array_equal(got[r], ref), "rank %d differs from the 1-rank result" % r
    # and the 1-rank result is a correct GCN (fp64 oracle on the same bf16-rounded inputs;
    # loose Frobenius bound: two bf16 layers)
    ip, ic, vals, H, Ws, bs = _problem()
    _, v64 = graphs.round16(vals, "bf16")
    h = graphs.round16(H, "bf16")[1]
    for W, b, relu in ((Ws[0], bs[0], True), (Ws[1], bs[1], False)):
        h, _ = oracle.gcn_layer(ip, ic, v64, h, graphs.round16(W, "bf16")[1], b, relu)
    y = np.empty_like(h)
    y[perm] = graphs.bf16_bits_to_f64(ref.view(np.uint16))
    assert np.linalg.norm(y - h) <= 2e-2 * np.linalg.norm(h)


def test_bench_two_ranks_gloo_on_one_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    env = dict(os.environ, NM_DIST_BACKEND="gloo")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
           "--master-addr", "127.0.0.1", "--master-port", str(_free_port()), os.path.join(ROOT, "bench.py"),
           "--gpus", "2", "--steps", "5", "--warmup", "3", "--workload", "c1-er-n2048-f32-1:2:4"]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=900, env=env, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, r.stdout[-2000:]
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["value"] > 0 and d["steps"] == 5


def test_gcn_layer_bcast_stores_into_every_destination():
    """nm_gcn_layer_bcast (the all-gather fused into the layer's last kernel): each of three
    destination buffers receives exactly nm_gcn_layer's rows at dst_row0, bitwise, and no other
    row is touched (one GPU: the destinations stand for the ranks' peer-mapped buffers)."""
    from paper_conf_ppopp_chensz0s25_b200 import api, graphs
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    dev = torch.device("cuda:0")
    ip, ic, vals, H, Ws, bs = _problem()
    n = len(ip) - 1
    perm = np.random.default_rng(3).permutation(n).astype(np.int32)
    rb, re = 1024, 2304
    P = api.pack(ip, ic, perm, 1, 2, 4, dtype="bf16", val=vals, row_begin=rb, row_end=re)
    Hd = torch.from_numpy(graphs.round16(H, "bf16")[0].view(np.int16)).to(dev).view(torch.bfloat16)
    W = torch.from_numpy(graphs.round16(Ws[0], "bf16")[0].view(np.int16)).to(dev).view(torch.bfloat16)
    b = torch.from_numpy(bs[0]).to(dev)
    ws = torch.empty(api.gcn_workspace_bytes(n, 64, 64), dtype=torch.uint8, device=dev)
    ref = torch.empty((re - rb, 64), dtype=torch.bfloat16, device=dev)
    api.gcn_layer(P, Hd, W, b, ref, ws, relu=True)
    sentinel = -12345
    dsts = [torch.full((4000, 64), sentinel, dtype=torch.int16, device=dev) for _ in range(3)]
    for order in ("linear", "aggregate"):
        api.gcn_layer(P, Hd, W, b, ref, ws, relu=True, order=order)
        api.gcn_layer_bcast(P, Hd, W, b, [d.data_ptr() for d in dsts], 700, 64, ws, relu=True, order=order)
        torch.cuda.synchronize()
        for d in dsts:
            assert torch.equal(d[700:700 + re - rb], ref.view(torch.int16))
            assert bool((d[:700] == sentinel).all()) and bool((d[700 + re - rb:] == sentinel).all())


def test_gcn_forward_fused_world1_equals_collective_forward():
    """dist.gcn_forward_fused with the real layer (nm_gcn_layer_bcast) and a local buffer at
    world 1 returns exactly dist.gcn_forward's output."""
    from paper_conf_ppopp_chensz0s25_b200 import api, graphs
    from paper_conf_ppopp_chensz0s25_b200 import dist as nmdist
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    dev = torch.device("cuda:0")
    ip, ic, vals, H, Ws, bs = _problem()
    n = len(ip) - 1
    perm = np.random.default_rng(3).permutation(n).astype(np.int32)
    P = api.pack(ip, ic, perm, 1, 2, 4, dtype="bf16", val=vals)

    def bf(a):
        return torch.from_numpy(graphs.round16(np.asarray(a, np.float32), "bf16")[0].view(np.int16)).to(dev).view(
            torch.bfloat16)

    layers = [(bf(W), torch.from_numpy(b).to(dev), relu) for W, b, relu in ((Ws[0], bs[0], True), (Ws[1], bs[1], False))]
    ws = torch.empty(api.gcn_workspace_bytes(n, 64, 64), dtype=torch.uint8, device=dev)

    def local_layer(li, Hf, W, b, relu, a, z):
        out = torch.empty((z - a, W.shape[1]), dtype=torch.bfloat16, device=dev)
        api.gcn_layer(P, Hf, W, b, out, ws, relu=relu)
        return out

    def local_layer_bcast(li, Hf, W, b, relu, a, z, ptrs, row0):
        api.gcn_layer_bcast(P, Hf, W, b, ptrs, row0, W.shape[1], ws, relu=relu)

    ref = nmdist.gcn_forward(bf(H), layers, local_layer)
    got = nmdist.gcn_forward_fused(bf(H), layers, local_layer_bcast, nmdist.LocalBuffers())
    torch.cuda.synchronize()
    assert torch.equal(ref.view(torch.int16), got.view(torch.int16))
