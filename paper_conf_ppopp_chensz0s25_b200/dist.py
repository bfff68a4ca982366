"""Row-partitioned multi-GPU driver (§4.4 L426 parallel GNNs where
"each node conducts the multiplications involving a portion of the adjacency matrix").

* ``shard_rows``: contiguous, panel-aligned (128-row) blocks of B = P A P^T, one per rank,
  equal panel counts (the last rank takes the remainder).
* ``balanced_bounds`` / ``panel_costs``: contiguous, panel-aligned blocks
  whose summed per-panel cost (stored entries of the panel's rows + a per-row term for the
  Y writes) is as equal as the panel granularity allows -- power-law rows make equal-row
  shards unequal in work.
* ``gcn_forward``: a K-layer GCN forward (Eq. 1) in the permuted vertex order with
  X replicated: per layer each rank computes its row block of Ahat (H W) with libnm
  (nm_gcn_layer) and the next layer's full operand is assembled with one NCCL
  ``all_gather_into_tensor`` over NVLink (in place: each rank's block of the receive buffer
  is its send buffer).  Shards are padded to equal row counts so the collective needs no
  reshuffle; with equal shards the padding sits at the end and the gathered buffer is used
  as is, otherwise the padding rows are dropped after the gather.
* ``gcn_forward_fused``: the same forward with the all-gather fused into each layer's last
  kernel (``nm_gcn_layer_bcast``): every rank stores its rows straight into all ranks'
  peer-mapped buffers (torch symmetric memory over NVLink), then one barrier per layer.
* ``local_layer`` / ``local_layer_bcast`` and the buffer provider are injectable so the host-
  side logic (sharding, padding, offsets, buffer alternation) is testable with the ``gloo``
  backend on CPU (tests/test_dist.py).
"""
from __future__ import annotations

PANEL = 128


def shard_rows(n: int, world: int, rank: int, panel: int = PANEL):
    """[row_begin, row_end) of rank's block: panel-aligned, equal panel counts."""
    P = (n + panel - 1) // panel
    per = (P + world - 1) // world
    rb = min(n, rank * per * panel)
    re = min(n, (rank + 1) * per * panel)
    return rb, re


def padded_rows(n: int, world: int, panel: int = PANEL) -> int:
    """Rows per rank after padding (the all-gather block size)."""
    P = (n + panel - 1) // panel
    return ((P + world - 1) // world) * panel


def panel_costs(ip, perm, panel: int = PANEL, row_weight: float = 8.0):
    """Per-panel cost of B = P A P^T: sum over the panel's rows p of deg(perm[p]) +
    row_weight (the Y row write, in units of one stored entry).  ip: CSR row pointer of A."""
    import numpy as np
    deg = np.diff(np.asarray(ip, dtype=np.int64))[np.asarray(perm, dtype=np.int64)]
    n = deg.shape[0]
    P = (n + panel - 1) // panel
    pad = np.zeros(P * panel, dtype=np.float64)
    pad[:n] = deg + row_weight
    return pad.reshape(P, panel).sum(axis=1)


def balanced_bounds(costs, n: int, world: int, panel: int = PANEL):
    """[(row_begin, row_end)] per rank: contiguous panel ranges minimising the largest summed
    cost (the linear-partition bottleneck: bisection on the bound, greedy packing decides
    feasibility), so no contiguous panel-aligned split -- equal rows included -- has a smaller
    maximum.  Trailing ranks may be empty."""
    import numpy as np
    costs = np.asarray(costs, dtype=np.float64)
    P = costs.shape[0]

    def pack(T):  # greedy: start a new block when the next panel would exceed T
        cuts, acc = [0], 0.0
        for i, c in enumerate(costs):
            if acc + c > T and acc > 0:
                cuts.append(i)
                acc = 0.0
            acc += c
        return cuts

    lo, hi = (float(costs.max()) if P else 0.0), float(costs.sum())
    for _ in range(64):
        mid = 0.5 * (lo + hi)
        if len(pack(mid)) <= world:
            hi = mid
        else:
            lo = mid
    cuts = pack(hi)
    cuts = cuts + [P] * (world + 1 - len(cuts))
    return [(min(n, a * panel), min(n, b * panel)) for a, b in zip(cuts[:-1], cuts[1:])]


def gcn_forward(H, layers, local_layer, group=None, bounds=None):
    """Multi-layer GCN forward with one all-gather per layer.

    H: full [n x F0] input (permuted order, replicated on every rank).
    layers: list of (W, bias, relu) per layer.
    local_layer(l, H_full, W, bias, relu, rb, re) -> this rank's rows [re-rb x F_out] of
        act(Ahat (H_full W) + bias) for layer l.
    bounds: optional [(row_begin, row_end)] per rank (e.g. balanced_bounds); default equal
        panel counts (shard_rows).  Shards are padded to the largest one for the collective.
    Returns the full [n x F_L] output on every rank.
    """
    import torch
    import torch.distributed as dist

    world = dist.get_world_size(group) if dist.is_initialized() else 1
    rank = dist.get_rank(group) if dist.is_initialized() else 0
    n = H.shape[0]
    if bounds is None:
        bounds = [shard_rows(n, world, r) for r in range(world)]
    assert len(bounds) == world and bounds[0][0] == 0 and bounds[-1][1] == n
    rb, re = bounds[rank]
    rows_pad = max(1, max(b - a for a, b in bounds))
    cur = H
    for li, (W, bias, relu) in enumerate(layers):
        out_loc = local_layer(li, cur, W, bias, relu, rb, re)
        if world == 1:
            cur = out_loc
            continue
        f = out_loc.shape[1]
        full = torch.empty((rows_pad * world, f), dtype=out_loc.dtype, device=out_loc.device)
        mine = full[rank * rows_pad: (rank + 1) * rows_pad]  # in-place all-gather: send = own block
        mine[: re - rb] = out_loc
        if re - rb < rows_pad:
            mine[re - rb:].zero_()
        dist.all_gather_into_tensor(full, mine, group=group)
        if all(b - a == rows_pad for a, b in bounds[:-1]):
            cur = full[:n]  # equal shards: the padding is all at the end, no copy
        else:  # drop each rank's padding rows
            cur = torch.cat([full[r * rows_pad: r * rows_pad + (b - a)] for r, (a, b) in enumerate(bounds)], dim=0)
    return cur


class SymmetricBuffers:
    """Peer-mapped layer buffers for ``gcn_forward_fused`` on one NVLink node: every rank owns
    a [rows_pad * world x F] buffer, allocated with torch's symmetric memory and exchanged
    (rendezvous) so each rank holds the device addresses of all ranks' copies."""

    def __init__(self, group=None):
        self.group = group
        self._h = {}

    def alloc(self, key, shape, dtype, device):
        import torch.distributed as dist
        import torch.distributed._symmetric_memory as symm_mem
        t = symm_mem.empty(shape, dtype=dtype, device=device)
        h = symm_mem.rendezvous(t, self.group if self.group is not None else dist.group.WORLD)
        self._h[key] = h
        return t, list(h.buffer_ptrs)

    def barrier(self, key):
        self._h[key].barrier()


class LocalBuffers:
    """Single-process stand-in for SymmetricBuffers (world = 1): the only destination is the
    local buffer, the barrier is a no-op."""

    def alloc(self, key, shape, dtype, device):
        import torch
        t = torch.empty(shape, dtype=dtype, device=device)
        return t, [t.data_ptr()]

    def barrier(self, key):
        pass


def gcn_forward_fused(H, layers, local_layer_bcast, buffers, group=None, bounds=None):
    """Multi-layer GCN forward with the all-gather FUSED into each layer's last kernel
    (nm_gcn_layer_bcast): rank r stores its output rows [rb, re) straight into rows
    [r * rows_pad, ...) of every rank's copy of the next layer's operand (peer-mapped buffers
    from ``buffers``), then one barrier orders the ranks -- no separate collective and no
    staging copy.  Two buffers alternate between layers: a rank writes layer l + 1's rows into
    peers' buffer (l + 1) % 2 only after the barrier of layer l, i.e. after every rank has
    finished reading it as layer l - 1's output.

    local_layer_bcast(l, H_full, W, bias, relu, rb, re, dst_ptrs, dst_row0) runs the layer on
        this rank's rows and stores them at dst_row0 of every buffer in dst_ptrs.
    Returns the full [n x F_L] output on every rank (a view of the last buffer when the shards
    are equal, else a compacted copy)."""
    import torch
    import torch.distributed as dist

    world = dist.get_world_size(group) if dist.is_initialized() else 1
    rank = dist.get_rank(group) if dist.is_initialized() else 0
    n = H.shape[0]
    if bounds is None:
        bounds = [shard_rows(n, world, r) for r in range(world)]
    assert len(bounds) == world and bounds[0][0] == 0 and bounds[-1][1] == n
    rb, re = bounds[rank]
    rows_pad = max(1, max(b - a for a, b in bounds))
    equal = all(b - a == rows_pad for a, b in bounds[:-1])
    bufs = {}
    cur = H
    for li, (W, bias, relu) in enumerate(layers):
        f = W.shape[1]
        key = (li % 2, f)
        if key not in bufs:
            bufs[key] = buffers.alloc(key, (rows_pad * world, f), H.dtype, H.device)
        full, ptrs = bufs[key]
        local_layer_bcast(li, cur, W, bias, relu, rb, re, ptrs, rank * rows_pad)
        buffers.barrier(key)
        if equal:
            cur = full[:n]
        else:
            cur = torch.cat([full[r * rows_pad: r * rows_pad + (b - a)] for r, (a, b) in enumerate(bounds)], dim=0)
    return cur
