"""Row-partitioned multi-GPU driver (§4.4 L426 parallel GNNs where
"each node conducts the multiplications involving a portion of the adjacency matrix").

* ``shard_rows``: contiguous, panel-aligned (128-row) blocks of B = P A P^T, one per rank,
  equal panel counts (the last rank takes the remainder).
* ``gcn_forward``: a K-layer GCN forward (Eq. 1) in the permuted vertex order with
  X replicated: per layer each rank computes its row block of Ahat (H W) with libnm
  (nm_gcn_layer) and the next layer's full operand is assembled with one NCCL
  ``all_gather_into_tensor`` over NVLink.  Shards are padded to equal row counts so the
  collective needs no reshuffle; padding rows are dropped after the gather.
* ``local_layer`` is injectable so the host-side logic (sharding, padding, collective order)
  is testable with the ``gloo`` backend on CPU (tests/test_dist.py).
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


def gcn_forward(H, layers, local_layer, group=None):
    """Multi-layer GCN forward with one all-gather per layer.

    H: full [n x F0] input (permuted order, replicated on every rank).
    layers: list of (W, bias, relu) per layer.
    local_layer(l, H_full, W, bias, relu, rb, re) -> this rank's rows [re-rb x F_out] of
        act(Ahat (H_full W) + bias) for layer l.
    Returns the full [n x F_L] output on every rank.
    """
    import torch
    import torch.distributed as dist

    world = dist.get_world_size(group) if dist.is_initialized() else 1
    rank = dist.get_rank(group) if dist.is_initialized() else 0
    n = H.shape[0]
    rb, re = shard_rows(n, world, rank)
    rows_pad = padded_rows(n, world)
    cur = H
    for li, (W, bias, relu) in enumerate(layers):
        out_loc = local_layer(li, cur, W, bias, relu, rb, re)
        if world == 1:
            cur = out_loc
            continue
        f = out_loc.shape[1]
        send = torch.zeros((rows_pad, f), dtype=out_loc.dtype, device=out_loc.device)
        send[: re - rb] = out_loc
        full = torch.empty((rows_pad * world, f), dtype=out_loc.dtype, device=out_loc.device)
        dist.all_gather_into_tensor(full, send, group=group)
        # drop each rank's padding rows
        parts = []
        for r in range(world):
            a, b = shard_rows(n, world, r)
            parts.append(full[r * rows_pad: r * rows_pad + (b - a)])
        cur = torch.cat(parts, dim=0)
    return cur
