"""Multi-GPU level loop.

The paper's backend runs Algorithm 1 and submits every gate of `C - finished` as an independent job
(P:198-203); its only communication is shipping 2.46 KB ciphertexts.  On one 8xB200 box
the same structure becomes: every rank holds the keys (P:239's broadcast, done once at load) and the whole wire
array; each level's gates are split into R contiguous chunks, rank r evaluates chunk r, and one in-place
all-gather over NCCL/NVLink completes the level's output rows on every rank before the next level starts --
or, fused, the key-switch kernels store each output row straight into every rank's wire array over NVLink
(peer memory) and the level ends with a barrier.
Output bytes are independent of R (integer-exact kernels), so the result is byte-identical for R = 1..8.
"""
from __future__ import annotations


def shard(n_gates: int, world: int, rank: int):
    """(g0, g1, chunk): rank's contiguous gate range of a level and the padded chunk size."""
    chunk = -(-n_gates // world) if n_gates else 0
    g0 = min(rank * chunk, n_gates)
    g1 = min((rank + 1) * chunk, n_gates)
    return g0, g1, chunk


def slack_rows(levels, n_rows: int, world: int) -> int:
    """Rows past n_rows that the padded all-gather of some level may touch."""
    need = 0
    for row0, ng in levels:
        _, _, chunk = shard(ng, world, 0)
        need = max(need, row0 + world * chunk - n_rows)
    return need


def barrier(group, device=None):
    """Stream-ordered barrier across ranks: with NCCL a one-element all-reduce on the current stream (every
    rank's earlier kernels on that stream are done before any rank passes it); otherwise synchronise the
    device and take the backend's barrier."""
    import torch
    import torch.distributed as dist
    if dist.get_backend(group) == "nccl":
        dist.all_reduce(torch.zeros(1, device=device), group=group)
    else:
        if device is not None and torch.device(device).type == "cuda":
            torch.cuda.synchronize(device)
        dist.barrier(group=group)


def level_loop(levels, wires, run_level, group=None, fused=False, early=None):
    """levels: [(row0, n_gates)] for levels 1..L; run_level(level, g0, g1) evaluates a gate range of a level
    into `wires` (a [rows, stride] tensor).  With a process group of R > 1 ranks every level's output rows must
    reach all ranks before the next level: fused=True means run_level's kernels already stored them into every
    rank's array (fused all-gather), so only a barrier is taken; otherwise they are all-gathered in place.

    early: per level, how many gates at the start of this rank's chunk read only rows that are
    already local once this rank has run its own part of the previous level (a netlist planned for R ranks,
    tb_set_plan_world).  Those gates run before the previous level's exchange, so the exchange and its barrier
    overlap this rank's next work:  run the rest of level L, run the early part of level L + 1, exchange L."""
    import torch.distributed as dist
    R = dist.get_world_size(group) if group is not None else 1
    r = dist.get_rank(group) if group is not None else 0
    nL = len(levels)
    if not fused:
        # the padded all-gather of level L writes R * chunk rows, i.e. also the first rows of level L + 1: gates of
        # level L + 1 evaluated before it would be overwritten.  Early start needs the fused exchange.
        early = None
    for L, (row0, ng) in enumerate(levels, start=1):
        g0, g1, chunk = shard(ng, R, r)
        if R > 1 and not fused and row0 + R * chunk > wires.shape[0]:
            raise ValueError("wire array needs slack rows for the padded all-gather (see slack_rows)")
        # level 1 reads only inputs; later levels: their early part already ran before the previous exchange
        start = g0 if (early is None or L == 1) else min(g0 + int(early[L - 1]), g1)
        if g1 > start:
            run_level(L, start, g1)
        if early is not None and L < nL:                    # the next level's locally ready gates, before exchange L
            ra, rb, _ = shard(levels[L][1], R, r)
            e = min(int(early[L]), rb - ra)
            if e > 0:
                run_level(L + 1, ra, ra + e)
        if R > 1 and chunk:
            if fused:
                barrier(group, wires.device)
            else:
                dist.all_gather_into_tensor(wires[row0:row0 + R * chunk],
                                            wires[row0 + r * chunk:row0 + (r + 1) * chunk], group=group)
