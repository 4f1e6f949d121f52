"""Multi-rank level loop on CPU (gloo, world sizes 2 and 3): sharding of each level, the padded in-place
all-gather of output rows, and the wire layout from the native plan (tb_netlist_plan).  The per-gate work is
a plaintext stand-in (the gate's truth table on bits), so this checks the distributed plumbing that the GPU
path uses unchanged (paper_conf_ispass_maxw23_b200.parallel.level_loop); the kernels are covered by -m gpu.
Expected values come from the oracle's plaintext simulator (oracle/plain.py).
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from oracle.plain import gate_bits, simulate


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _netlist(seed):
    from test_host import random_dag
    return random_dag(seed, n_inputs=7, n_gates=90)


def _worker(rank, world, port, seed, q, shared=None, early_start=False):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import paper_conf_ispass_maxw23_b200 as tb
        from paper_conf_ispass_maxw23_b200 import parallel
        n_in, t, a, b, c = _netlist(seed)
        net = tb.Netlist(n_in, t, a, b, c)
        early = None
        if early_start:
            levels, rows, early_all = net.plan_world(world)
            early = early_all[:, rank].tolist()
        else:
            levels, rows = net.plan()
        lvl_of_row = np.zeros(net.n_wires, np.int64)
        for L, (row0, ng) in enumerate(levels, start=1):
            lvl_of_row[row0:row0 + ng] = L
        passed = [0]                                    # barriers passed = highest level exchanged to every rank
        own = set()
        if early_start:
            real_barrier = parallel.barrier

            def counting_barrier(group, device=None):
                real_barrier(group, device)
                passed[0] += 1
            parallel.barrier = counting_barrier
        order = np.argsort(rows[n_in:])                  # level-sorted position -> original gate index
        bits = np.random.default_rng(seed).integers(0, 2, n_in).astype(np.int32)
        slack = parallel.slack_rows(levels, net.n_wires, world)
        fused = shared is not None                    # every rank's array in shared memory: the "peer" stores
        wires = shared[rank] if fused else torch.full((net.n_wires + slack, 3), -1, dtype=torch.int32)
        wires[:n_in, 0] = torch.from_numpy(bits)
        calls = []

        def run_level(L, g0, g1):
            row0, ng = levels[L - 1]
            calls.append((L, g0, g1))
            for k in range(row0 - n_in + g0, row0 - n_in + g1):
                g = order[k]
                if early_start:                          # every input row must be visible to this rank now:
                    for w in ([a[g], b[g]] if t[g] != 3 else [a[g]]) + ([c[g]] if t[g] == 16 else []):
                        rw = rows[w]                     # a primary input, exchanged, or computed here
                        assert lvl_of_row[rw] <= passed[0] or rw in own, (rank, L, int(rw))
                own.add(n_in + k)
                x = int(wires[rows[a[g]], 0])
                y = int(wires[rows[b[g]], 0]) if t[g] != 3 else 0
                z = int(wires[rows[c[g]], 0]) if t[g] == 16 else 0
                v = int(gate_bits(int(t[g]), x, y, z))
                for dst in (shared if fused else [wires]):  # fused: the row goes to every rank's array
                    dst[n_in + k, 0] = v
                    dst[n_in + k, 1] = rank                # who computed it

        parallel.level_loop(levels, wires, run_level, group=dist.group.WORLD, fused=fused, early=early)
        q.put((rank, wires[:net.n_wires].numpy().copy(), calls, rows))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,seed", [(2, 1), (3, 2), (2, 5)])
def test_level_loop_all_gather_matches_simulation(world, seed):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, seed, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    n_in, t, a, b, c = _netlist(seed)
    bits = np.random.default_rng(seed).integers(0, 2, n_in)
    want = simulate(n_in, t, a, b, c, bits)[0]
    for rank, w, calls, rows in res:
        assert (w[rows, 0] == want).all(), "rank %d wire values differ from the plaintext simulation" % rank
    # every rank holds identical rows after the gathers, and each gate was computed by exactly one rank
    ref = res[0][1]
    for _, w, _, _ in res[1:]:
        assert (w == ref).all()
    owners = ref[n_in:, 1]
    assert set(owners.tolist()) <= set(range(world))
    computed = sorted(k for _, _, calls, _ in res for (L, g0, g1) in calls for k in range(g0, g1) for _ in [L])
    assert len(computed) == len(t)


@pytest.mark.parametrize("world,seed", [(2, 3), (3, 4)])
def test_level_loop_fused_exchange_matches_simulation(world, seed):
    """fused exchange: run_level stores every output row into all ranks' arrays (here
    shared-memory CPU tensors stand in for the CUDA-IPC peer arrays) and the loop takes only a barrier per level;
    every rank must end with the plaintext simulation's values and identical arrays"""
    n_in, t, a, b, c = _netlist(seed)
    import paper_conf_ispass_maxw23_b200 as tb
    rows_total = tb.Netlist(n_in, t, a, b, c).n_wires
    shared = [torch.full((rows_total, 3), -1, dtype=torch.int32).share_memory_() for _ in range(world)]
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, seed, q, shared)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    bits = np.random.default_rng(seed).integers(0, 2, n_in)
    want = simulate(n_in, t, a, b, c, bits)[0]
    for rank, w, calls, rows in res:
        assert (w[rows, 0] == want).all(), "rank %d wire values differ from the plaintext simulation" % rank
    for _, w, _, _ in res[1:]:
        assert (w == res[0][1]).all()
    assert sum(g1 - g0 for _, _, calls, _ in res for (L, g0, g1) in calls) == len(t)


@pytest.mark.parametrize("world,seed", [(2, 6), (3, 7), (2, 8)])
def test_level_loop_fused_early_start_matches_simulation(world, seed):
    """with the level order planned for R ranks (tb_netlist_plan_world), each rank runs the next
    level's locally ready gates before the current level's barrier.  Every input a rank reads must be a primary
    input, a row exchanged at a barrier it has passed, or a row it computed itself (asserted inside run_level);
    the results equal the plaintext simulation and some gates really ran early."""
    n_in, t, a, b, c = _netlist(seed)
    import paper_conf_ispass_maxw23_b200 as tb
    net = tb.Netlist(n_in, t, a, b, c)
    levels, rows, early = net.plan_world(world)
    rows_total = net.n_wires
    shared = [torch.full((rows_total, 3), -1, dtype=torch.int32).share_memory_() for _ in range(world)]
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, seed, q, shared, True)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    bits = np.random.default_rng(seed).integers(0, 2, n_in)
    want = simulate(n_in, t, a, b, c, bits)[0]
    for rank, w, calls, rws in res:
        assert (w[rws, 0] == want).all(), "rank %d wire values differ from the plaintext simulation" % rank
    assert sum(g1 - g0 for _, _, calls, _ in res for (L, g0, g1) in calls) == len(t)
    assert early[1:].sum() > 0                      # the schedule found locally ready gates beyond level 1


def test_plan_world_partitions_levels():
    """tb_netlist_plan_world: the same levels as Algorithm 1, each level a permutation of its gates, and every
    early gate of rank r reads level-(L-1) rows only from r's own chunk"""
    import paper_conf_ispass_maxw23_b200 as tb
    from paper_conf_ispass_maxw23_b200 import parallel
    for seed in range(4):
        n_in, t, a, b, c = _netlist(seed)
        net = tb.Netlist(n_in, t, a, b, c)
        lv1, rows1 = net.plan()
        for world in (1, 2, 3, 5):
            lv, rows, early = net.plan_world(world)
            assert [ng for _, ng in lv] == [ng for _, ng in lv1]
            order = np.argsort(rows[n_in:])
            for L in range(2, len(lv) + 1):
                row0, ng = lv[L - 1]
                prow0, png = lv[L - 2]
                for r in range(world):
                    g0, g1, _ = parallel.shard(ng, world, r)
                    p0, p1, _ = parallel.shard(png, world, r)
                    assert early[L - 1, r] <= g1 - g0
                    for k in range(g0, g0 + early[L - 1, r]):
                        g = order[row0 - n_in + k]
                        for w in (a[g], b[g], c[g]):
                            if w >= 0 and prow0 <= rows[w] < prow0 + png:
                                assert prow0 + p0 <= rows[w] < prow0 + p1


def test_shard_and_slack():
    from paper_conf_ispass_maxw23_b200 import parallel
    assert parallel.shard(10, 4, 0) == (0, 3, 3) and parallel.shard(10, 4, 3) == (9, 10, 3)
    assert parallel.shard(2, 4, 3) == (2, 2, 1)
    assert parallel.shard(0, 8, 5) == (0, 0, 0)
    # padded gather of the last level may run past n_rows by at most world*chunk - n_gates
    assert parallel.slack_rows([(10, 10)], 20, 4) == 2
    for ng in range(1, 50):
        for R in (1, 2, 3, 8):
            spans = [parallel.shard(ng, R, r) for r in range(R)]
            assert sum(g1 - g0 for g0, g1, _ in spans) == ng
            assert all(spans[r][1] == spans[r + 1][0] for r in range(R - 1))


def test_shard_io_covers_inputs_and_outputs_once():
    """Context.shard_io (the per-rank I/O plan of the sharded end-to-end path, run_netlist_host_sharded): every
    rank's input rows contain every primary input its gate ranges read, and over the ranks every requested output
    is returned exactly once -- by the rank that produced it, or by rank 0 for an input passed through (host
    logic, no GPU)"""
    from types import SimpleNamespace

    import paper_conf_ispass_maxw23_b200 as tb
    from paper_conf_ispass_maxw23_b200 import parallel
    for seed in range(3):
        n_in, t, a, b, c = _netlist(seed)
        net = tb.Netlist(n_in, t, a, b, c)
        lv, rows = net.plan()
        dnet = SimpleNamespace(net=net, row_of_wire=rows, n_rows=net.n_wires,
                               levels=[(row0, ng, 0, 0) for row0, ng in lv])
        outs = np.random.default_rng(seed).choice(net.n_wires, 25, replace=False)
        order = np.argsort(rows[n_in:])
        for world in (1, 2, 3):
            seen = []
            for r in range(world):
                in_rows, o = tb.Context.shard_io(None, dnet, world, r, outs)
                seen += [k for k, _ in o]
                assert all(rows[outs[k]] == row for k, row in o)
                for row0, ng in lv:
                    g0, g1, _ = parallel.shard(ng, world, r)
                    for k in range(row0 - n_in + g0, row0 - n_in + g1):
                        g = order[k]
                        for w in (a[g], b[g], c[g]):
                            if 0 <= w < n_in and (w != b[g] or t[g] != 3) and (w != c[g] or t[g] == 16):
                                assert w in in_rows
            assert sorted(seen) == list(range(outs.size))      # pass-through inputs come from rank 0
            in0, _ = tb.Context.shard_io(None, dnet, world, 0, outs)
            assert all(rows[w] in in0 for w in outs if rows[w] < n_in)
