"""Multi-rank execution of real netlists on the GPU kernels (-m gpu): R = 2 and 3 processes share the one
B200 of the test box, each running its shard of every level through tb_run_level, with the level's output rows
exchanged either by an in-place all-gather in torch.distributed (gloo on CUDA tensors here; NCCL on a
multi-GPU box -- the level loop, paper_conf_ispass_maxw23_b200.parallel.level_loop, is the same code) or by the
fused all-gather (key-switch stores into the other ranks' arrays, mapped with CUDA IPC).  Every rank's wire array
must equal the oracle's level-by-level evaluation byte for byte (R-invariance).
"""
import os
import socket
import tempfile

import numpy as np
import pytest

import oracle as O
import synth

pytestmark = pytest.mark.gpu


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _netlist():
    from test_host import random_dag
    n_in, t, a, b, c = random_dag(21, n_inputs=6, n_gates=40)
    return dict(n_inputs=n_in, type=t, in0=a, in1=b, in2=c)


def _worker(rank, world, port, keyfile, ctsfile, q, exchange, early_start=False):
    import torch
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import paper_conf_ispass_maxw23_b200 as tb
        k = np.load(keyfile)
        ctx = tb.Context(0)
        ctx.load_keys(k["bk"], k["ksk"])
        n = _netlist()
        net = tb.Netlist(n["n_inputs"], n["type"], n["in0"], n["in1"], n["in2"])
        dnet = ctx.upload(net, world=world if early_start else 1)   # early start: level order for R ranks
        wires = ctx.wire_array(dnet, slack_rows=tb.slack_rows(dnet, world))
        cts = np.load(ctsfile)
        wires[:n["n_inputs"], :631] = ctx.to_device(cts)[:, :631]
        ctx.run_netlist(dnet, wires, group=dist.group.WORLD, exchange=exchange)
        torch.cuda.synchronize()
        q.put((rank, ctx.to_host(wires[:dnet.n_rows])[dnet.row_of_wire]))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,exchange,early", [(2, "allgather", False), (3, "allgather", False),
                                                  (2, "fused", False), (3, "fused", False), (2, "fused", True),
                                                  (3, "fused", True)])
def test_sharded_netlist_matches_oracle(world, exchange, early):
    """exchange="fused": the key-switch kernels store each output row into every rank's wire array through CUDA
    IPC peer mappings (the fused all-gather; same-device IPC between processes here, NVLink peers on a box).
    early=True: the netlist is planned for R ranks and each rank runs the next level's locally ready gates
    before the current level's barrier."""
    import torch
    import torch.multiprocessing as mp
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    import paper_conf_ispass_maxw23_b200 as tb
    tb.build()
    keys = O.keygen(O.DEFAULT, seed=555)
    n = _netlist()
    cts = O.encrypt_bits(keys, synth.random_bits(n["n_inputs"], 8), 9)
    with tempfile.TemporaryDirectory() as d:
        kf, cf = os.path.join(d, "keys.npz"), os.path.join(d, "cts.npy")
        np.savez(kf, bk=keys.bk, ksk=keys.ksk)
        np.save(cf, cts)
        ctx = mp.get_context("spawn")
        q = ctx.Queue()
        port = _port()
        procs = [ctx.Process(target=_worker, args=(r, world, port, kf, cf, q, exchange, early))
                 for r in range(world)]
        for p in procs:
            p.start()
        res = [q.get(timeout=600) for _ in range(world)]
        for p in procs:
            p.join(timeout=120)
            assert p.exitcode == 0
    from test_gpu_workloads import run_oracle_levels
    ref = run_oracle_levels(keys, n, cts)
    for rank, w in res:
        assert (w == ref).all(), "rank %d differs from the oracle" % rank
