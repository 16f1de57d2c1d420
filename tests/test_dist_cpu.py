"""Host logic of the N > 1 path, with world_size-2 gloo process groups on CPU:
the NCCL unique-id broadcast bench.py performs before a sharded init, and the
weak-scaling instance every rank generates independently (it must be
identical on all ranks, or the shards would not describe one problem)."""
import hashlib
import os
import socket

import numpy as np
import pytest
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _digest(inst):
    h = hashlib.sha256()
    for arr in (inst.A.rowptr, inst.A.col, inst.B.rowptr, inst.B.col, inst.L.a, inst.L.b, inst.L.w):
        h.update(np.ascontiguousarray(arr).tobytes())
    return h.hexdigest()


def _worker(rank, world, port, q):
    import sys
    sys.path.insert(0, ROOT)
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import paper_conf_sc_xiangkfah23_b200 as ca
        from synth import make_config
        # 1. the unique id is created on rank 0 and broadcast (bench.py shard_kw)
        obj = [ca.nccl_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        ids = [None] * world
        dist.all_gather_object(ids, obj[0])
        # 2. the weak-scaling instance (O at scale 0.002 x world) is identical
        inst = make_config("O", scale=0.002 * world)
        digs = [None] * world
        dist.all_gather_object(digs, _digest(inst))
        q.put((rank, len(obj[0]), len(set(ids)), len(set(digs)), inst.L.m))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2])
def test_gloo_id_broadcast_and_identical_instances(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for rank, idlen, n_ids, n_digs, m in res:
        assert idlen == 128
        assert n_ids == 1, "all ranks must hold the same NCCL unique id"
        assert n_digs == 1, "all ranks must generate the same instance"
        assert m > 0
