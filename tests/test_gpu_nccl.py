"""The NCCL transport of the sharded path, run for real.

`test_gpu_shard.py` checks the sharded algorithm with in-process virtual
shards (device copies in place of collectives).  Here `world` separate
processes each hold one shard and exchange through libnccl (torch's), all on
the one GPU this sandbox has: each rank gets its own NCCL_HOSTID, so NCCL
treats the ranks as different hosts and connects them over its socket
transport instead of rejecting a duplicate device.  The result must equal the
unsharded handle BIT FOR BIT (per-edge state on every owned slice, every
round's scores / overlaps / cardinalities, the best matching).
"""
import os
import socket
import subprocess
import sys

import numpy as np
import pytest

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _run(tmp_path, world, config, scale, iters, flags=0):
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    port = _free_port()
    procs = []
    for r in range(world):
        env = dict(os.environ)
        env.update(RANK=str(r), WORLD_SIZE=str(world), LOCAL_RANK="0", MASTER_ADDR="127.0.0.1",
                   MASTER_PORT=str(port), NCCL_HOSTID=f"cualign-nccl-test-{r}", NCCL_SOCKET_IFNAME="lo",
                   NCCL_IB_DISABLE="1", NCCL_NVLS_ENABLE="0", CUDA_VISIBLE_DEVICES=env.get("CUDA_VISIBLE_DEVICES", "0"))
        cmd = [sys.executable, os.path.join(ROOT, "tests", "nccl_worker.py"), "--config", config, "--scale",
               str(scale), "--iters", str(iters), "--flags", str(flags), "--out", str(tmp_path)]
        procs.append(subprocess.Popen(cmd, env=env, stdout=subprocess.PIPE, stderr=subprocess.STDOUT, cwd=ROOT))
    outs = []
    for p in procs:
        try:
            out, _ = p.communicate(timeout=420)
        except subprocess.TimeoutExpired:
            for q in procs:
                q.kill()
            raise
        outs.append(out.decode(errors="replace"))
    for r, (p, out) in enumerate(zip(procs, outs)):
        assert p.returncode == 0, f"rank {r} exited {p.returncode}:\n{out[-4000:]}"
    return [np.load(os.path.join(tmp_path, f"rank{r}.npz")) for r in range(world)]


def _check(res, world):
    ref = res[0]
    covered = 0
    prev = 0
    for r in range(world):
        d = res[r]
        e0, e1 = int(d["e0"]), int(d["e1"])
        assert e0 == prev, "shards must tile the edge ids in rank order"
        prev = e1
        covered += e1 - e0
        for k in ("yc", "zc", "yp", "zp", "d"):
            bad = np.nonzero(d[k] != ref["ref_" + k][e0:e1])[0]
            assert bad.size == 0, f"rank {r} {k}: {bad.size} entries differ from the unsharded run"
        assert np.array_equal(d["rounds"], ref["ref_rounds"]), f"rank {r}: round infos differ"
        assert np.array_equal(d["mate"], ref["ref_mate"]), f"rank {r}: best matching differs"
    assert covered == ref["ref_yc"].size


@pytest.mark.parametrize("world", [2, 3])
def test_nccl_shards_bitwise_O_small(tmp_path, world):
    res = _run(tmp_path, world, "O", 0.01, 6)
    _check(res, world)
    assert int(res[0]["merge_rounds"]) >= 1


def test_nccl_shards_bitwise_P_literal_damped(tmp_path):
    import paper_conf_sc_xiangkfah23_b200 as ca
    res = _run(tmp_path, 2, "P", 0.05, 5, ca.FLAG_OTHERMAX_LITERAL | ca.FLAG_ROUND_DAMPED)
    _check(res, 2)
