"""Multi-process host logic on CPU (gloo, world_size 2): the replica
aggregation bench.py uses (value = all ranks' ops / max-over-ranks time), and
the reference arm's rank behaviour under torchrun."""
import json
import os
import socket
import subprocess
import sys

import pytest
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank), WORLD_SIZE=str(world))
    sys.path.insert(0, ROOT)
    import bench
    d = bench.Dist(rank, world, "gloo")
    d.barrier()
    ops = 1000.0 * (rank + 1)            # rank r processed 1000*(r+1) ops
    ms = 10.0 * (rank + 1)               # in 10*(r+1) ms of device time
    value, ms_max, total = bench.aggregate(d, ops, ms)
    q.put((rank, value, ms_max, total, d.max(float(rank)), d.sum(1.0)))
    d.close()


def test_gloo_world2_replica_aggregation():
    world, port = 2, _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = sorted(q.get(timeout=120) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for rank, value, ms_max, total, mx, sm in res:
        assert ms_max == 20.0 and total == 3000.0            # slowest rank, all ops
        assert value == pytest.approx(3000.0 / 0.020)        # whole-job ops/s
        assert mx == 1.0 and sm == 2.0


def test_reference_arm_nonzero_rank_exits_quietly():
    env = dict(os.environ, RANK="1", WORLD_SIZE="2", LOCAL_RANK="1")
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--gpus", "2"],
                         capture_output=True, text=True, env=env, timeout=120)
    assert out.returncode == 0 and out.stdout.strip() == ""


def test_reference_arm_line():
    """--impl reference times the CPU oracle on a bounded sample and prints the
    contract's JSON line (rank 0, N=1)."""
    env = dict(os.environ, RANK="0", WORLD_SIZE="1")
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--steps", "1",
                          "--warmup", "1", "--scale", "64"], capture_output=True, text=True, env=env, timeout=300)
    assert out.returncode == 0, out.stderr[-2000:]
    line = json.loads(out.stdout.strip().splitlines()[-1])
    assert line["impl"] == "reference" and line["value"] > 0 and line["unit"] == "ops/s"
    assert line["cpu_baseline"]["kind"] == "oracle" and line["e2e"]["h2d_bytes_per_step"] == 0
    assert line["higher_is_better"] is True
