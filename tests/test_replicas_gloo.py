"""Multi-process (world_size 2, gloo, CPU) test of the replica aggregation bench.py uses
for N > 1 GPUs: one independent heap per rank (the queue does not shard),
timed as the max over ranks, throughput = all ranks' keys / that time."""
import os
import socket

import pytest
import torch.distributed as dist
import torch.multiprocessing as mp

import bench


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    local_ms = [100.0, 250.0][rank]
    got = bench.max_over_ranks(local_ms, dist, device="cpu")
    q.put((rank, got, bench.job_throughput(1 << 20, 3, world, got)))
    dist.barrier()
    dist.destroy_process_group()


def test_max_over_ranks_two_ranks_gloo():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = sorted(q.get(timeout=120) for _ in range(2))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert [r[1] for r in res] == [250.0, 250.0]
    assert res[0][2] == pytest.approx(2 * (1 << 20) * 3 / 0.25)


def test_single_rank_is_identity():
    assert bench.max_over_ranks(12.5) == 12.5
    assert bench.job_throughput(1000, 2, 1, 1000.0) == 2000.0
