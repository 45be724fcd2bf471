"""N>1 host logic of the batch-sharded replicas on CPU: world_size-2 gloo process group."""
import os
import socket

import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_asplos_xiazswwyfc24_b200 import replicas as R


def test_shard_covers_every_request_once():
    for n in (0, 1, 7, 64, 129):
        for ws in (1, 2, 3, 8):
            ids = [i for r in range(ws) for i in R.shard(n, ws, r)]
            assert ids == list(range(n))
            sizes = [len(R.shard(n, ws, r)) for r in range(ws)]
            assert max(sizes) - min(sizes) <= 1


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, ws, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=ws)
    try:
        assert R.world() == (ws, rank)
        # every rank "times" a different duration; the job time is the max
        t = R.max_over_ranks(1.0 + rank)
        rate = R.aggregate_rate(10, t)
        # each rank's replica output = its shard of request ids, gathered on rank 0 for checking
        mine = torch.tensor([float(i) for i in R.shard(6, ws, rank)])
        got = R.gather_to_rank0(mine)
        if rank == 0:
            q.put((t, rate, got.reshape(-1).tolist()))
        else:
            assert got is None
    finally:
        dist.destroy_process_group()


@pytest.mark.timeout(120)
def test_gloo_world_size_2():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    for p in ps:
        p.join(100)
        assert p.exitcode == 0
    t, rate, ids = q.get(timeout=10)
    assert t == 2.0                      # max over ranks
    assert rate == 2 * 10 / 2.0          # units of all ranks / slowest time
    assert ids == [0, 1, 2, 3, 4, 5]     # shards gathered in rank order cover the stream once
