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


def _worker(rank, ws, port, q, n_req):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=ws)
    try:
        assert R.world() == (ws, rank)
        # every rank "times" a different duration; the job time is the max
        t = R.max_over_ranks(1.0 + rank)
        rate = R.aggregate_rate(10, t)
        # each rank's replica output = its shard of request ids, gathered on rank 0 for checking
        mine = torch.tensor([[float(i), 10.0 * i] for i in R.shard(n_req, ws, rank)]).reshape(-1, 2)
        got = R.gather_to_rank0(mine)
        if rank == 0:
            q.put((t, rate, got[:, 0].tolist(), got[:, 1].tolist()))
        else:
            assert got is None
    finally:
        dist.destroy_process_group()


@pytest.mark.timeout(180)
@pytest.mark.parametrize("ws,n_req", [(2, 6), (3, 7), (3, 2)])
def test_gloo_replicas(ws, n_req):
    """world_size 2 with equal shards, 3 ranks x 7 requests (shards 3/2/2) and 3 ranks x 2 requests
    (one rank has an EMPTY shard): max-over-ranks time, aggregate rate, ordered gather."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, ws, port, q, n_req)) for r in range(ws)]
    for p in ps:
        p.start()
    for p in ps:
        p.join(150)
        assert p.exitcode == 0
    t, rate, ids, tens = q.get(timeout=10)
    assert t == float(ws)                    # max over ranks (rank r "took" 1 + r)
    assert rate == ws * 10 / float(ws)       # units of all ranks / slowest time
    assert ids == [float(i) for i in range(n_req)]   # shards gathered in rank order cover the stream once
    assert tens == [10.0 * i for i in range(n_req)]
