"""Multi-GPU host logic (paper_conf_dsn_zhaoxcqzj24_b200/dist.py) with world-size-2 gloo on CPU: run sharding,
kernel-sequence gathering and the byte all-to-all of the exchange.  (The merge of the owners' rows is a
library call, owl_merge_leaks / owl_merge_diffs, checked against the oracle in tests/test_gpu_sequences.py.)"""
import os
import socket

import pytest
import torch.multiprocessing as mp



def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    import torch
    import torch.distributed as dist

    from paper_conf_dsn_zhaoxcqzj24_b200 import dist as D
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        runs = list(range(11))
        mine = D.shard(runs, world, rank)
        meta = {r: (r % 2, [100 + r, 7]) for r in mine}
        allm = D.gather_sequences(meta)
        # rank k sends (k+1) bytes valued 10k+j to owner j
        counts = [rank + 1] * world
        send = torch.cat([torch.full((rank + 1,), 10 * rank + j, dtype=torch.uint8) for j in range(world)])
        recv, rc = D.exchange_bytes(send, counts)
        q.put((rank, mine, sorted(allm.items()), rc, recv.tolist()))
    finally:
        dist.destroy_process_group()


def test_gloo_world2_shard_gather_exchange():
    world, port = 2, _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    ps = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in ps:
        p.start()
    out = {}
    for _ in range(world):
        rank, mine, allm, rc, recv = q.get(timeout=120)
        out[rank] = (mine, allm, rc, recv)
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert out[0][0] + out[1][0] == list(range(11)) and abs(len(out[0][0]) - len(out[1][0])) <= 1
    want = [(r, (r % 2, [100 + r, 7])) for r in range(11)]
    assert out[0][1] == want and out[1][1] == want
    for j in range(world):  # owner j receives rank k's bucket j, rank 0's first
        assert out[j][2] == [k + 1 for k in range(world)]
        assert out[j][3] == [10 * k + j for k in range(world) for _ in range(k + 1)]


def test_shard_balanced_and_contiguous():
    from paper_conf_dsn_zhaoxcqzj24_b200 import dist as D
    for n in (0, 1, 7, 200):
        for world in (1, 2, 3, 8):
            parts = [D.shard(range(n), world, r) for r in range(world)]
            assert sum(parts, []) == list(range(n))
            assert max(map(len, parts)) - min(map(len, parts)) <= 1
