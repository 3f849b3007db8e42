"""Multi-process host logic of the multi-GPU paths on CPU (gloo, world_size 2):
source sharding, unique-id broadcast, max-over-ranks timing reduction, and the
bench's weak-scaling bookkeeping.  (The CUDA/NCCL data path needs GPUs and is
covered by the -m gpu tests with logical partitions and an NCCL world of 1.)"""
import os
import socket

import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_asplos_0003wh0dhwy0lyl25_b200 import distributed as tgd


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        sources = list(range(100, 164))
        mine = tgd.shard_sources(sources, rank, world)
        allm = [None] * world
        dist.all_gather_object(allm, mine)
        flat = [x for blk in allm for x in blk]
        uid = bytes(range(128)) if rank == 0 else None
        got = tgd.broadcast_bytes(uid, 128, 0)
        mx = tgd.max_over_ranks(10.0 + rank)
        q.put((rank, flat == sources, got == bytes(range(128)), mx, len(mine)))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2])
def test_gloo_world2(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in ps:
        p.start()
    res = [q.get(timeout=120) for _ in ps]
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    for rank, cover, uid_ok, mx, nmine in res:
        assert cover and uid_ok and mx == 10.0 + world - 1 and nmine == 64 // world


def test_shard_sources_partition():
    s = list(range(37))
    for world in (1, 2, 3, 8):
        blocks = [tgd.shard_sources(s, r, world) for r in range(world)]
        assert [x for b in blocks for x in b] == s
        assert max(map(len, blocks)) - min(map(len, blocks)) <= 1
