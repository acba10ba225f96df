"""Multi-process host logic of the N>1 path on CPU (gloo, world size 2) -m "not gpu".

The B200 path runs the same functions over NCCL (bench.py under torchrun); here they are
checked with gloo: query sharding, the one-time arena broadcast, max-over-ranks timing,
the optional output gather, and that shards generated independently per rank equal the
corresponding slices of the single-process query stream."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_isca_hauswaldklclmdm15_b200 import parallel


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from datagen import recipes
        # 1. arena broadcast: rank 0's packed bytes reach every rank unchanged
        buf = torch.zeros(1 << 16, dtype=torch.uint8)
        if rank == 0:
            buf.copy_(torch.from_numpy(np.random.RandomState(5).randint(0, 256, 1 << 16).astype(np.uint8)))
        parallel.broadcast_buffer(buf, src=0)
        # 2. max over ranks
        t = parallel.max_over_ranks(10.0 + rank)
        # 3. weak-scaling shard of the counter-based stream
        r0, n = parallel.weak_shard(300, rank)
        shard = recipes.gen_input_rows("asr", r0, n, "bf16")
        # 4. strong-scaling split of whole queries
        sr0, sn = parallel.query_shard(7, 548, world, rank)
        # 5. gather of output rows
        out = torch.full((3 + rank, 4), float(rank))
        g = parallel.gather_rows(out, dst=0)
        q.put((rank, int(buf.sum()), t, shard, (sr0, sn), None if g is None else [x.shape[0] for x in g]))
    finally:
        dist.destroy_process_group()


def test_world2_host_logic():
    world, port = 2, _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = {}
    for _ in range(world):
        r = q.get(timeout=300)
        res[r[0]] = r
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    expect_sum = int(np.random.RandomState(5).randint(0, 256, 1 << 16).astype(np.uint8).astype(np.int64).sum())
    from datagen import recipes
    full = recipes.gen_input_rows("asr", 0, 600, "bf16")
    for r in range(world):
        assert res[r][1] == expect_sum                      # broadcast delivered rank 0's bytes
        assert res[r][2] == 11.0                            # max over ranks
        np.testing.assert_array_equal(res[r][3], full[300 * r: 300 * (r + 1)])
    assert res[0][4] == (0, 4 * 548) and res[1][4] == (4 * 548, 3 * 548)
    assert res[0][5] == [3, 4] and res[1][5] is None


@pytest.mark.parametrize("nq,world", [(7, 2), (16, 8), (5, 8), (1024, 3)])
def test_query_shard_partitions_whole_queries(nq, world):
    rows = []
    for r in range(world):
        r0, n = parallel.query_shard(nq, 28, world, r)
        assert r0 % 28 == 0 and n % 28 == 0
        rows.append((r0, n))
    assert rows[0][0] == 0
    for (a0, an), (b0, _) in zip(rows, rows[1:]):
        assert a0 + an == b0                               # contiguous
    assert sum(n for _, n in rows) == nq * 28              # complete
    assert max(n for _, n in rows) - min(n for _, n in rows) <= 28   # balanced
