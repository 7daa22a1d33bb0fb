"""Multi-process (world_size 2, gloo, CPU) tests of the N > 1 plumbing in dist.py:
index-blob broadcast, counter all-reduce (sum / max), and the queue-slice partition
(chunk c of D' -> rank c mod world) being a disjoint cover.  The GPU side of the same
path (slices joined on a real device, blob round trip) is in test_parity_gpu.py."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


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
        import paper_conf_ipps_galletg19_b200 as sj
        from paper_conf_ipps_galletg19_b200 import dist as sjdist

        res = {}
        # 1. blob broadcast (the index blob of sj_export_index is an opaque uint8 buffer)
        blob = None
        if rank == 0:
            g = torch.Generator().manual_seed(7)
            blob = torch.randint(0, 256, (100_003,), dtype=torch.uint8, generator=g)
        got = sjdist.broadcast_blob(blob, src=0, device="cpu")
        res["blob_sum"] = int(got.to(torch.int64).sum())
        res["blob_len"] = int(got.numel())
        # 2. counters
        res["sum"] = sjdist.allreduce_counts([rank + 1, 10 * rank], device="cpu")
        res["max"] = sjdist.allreduce_counts([100 + rank], device="cpu", op=dist.ReduceOp.MAX)
        # 3. queue slices of this rank, gathered
        n = 10_007  # WorkQueue chunks
        mine = torch.from_numpy(sj.sj_slice_chunks(n, rank, world).astype(np.int64))
        sizes = [torch.zeros(1, dtype=torch.int64) for _ in range(world)]
        dist.all_gather(sizes, torch.tensor([mine.numel()]))
        maxlen = int(max(s.item() for s in sizes))
        padded = torch.full((maxlen,), -1, dtype=torch.int64)
        padded[: mine.numel()] = mine
        allp = [torch.empty(maxlen, dtype=torch.int64) for _ in range(world)]
        dist.all_gather(allp, padded)
        cat = torch.cat([a[a >= 0] for a in allp])
        res["cover"] = bool(torch.equal(torch.sort(cat).values, torch.arange(n)))
        res["disjoint"] = bool(cat.numel() == n)
        res["balanced"] = int(max(s.item() for s in sizes) - min(s.item() for s in sizes))
        q.put((rank, res))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2])
def test_gloo_plumbing(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    out = dict(q.get(timeout=120) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    g = torch.Generator().manual_seed(7)
    ref = torch.randint(0, 256, (100_003,), dtype=torch.uint8, generator=g)
    for r in range(world):
        res = out[r]
        assert res["blob_len"] == ref.numel() and res["blob_sum"] == int(ref.to(torch.int64).sum())
        assert res["sum"] == [sum(i + 1 for i in range(world)), sum(10 * i for i in range(world))]
        assert res["max"] == [100 + world - 1]
        assert res["cover"] and res["disjoint"]
        assert res["balanced"] <= 1  # ranks differ by at most one chunk
