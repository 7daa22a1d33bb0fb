"""The multi-GPU path end to end on ONE device: two processes (gloo process group, both on
cuda:0) run exactly what bench.py runs per rank -- rank 0 builds the index, the blob is
broadcast (host blob through gloo here; a device blob through NCCL in bench.py), the other
rank rebuilds a handle from it, every rank joins its queue slice, and the counts are
all-reduced.  The union of the slices must equal the oracle, with no pair twice."""
import os
import socket

import numpy as np
import pytest

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)

import torch.distributed as dist  # noqa: E402
import torch.multiprocessing as mp  # noqa: E402


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, cfg_name, n, q, mode="broadcast"):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import paper_conf_ipps_galletg19_b200 as sj
        import workloads
        from paper_conf_ipps_galletg19_b200 import dist as sjdist

        torch.cuda.set_device(0)
        cfg = workloads.get_config(cfg_name).scaled(n)
        pts = torch.from_numpy(cfg.points()).cuda()
        if mode == "replicated":  # every rank builds from its own copy (bench.py --mp replicated)
            with sj.Handle(pts, cfg.eps, k=8) as h0:
                cap = h0.count()
            out = torch.empty((max(cap, 1), 2), dtype=torch.int32, device="cuda")
            h, local, total = sjdist.replicated_self_join(pts, cfg.eps, out, max(cap, 1), k=8)
            pairs = out[:local].cpu().numpy().view(np.uint32).reshape(-1, 2).copy()
            st = h.stats()
            h.close()
            q.put((rank, pairs, total, st["dist_calcs"], 0))
            return
        h = None
        if rank == 0:
            h = sj.Handle(pts, cfg.eps, k=8)
        h, blob = sjdist.replicate_index(h, 0, None, device="cpu")
        if mode == "view" and rank != 0:  # the broadcast blob on the device, aliased (zero copy)
            h.close()
            dblob = blob.cuda()
            h = sj.Handle.from_index(dblob, dblob.numel(), view=True)
        h.set_slice(rank, world)
        pairs = sj.self_join_pairs(h, "cuda").cpu().numpy().view(np.uint32).reshape(-1, 2).copy()
        total = sjdist.allreduce_counts([pairs.shape[0]], device="cpu")[0]
        st = h.stats()
        h.close()
        q.put((rank, pairs, total, st["dist_calcs"], int(blob.numel())))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,cfg_name,n,mode", [(2, "c5", 80_000, "broadcast"), (3, "c3k64", 60_000, "broadcast"),
                                                   (2, "c5", 80_000, "view"), (3, "c2k64", 60_000, "replicated"),
                                                   (2, "c4k32", 20_000, "replicated")])
def test_slices_across_processes(world, cfg_name, n, mode):
    import oracle
    import workloads

    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, cfg_name, n, q, mode)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict((r[0], r[1:]) for r in (q.get(timeout=300) for _ in range(world)))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    cfg = workloads.get_config(cfg_name).scaled(n)
    want = oracle.grid_pairs(cfg.points(), cfg.eps)
    parts = [res[r][0] for r in range(world)]
    cat = np.concatenate(parts)
    assert cat.shape == want.shape  # disjoint slices: no pair evaluated twice
    np.testing.assert_array_equal(oracle.canonical(cat), want)
    for r in range(world):
        assert res[r][1] == want.shape[0]          # all-reduced count
        assert res[r][2] == res[0][2]              # same index on every rank
        assert res[r][3] == res[0][3]              # same blob size
