"""N > 1 host logic on CPU (world size 2, gloo): the replica path has no data
collective -- every rank plans the same graph independently (identical plans),
and the only cross-rank traffic is the barrier and the max of the timings
(bench.reduce_max), SURVEY.md §8(e)."""
import os
import socket

import pytest
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import bench
    from paper_conf_dac_huangdxz25_b200 import pask as P
    from paper_conf_dac_huangdxz25_b200.model import DeviceModel
    from workloads import build_model
    spec, _ = build_model("resnet50")
    plan, st = P.plan(DeviceModel(spec, alloc=False).graph)
    dist.barrier()
    # fake per-rank timings: rank r is slower by r
    mx = bench.reduce_max([1.0 + rank, 10.0 - rank, 3.0], dist)
    digests = [None] * world
    dist.all_gather_object(digests, hash(tuple(tuple(b) for b in plan)))
    q.put((rank, mx, digests, st["kernels_loaded"]))
    dist.destroy_process_group()


def test_two_replicas_plan_and_max():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in procs]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for rank, mx, digests, kl in res:
        assert mx == [2.0, 10.0, 3.0]
        assert digests[0] == digests[1]
        assert kl == 5
