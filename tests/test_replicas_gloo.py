"""N > 1 host logic on CPU (world size 2, gloo): the replica path has no data
collective -- every rank plans the same graph independently (identical plans),
and the only cross-rank traffic is the barrier, the max of the timings
(bench.reduce_max) and the gather of the replica statistics, SURVEY.md §8(e).
The concurrent cold-start choreography (bench.replica_cold_trials) and the
replica block (bench.replica_summary: per-replica cold lists, contention
cold(N)/cold(1), kernels loaded per replica, aggregate / per-GPU imgs/s) run
here with a fake child in place of the native pask_cold process."""
import os
import socket
import time

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

    # concurrent cold starts with a fake child: it records when it was released;
    # all ranks' children of one trial must be released after the same barrier
    releases = []

    def fake_child():
        box = {}

        def release():
            box["t"] = time.time()
            releases.append(box["t"])

        def collect():
            solo = len(releases) > trials
            return {"cold_us": (400.0 if solo else 500.0 + 10 * rank), "kernels_loaded": 2, "t": box["t"]}
        return release, collect
    trials = 3
    conc, solo = bench.replica_cold_trials(fake_child, dist, rank, trials)
    gathered = [None] * world
    dist.all_gather_object(gathered, {"conc": conc, "solo": solo, "hot_ms": 0.25 + 0.05 * rank})
    summary = None
    if rank == 0:
        summary = bench.replica_summary([g["conc"] for g in gathered], gathered[0]["solo"],
                                        [g["hot_ms"] for g in gathered], 1)
    q.put((rank, mx, digests, st["kernels_loaded"], conc, solo, summary))
    dist.destroy_process_group()


def test_two_replicas_plan_max_and_replica_block():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = sorted([q.get(timeout=300) for _ in procs], key=lambda r: r[0])
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for rank, mx, digests, kl, conc, solo, _ in res:
        assert mx == [2.0, 10.0, 3.0]
        assert digests[0] == digests[1]
        assert kl == 5
        assert len(conc) == 3
        assert len(solo) == (3 if rank == 0 else 0)      # cold(1): rank 0 alone
    # trial t of both ranks released between the same two barriers: before any
    # child of trial t + 1
    c0, c1 = res[0][4], res[1][4]
    for t in range(2):
        assert max(c0[t]["t"], c1[t]["t"]) < min(c0[t + 1]["t"], c1[t + 1]["t"])
    s = res[0][6]
    assert s["n_replicas"] == 2
    assert [r["cold_med_ms"] for r in s["per_replica"]] == [0.5, 0.51]
    assert [r["kernels_loaded"] for r in s["per_replica"]] == [[2], [2]]
    assert s["cold_1_med_ms"] == 0.4
    assert s["contention"] == pytest.approx(0.505 / 0.4, abs=1e-3)
    assert s["hot_imgs_s_aggregate"] == pytest.approx(4000 + 1000 / 0.3, abs=0.2)
    assert s["hot_imgs_s_per_gpu"] == pytest.approx(s["hot_imgs_s_aggregate"] / 2, abs=0.1)
