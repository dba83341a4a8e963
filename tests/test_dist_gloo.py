"""Multi-process host logic with torch.distributed (gloo, world size 2, CPU).

The hot path shards by clip with no data-path collective. These tests run the
per-rank pieces in two processes: each rank plans its own clips with the product's host planner,
the ranks exchange them over gloo, and the union must be every clip exactly once per epoch
 with per-clip plans independent of the rank; bench.py's max-over-ranks timing and its
counter all-gather (the run's only collective) are exercised with the same process group.
"""
import os
import socket
import sys

import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, q):
    sys.path.insert(0, ROOT)
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import bench
        import paper_conf_sosp_yelllhkh25_b200 as sand
        from paper_conf_sosp_yelllhkh25_b200 import configs
        w = configs.k400()
        w.spec.world_size = world
        vids = [(1000 + i, w.n_frames, w.width, w.height) for i in range(50)]
        results = {}
        for epoch in (0, 1):
            mine = sand.plan_rank_clips(w.spec, [v[0] for v in vids], epoch, rank)
            gathered = [None] * world
            dist.all_gather_object(gathered, mine)
            results[epoch] = gathered
            # per-clip plans do not depend on the rank that plans them
            plans = {c: tuple(sand.plan_clip(w.spec, vids, epoch, c).frames[0][:16]) for c in mine[:4]}
            allp = [None] * world
            dist.all_gather_object(allp, plans)
            results[f"plans{epoch}"] = allp
        # bench.py aggregation helpers over the same group (CPU tensors for gloo)
        mx = bench.max_over_ranks([10.0 * (rank + 1), 1.0 + rank], world, "cpu")
        tot, per = bench.gather_counters([rank + 1, 10 * (rank + 1), 3], world, "cpu")
        results["max"] = mx
        results["counters"] = (tot, per)
        q.put((rank, results))
    finally:
        dist.destroy_process_group()


@pytest.mark.timeout(300)
def test_two_rank_partition_and_aggregation():
    world = 2
    port = _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    out = dict(q.get(timeout=240) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for epoch in (0, 1):
        lists = out[0][epoch]
        assert lists == out[1][epoch]
        union = sorted(c for lst in lists for c in lst)
        assert union == list(range(50))                       # 50 clips, W=2: exactly once
        assert len(lists[0]) == len(lists[1]) == 25
        # the same clip planned by either rank gives the same frames
        merged = {}
        for d in out[0][f"plans{epoch}"]:
            for c, fr in d.items():
                assert merged.setdefault(c, fr) == fr
    assert out[0]["max"] == out[1]["max"] == [20.0, 2.0]
    tot, per = out[0]["counters"]
    assert tot == [3, 30, 6] and per == [[1, 10, 3], [2, 20, 3]]
