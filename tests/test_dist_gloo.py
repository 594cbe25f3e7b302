"""World-size-2 tests of the multi-rank host path on CPU (gloo backend): the unique-id
exchange and the max/sum timing reductions bench.py uses, and the merge schedule of the C++
coordinator — every rank must issue the same number of merge collectives per epoch whatever its
(adaptive, rank-specific) batch sizes, or NCCL would deadlock."""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank),
                      WORLD_SIZE=str(world), LOCAL_RANK=str(rank))
    import torch.distributed as dist
    from paper_conf_ipps_marws21_b200 import dist as hbd
    try:
        r, w, loc = hbd.init("gloo")
        assert (r, w, loc) == (rank, world, rank)
        uid = hbd.share_bytes(bytes(range(128)) if rank == 0 else None)
        assert uid == bytes(range(128))
        t = hbd.reduce_scalar(10.0 + rank, "max")
        s = hbd.reduce_scalar(1.0 + rank, "sum")
        # rank-specific adaptive-looking batch sequences (powers of two in [32, 8192])
        rng = np.random.default_rng(100 + rank)
        res = []
        for N, M in [(581012, 4), (64700, 8), (10000, 3), (1000, 16)]:
            b = 2 ** rng.integers(5, 14, size=4000)
            res.append(hbd.merge_schedule(N, M, b))
        out = [None] * world
        dist.all_gather_object(out, res)
        q.put((rank, t, s, out))
        dist.destroy_process_group()
    except Exception as e:  # pragma: no cover - reported to the parent
        q.put((rank, "error", repr(e), None))


def test_two_rank_plumbing_and_merge_schedule_gloo():
    world, port = 2, _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    ps = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in ps:
        p.start()
    got = [q.get(timeout=240) for _ in range(world)]
    for p in ps:
        p.join(timeout=60)
    for rank, t, s, out in got:
        assert t != "error", s
        assert t == 11.0 and s == 3.0
        per_rank = out
        # every rank performs exactly M merges per epoch ...
        for Mi, M in enumerate([4, 8, 3, 16]):
            assert all(r[Mi][1] == M for r in per_rank)
        # ... even though their mid-epoch merge points differ
    assert got[0][3] == got[1][3]


def test_merge_schedule_single_rank_properties():
    from paper_conf_ipps_marws21_b200 import dist as hbd
    assert hbd.merge_schedule(100, 4, [25, 25, 25, 25]) == (3, 4)      # thresholds 25, 50, 75 crossed
    assert hbd.merge_schedule(100, 4, [100]) == (1, 4)                 # several thresholds in one batch
    assert hbd.merge_schedule(100, 0, [10] * 10) == (0, 0)
    assert hbd.merge_schedule(100, 2, [60, 60]) == (1, 2)              # second batch not served
    with pytest.raises(Exception):
        hbd.merge_schedule(0, 2, [1])
