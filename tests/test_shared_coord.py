"""The cross-process coordinator (hb_coord_create): one Algorithm 2 state and one
epoch cursor over 𝔹 in POSIX shared memory, shared by the processes of a node (one per GPU).

Host-only tests (no GPU): the shared state replays the oracle's virtual-clock schedule exactly
when the ScheduleWork messages arrive in the oracle's order — from one process, and from two
processes (gloo world size 2) that each own some of the workers and take turns."""
import os
import socket
import uuid

import numpy as np
import pytest
import torch.multiprocessing as mp

import paper_conf_ipps_marws21_b200 as hb
from oracle import coord as ocoord
from tests.test_abi import same, to_c_policy

D2 = ocoord.Policy(kind=ocoord.ADAPTIVE, alpha=2, eta0=0.1, b0=8,
                   workers=[ocoord.WorkerSpec(2, 8, 2, 0.0, 1.0), ocoord.WorkerSpec(4, 16, 16, 2.0, 0.25)])
THREE = ocoord.Policy(kind=ocoord.ADAPTIVE, alpha=2, eta0=0.5, b0=4, credit="dispatch",
                      workers=[ocoord.WorkerSpec(1, 8, 8, 0.5, 0.25), ocoord.WorkerSpec(2, 4, 2, 1.0, 1.0),
                               ocoord.WorkerSpec(1, 16, 1, 0.0, 2.0, 2.0)])


def replay(coord, recs, owned):
    """Feed the oracle's ScheduleWork order to the shared state (only the `owned` workers' messages;
    the caller interleaves processes).  Returns the records the shared coordinator produced."""
    out = []
    for r in recs:
        if r.worker not in owned:
            continue
        out.append(coord.schedule(r.worker, r.vtime))
        if not r.served:
            coord.idle(r.worker)
    return out


def test_shared_state_replays_the_oracle_trace_in_one_process():
    for pol, N, epochs in [(D2, 40, 2), (THREE, 97, 3)]:
        recs = ocoord.run(pol, N, epochs)
        c = hb.Coord(f"/hbtest_{uuid.uuid4().hex[:12]}", to_c_policy(pol), N, 1, 0)
        try:
            got = replay(c, recs, set(range(len(pol.workers))))
            same(got, [r.astuple() for r in recs])
            # a reset starts a fresh run of the same policy
            c.reset(to_c_policy(pol), N)
            same(replay(c, recs, set(range(len(pol.workers)))), [r.astuple() for r in recs])
        finally:
            c.close()


def test_shared_state_argument_errors():
    c = hb.Coord(f"/hbtest_{uuid.uuid4().hex[:12]}", to_c_policy(D2), 40, 1, 0)
    try:
        with pytest.raises(hb.HogbatchError):
            c.schedule(2, 0.0)       # worker id out of range
        with pytest.raises(hb.HogbatchError):
            c.idle(-1)
    finally:
        c.close()
    with pytest.raises(hb.HogbatchError):
        hb.Coord("no_slash", to_c_policy(D2), 40, 1, 0)
    with pytest.raises(hb.HogbatchError):
        hb.Coord(f"/hbtest_{uuid.uuid4().hex[:12]}", to_c_policy(D2), 40, 2, 2)   # rank >= nranks


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


OWNERS = {"D2": [{0}, {1}], "THREE": [{0, 2}, {1}]}


def _rank(rank, world, port, name, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank),
                      WORLD_SIZE=str(world), LOCAL_RANK=str(rank))
    import torch.distributed as dist
    try:
        dist.init_process_group("gloo")
        res = {}
        for key, pol, N, epochs in [("D2", D2, 40, 2), ("THREE", THREE, 97, 3)]:
            shm = name + key
            if rank == 0:
                c = hb.Coord(shm, to_c_policy(pol), N, world, 0)
            dist.barrier()
            if rank != 0:
                c = hb.Coord(shm, to_c_policy(pol), N, world, rank)
            recs = ocoord.run(pol, N, epochs)
            mine = OWNERS[key][rank]
            got = []
            for r in recs:  # the processes take turns in the oracle's message order
                if r.worker in mine:
                    got.append(c.schedule(r.worker, r.vtime))
                    if not r.served:
                        c.idle(r.worker)
                dist.barrier()
            res[key] = got
            dist.barrier()
            c.close()
        q.put((rank, res))
        dist.destroy_process_group()
    except Exception as e:  # pragma: no cover - reported to the parent
        q.put((rank, repr(e)))


def test_two_processes_share_one_schedule_gloo():
    world, port = 2, _free_port()
    name = f"/hbtest_{uuid.uuid4().hex[:10]}"
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    ps = [ctx.Process(target=_rank, args=(r, world, port, name, q)) for r in range(world)]
    for p in ps:
        p.start()
    got = dict(q.get(timeout=300) for _ in range(world))
    for p in ps:
        p.join(timeout=60)
    for r in range(world):
        assert isinstance(got[r], dict), got[r]
    for key, pol, N, epochs in [("D2", D2, 40, 2), ("THREE", THREE, 97, 3)]:
        merged = sorted(got[0][key] + got[1][key], key=lambda t: t[0])
        same(merged, [r.astuple() for r in ocoord.run(pol, N, epochs)])
        # each process saw only its own workers' records, and the ranges served across the
        # processes are disjoint and contiguous within each epoch (one 𝔹 for all GPUs)
        for rank in range(world):
            assert {t[2] for t in got[rank][key]} <= OWNERS[key][rank]
        for e in range(epochs):
            served = sorted((t[10], t[7]) for t in merged if t[1] == e and t[9])
            assert served and served[0][0] == 0
            assert all(a[0] + a[1] == b[0] for a, b in zip(served, served[1:]))
