"""N > 1 host-side logic on CPU with world_size 2 (gloo): the ncclUniqueId bootstrap of
memxct_plan_set_comm, and the domain-decomposition helper every rank runs redundantly
(memxct_partition_ranges, reading R12 / P:723-729) giving identical, covering, balanced ranges."""
import os
import socket

import numpy as np
import pytest


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, q):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_sc_hidayetoglubgrg19_b200 import bootstrap_unique_id, partition_ranges
        uid = bootstrap_unique_id(rank)
        rng = np.random.default_rng(42)              # same weights on every rank
        w = rng.integers(1, 1000, size=777)
        b = partition_ranges(w, 8)
        got = [None] * world
        dist.all_gather_object(got, (uid, b.tolist()))
        q.put((rank, got, w.tolist()))
    finally:
        dist.destroy_process_group()


def test_gloo_world2_bootstrap_and_partition():
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=240) for _ in procs]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for rank, got, w in res:
        (u0, b0), (u1, b1) = got
        assert len(u0) == 128 and u0 == u1            # every rank holds rank 0's id
        assert b0 == b1                               # identical decomposition on every rank
        b = np.array(b0)
        assert b[0] == 0 and b[-1] == len(w) and np.all(np.diff(b) > 0)
        loads = [sum(w[b[i]:b[i + 1]]) for i in range(8)]
        assert max(loads) <= sum(w) / 8 + max(w)     # greedy prefix split: off by < one tile


def test_partition_ranges_edge_cases():
    from paper_conf_sc_hidayetoglubgrg19_b200 import partition_ranges
    assert partition_ranges([1, 1, 1, 1], 4).tolist() == [0, 1, 2, 3, 4]
    assert partition_ranges([0, 0, 0], 2).tolist()[0] == 0
    b = partition_ranges([10], 1)
    assert b.tolist() == [0, 1]
    b = partition_ranges([1] * 100, 3)
    assert b.tolist() == [0, 33, 67, 100]
    with pytest.raises(Exception):
        partition_ranges([-1, 2], 2)


def _host_comm_worker(rank, world, port, q, rounds):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_sc_hidayetoglubgrg19_b200.memxct import bootstrap_host_comm_name, host_comm_probe
        out = []
        for k in range(rounds):   # a fresh segment per round: create, attach, unlink, reuse of names
            name = bootstrap_host_comm_name(rank)
            out.append((name, host_comm_probe(name, rank, world, 1000 * k + 7 * rank + 1).tolist()))
        q.put((rank, out))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_gloo_host_transport_rendezvous(world):
    """The host transport's host side (memxct_plan_set_comm_host's rendezvous: a shared-memory
    segment created by rank 0 and attached by the others, process-shared barriers, the host
    allgather) across `world` processes on CPU, the segment name bootstrapped over gloo."""
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    rounds = 3
    procs = [ctx.Process(target=_host_comm_worker, args=(r, world, port, q, rounds)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=180) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for k in range(rounds):
        names = {res[r][k][0] for r in range(world)}
        assert len(names) == 1
        expect = [1000 * k + 7 * r + 1 for r in range(world)]
        for r in range(world):
            assert res[r][k][1] == expect


def test_host_transport_missing_peer_fails_loudly(monkeypatch):
    """A rank whose peers never arrive gets MEMXCT_ERR_NCCL after the time-out, not a hang."""
    import subprocess
    import sys
    code = ("import sys; sys.path.insert(0, %r)\n"
            "from paper_conf_sc_hidayetoglubgrg19_b200.memxct import host_comm_probe, MemXCTError\n"
            "try:\n    host_comm_probe('/memxct-missing-peer-test', 1, 2, 5)\nexcept MemXCTError as e:\n"
            "    print('ERR', e)\n") % os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ, MEMXCT_HOST_COMM_TIMEOUT_S="1.5")
    r = subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, text=True, timeout=120)
    assert "ERR" in r.stdout and "NCCL" in r.stdout, (r.stdout, r.stderr)
