"""N > 1 host-side path on CPU: world_size-2 gloo, one library instance per rank.

Each rank runs the decision core (DECISIONS_ONLY, no device) on its own shard
of a workload, exactly as bench.py's ranks do on their own GPUs, and the ranks
combine timings with the same max-over-ranks helper.  Checks: the plumbing
works with gloo at world size 2, every rank's trace equals the oracle's on its
shard, and placement-only sharding loses/duplicates no job.
"""
import os
import socket

import pytest
import torch.multiprocessing as mp

import strings_workload as W


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank),
                      WORLD_SIZE=str(world), LOCAL_RANK=str(rank))
    try:
        from oracle.des import run_oracle
        from paper_conf_sc_senguptagsp14_b200 import parallel as par
        from paper_conf_sc_senguptagsp14_b200 import strings as S
        from paper_conf_sc_senguptagsp14_b200.runner import run_workload

        info = par.rank_info()
        g = par.init_groups(info, device_backend=None)
        full = W.config_c3()
        mine = par.shard_tenants(len(full.tenants), info.world, info.rank)
        remap = {t: i for i, t in enumerate(mine)}
        jobs = []
        for j in full.jobs:
            if j.tenant in remap:
                jj = W.JobSpec(**vars(j))
                jj.tenant = remap[j.tenant]
                jobs.append(jj)
        wl = W.Workload("shard", full.config, [full.tenants[t] for t in mine], jobs)
        par.barrier(g)
        r = run_workload(wl, timing_mode=S.DECISIONS_ONLY)
        same = r.trace == run_oracle(wl).trace
        span = max(i.t_done[2] for i in r.infos)
        mx = par.max_over_ranks(g, float(span))
        tot = par.sum_over_ranks(g, float(len(wl.jobs)))
        allx = par.gather_over_ranks(g, [float(rank)] * (rank + 1))
        assert allx == [0.0, 1.0, 1.0], allx                 # rank order, every rank's entries
        q.put((rank, same, span, mx, tot, r.stats.jobs_done))
        import torch.distributed as dist
        dist.destroy_process_group()
    except Exception as e:  # pragma: no cover - reported to the parent
        q.put((rank, repr(e)))


def test_world2_gloo_placement_sharding():
    world, port = 2, _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    ps = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in ps:
        p.start()
    res = sorted(q.get(timeout=240) for _ in ps)
    for p in ps:
        p.join(timeout=60)
    assert all(len(r) == 6 for r in res), res
    spans = [r[2] for r in res]
    assert all(r[1] for r in res)                      # each rank's trace == oracle on its shard
    assert all(r[3] == max(spans) for r in res)        # max over ranks
    assert all(r[4] == len(W.config_c3().jobs) for r in res)   # no job lost or duplicated
    assert sum(r[5] for r in res) == len(W.config_c3().jobs)


def test_shard_tenants_partition():
    from paper_conf_sc_senguptagsp14_b200 import parallel as par
    for world in (1, 2, 3, 8):
        parts = [par.shard_tenants(64, world, r) for r in range(world)]
        flat = sorted(t for p in parts for t in p)
        assert flat == list(range(64))


def test_whole_job_jain_helper():
    # the bench's whole-job Jain (Eq. 3, reading R-2): equal shares -> 1, one
    # tenant served of n -> 1/n, scale-invariant; single-rank gather is identity
    from paper_conf_sc_senguptagsp14_b200 import parallel as par
    assert par.jain([0.3] * 7) == pytest.approx(1.0)
    assert par.jain([0.0, 0.0, 2.5, 0.0]) == pytest.approx(0.25)
    xs = [0.1, 0.4, 0.2]
    assert par.jain(xs) == pytest.approx(par.jain([10 * x for x in xs]))
    assert par.gather_over_ranks(None, xs) == xs


def test_copy_threads_per_rank(monkeypatch):
    # 8 ranks on one node share its CPUs: each PMT copy pool gets its share
    from paper_conf_sc_senguptagsp14_b200 import parallel as par
    monkeypatch.setattr(par.os, "sched_getaffinity", lambda pid: set(range(224)))
    monkeypatch.setattr(par.os, "cpu_count", lambda: 224)
    assert par.copy_threads_per_rank(par.RankInfo(0, 8, 0, 8)) == 12          # 28 CPUs each -> capped
    monkeypatch.setattr(par.os, "sched_getaffinity", lambda pid: set(range(112)))   # bound to 1 of 2 nodes
    assert par.copy_threads_per_rank(par.RankInfo(0, 8, 0, 8)) == 12
    monkeypatch.setattr(par.os, "sched_getaffinity", lambda pid: set(range(16)))
    monkeypatch.setattr(par.os, "cpu_count", lambda: 16)
    assert par.copy_threads_per_rank(par.RankInfo(0, 4, 0, 4)) == 2            # 4 CPUs each
    assert par.copy_threads_per_rank(par.RankInfo(0, 1, 0, 1)) == 12


def _node_worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank),
                      WORLD_SIZE=str(world), LOCAL_RANK=str(rank))
    try:
        from oracle.des import run_oracle
        from paper_conf_sc_senguptagsp14_b200 import parallel as par
        from paper_conf_sc_senguptagsp14_b200 import strings as S
        from paper_conf_sc_senguptagsp14_b200.runner import run_workload

        info = par.rank_info()
        g = par.init_groups(info, device_backend=None, timeout_s=600)

        def work(group):
            # node mode: ONE library instance places every job of the whole
            # workload on one of G devices through the level-1 balancer
            wl = W.config_c3()                       # G = 4, MBF
            r = run_workload(wl, timing_mode=S.DECISIONS_ONLY)
            span = max(i.t_done[2] for i in r.infos)
            mx = par.max_over_ranks(group, float(span))
            gids = sorted({i.gid for i in r.infos})
            return (r.trace == run_oracle(wl).trace, span, mx, gids, r.stats.jobs_done)

        out = par.node_mode(info, g, work)
        q.put((rank, out))
        import torch.distributed as dist
        dist.destroy_process_group()
    except Exception as e:  # pragma: no cover - reported to the parent
        q.put((rank, repr(e)))


def test_world2_gloo_node_mode_rank0_drives_the_balancer():
    # bench.py --gpus N under torchrun: rank 0 owns the node (level-1 balancer
    # over all devices), rank 1 does no work, the timing max over ranks is rank 0's
    world, port = 2, _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    ps = [ctx.Process(target=_node_worker, args=(r, world, port, q)) for r in range(world)]
    for p in ps:
        p.start()
    res = dict(q.get(timeout=240) for _ in ps)
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert res[1] is None, res
    same, span, mx, gids, done = res[0]
    assert same                                   # the balancer's trace equals the oracle's
    assert mx == span                             # max over ranks = rank 0's span
    assert gids == [0, 1, 2, 3]                   # jobs spread over every device
    assert done == len(W.config_c3().jobs)
