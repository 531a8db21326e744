"""The N>1 bench path is replicas only: each rank runs its own
instance; the process group carries only the timing reductions.  This CPU
test runs bench.py's plumbing with world_size 2 over gloo."""
import os
import sys

import pytest
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _worker(rank, ws, port, q):
    os.environ.update(RANK=str(rank), LOCAL_RANK=str(rank), WORLD_SIZE=str(ws),
                      MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    sys.path.insert(0, ROOT)
    import bench
    w, r, local = bench.dist_setup(None, backend="gloo")
    bench.barrier(w)
    mx = bench.allmax(w, 10.0 + r)          # e.g. each replica's median latency
    sm = bench.allsum(w, 100.0 * (r + 1))   # e.g. each replica's batch jobs/s
    q.put((r, w, local, mx, sm))
    import torch.distributed as dist
    dist.destroy_process_group()


def test_replica_reductions_world_size_2():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = 29500 + (os.getpid() % 1000)
    ps = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    out = sorted(q.get(timeout=120) for _ in range(2))
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert [o[0] for o in out] == [0, 1]
    assert all(o[1] == 2 for o in out)
    assert all(o[3] == 11.0 for o in out)      # max over ranks
    assert all(o[4] == 300.0 for o in out)     # sum over ranks


def test_reference_arm_other_ranks_do_no_work(monkeypatch):
    sys.path.insert(0, ROOT)
    import bench
    monkeypatch.setenv("RANK", "1")

    class A:
        warmup, steps, seed, size = 1, 1, 0, 4096
    assert bench.reference_arm(A()) is None
