"""Multi-process (gloo, CPU) tests of the sharding / exchange logic of dist.py (-m "not gpu").

The CUDA steps are swapped for CPU stand-ins (oracle transpose, numpy unpack, oracle sweep) so
that the partitioning, the all-to-all block routing and the all-reduce are checked end to end
with real torch.distributed collectives at world sizes 2 and 4.
"""
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


def _worker(rank, world, port, fn, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        q.put((rank, fn(rank, world)))
    except Exception as e:  # surface the failure to the parent
        q.put((rank, e))
    finally:
        dist.destroy_process_group()


def run_world(world, fn):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, fn, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=300) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
    for r, v in res.items():
        if isinstance(v, Exception):
            raise v
    return res


def _cpu_transpose(x, o):
    import oracle
    o.copy_(torch.from_numpy(oracle.transpose(x.numpy())))


def _cpu_unpack(recv, out, G):
    M = recv.shape[1]
    r = recv.numpy().reshape(G, M, M)
    for s in range(G):
        out[:, s * M:(s + 1) * M] = torch.from_numpy(r[s])


def _sharded_transpose_job(rank, world):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import workloads
    from paper_conf_icppw_nakanomi14_b200 import dist as rdist
    N = 24 * world
    M = N // world
    A = workloads.random_bits(N, N, torch.float32, seed=5)
    shard = A[rank * M:(rank + 1) * M].contiguous()
    out = rdist.transpose_sharded(shard, local_transpose=_cpu_transpose, local_unpack=_cpu_unpack)
    expect = A.view(torch.int32).t().contiguous()[rank * M:(rank + 1) * M]
    return bool(torch.equal(out.view(torch.int32), expect))


def _sweep_job(rank, world):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import oracle
    from paper_conf_icppw_nakanomi14_b200 import dist as rdist

    def local(count, seed, first_trial=0, **kw):
        return torch.from_numpy(oracle.sweep(32, ["stride", "diagonal", "random"], ["ras", "rap"], seed,
                                             first_trial, count, threads=1).astype(np.int64))
    h = rdist.congestion_sweep(5003, seed=7, first_trial=11, local=local)
    return h.numpy()


@pytest.mark.parametrize("world", [2, 4])
def test_sharded_transpose_routing(world):
    res = run_world(world, _sharded_transpose_job)
    assert all(res.values())


@pytest.mark.parametrize("world", [2, 3])
def test_sweep_allreduce_equals_single_run(oracle, world):
    res = run_world(world, _sweep_job)
    one = oracle.sweep(32, ["stride", "diagonal", "random"], ["ras", "rap"], 7, 11, 5003).astype(np.int64)
    for r in range(world):
        assert np.array_equal(res[r], one)


def test_trial_slices_partition():
    from paper_conf_icppw_nakanomi14_b200.dist import trial_slice
    for n in (0, 1, 7, 1000, 10 ** 9 + 7):
        for world in (1, 2, 3, 8):
            s = [trial_slice(n, r, world, 5) for r in range(world)]
            assert s[0][0] == 5 and sum(c for _, c in s) == n
            assert all(s[i][0] + s[i][1] == s[i + 1][0] for i in range(world - 1))
