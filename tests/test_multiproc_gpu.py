"""Multi-process paths with the CUDA library on ONE GPU (-m gpu).

Only one B200 is available to the tests, so several ranks (gloo process group, 127.0.0.1) share
cuda:0.  That still crosses real process boundaries with the CUDA path:
  * the fused sharded transpose (NEXT-2, rap_transpose_to_peers) writes into the OTHER process's
    output shard through a CUDA IPC mapping of its allocation (transport "ipc"), not through
    local pointers;
  * the NCCL-path pieces (local rap_transpose, the all-to-all of M x M blocks, rap_unpack_blocks)
    and the histogram all-reduce run with the library's kernels on each rank (gloo stages the
    collectives through host memory);
  * bench.py itself under torchrun with RAP_BENCH_BACKEND=gloo (default / dist / dist_fused).
Every output is compared with the oracle (element by element) or with the oracle's stored
10^9-trial histogram.
"""
import json
import os
import socket
import subprocess
import sys

import numpy as np
import pytest
import torch

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, fn, args, q):
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        q.put((rank, fn(rank, world, *args)))
    except Exception as e:  # surface the failure to the parent
        import traceback
        q.put((rank, RuntimeError(f"rank {rank}: {e}\n{traceback.format_exc()}")))
    finally:
        dist.destroy_process_group()


def run_world(world, fn, *args):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, fn, args, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=600) for _ in range(world))
    for p in procs:
        p.join(timeout=120)
    for r, v in res.items():
        if isinstance(v, Exception):
            raise v
    return res


def _bits(t):
    import workloads
    return workloads.as_bits_numpy(t)


def _fused_ipc(rank, world, N, dtype_name, layout):
    import oracle
    import workloads
    from paper_conf_icppw_nakanomi14_b200 import dist as rdist
    dt = getattr(torch, dtype_name)
    M = N // world
    A = workloads.random_bits(N, N, dt, seed=N + world)             # the same matrix on every rank
    shard = A[rank * M:(rank + 1) * M].cuda()
    ft = rdist.FusedTranspose((M, N), dt, layout=layout, seed=7, transport="ipc")
    assert ft.ptrs[rank] == ft.out.data_ptr() and len(set(ft.ptrs)) == world
    for rep in range(2):                                             # twice: the barriers order reuse
        out = ft(shard)
        expect = oracle.transpose(_bits(A[:, rank * M:(rank + 1) * M]))   # rows rank*M.. of A^T
        assert np.array_equal(_bits(out), expect), (rank, rep)
        ft.out.zero_()
        torch.cuda.synchronize()
        import torch.distributed as dist
        dist.barrier()
    return True


@pytest.mark.parametrize("world,N,dtype,layout", [(2, 2048, "float32", "rap"), (2, 1024, "float64", "rap"),
                                                  (3, 1536, "float32", "raw"), (4, 4096, "float32", "rap")])
def test_fused_transpose_over_cuda_ipc_between_processes(world, N, dtype, layout):
    assert all(run_world(world, _fused_ipc, N, dtype, layout).values())


def _sharded_and_sweep(rank, world, N):
    import oracle
    import workloads
    from paper_conf_icppw_nakanomi14_b200 import dist as rdist
    M = N // world
    A = workloads.random_bits(N, N, torch.float32, seed=5)
    out = rdist.transpose_sharded(A[rank * M:(rank + 1) * M].cuda(), layout="rap", seed=3)
    assert np.array_equal(_bits(out), oracle.transpose(_bits(A[:, rank * M:(rank + 1) * M])))
    # the sweep: trial ranges per rank + one all-reduce; `out` already holds counts
    base = torch.full((5, 3, 33), 7, dtype=torch.int64, device="cuda")
    h = rdist.congestion_sweep(30000, seed=2, first_trial=1000, out=base)
    expect = oracle.sweep(32, ["contiguous", "stride", "diagonal", "random", "malicious"],
                          ["raw", "ras", "rap"], 2, 1000, 30000).astype(np.int64) + 7
    assert np.array_equal(h.cpu().numpy(), expect)
    return True


@pytest.mark.parametrize("world,N", [(2, 4096), (4, 2048)])
def test_sharded_transpose_and_sweep_between_processes(world, N):
    assert all(run_world(world, _sharded_and_sweep, N).values())


def _torchrun_bench(nproc, *argv):
    env = dict(os.environ, RAP_BENCH_BACKEND="gloo")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={nproc}",
           "--master-addr", "127.0.0.1", f"--master-port={_free_port()}", os.path.join(ROOT, "bench.py"),
           "--gpus", str(nproc), *argv]
    out = subprocess.run(cmd, capture_output=True, text=True, timeout=1200, env=env, cwd=ROOT)
    assert out.returncode == 0, out.stderr[-4000:]
    lines = [json.loads(l) for l in out.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, out.stdout
    return lines[0]


def test_bench_default_two_ranks_gloo():
    # every rank its own cfg4 transpose; the 10^9 cfg2 trials split over the ranks with one
    # all-reduce per step -- bench.py asserts the histogram equals the oracle's stored run
    line = _torchrun_bench(2, "--steps", "3", "--warmup", "3", "--no-cpu")
    assert line["n_gpus"] == 2 and line["value"] > 0 and line["unit"] == "GB/s"
    assert line["sweep"]["trials"] == 10 ** 9 and line["sweep"]["bit_identical_to_oracle_1e9"] is True
    assert set(line["cfg3_layouts"]["layouts"]) == {"raw", "pad", "xor", "ras", "rap"}
    assert line["e2e"]["h2d_bytes_per_step"] == 2 * 16384 * 16384 * 8


@pytest.mark.parametrize("workload", ["dist", "dist_fused"])
def test_bench_cfg5_two_ranks_gloo(workload):
    # cfg5 32768^2 float32 row-block-sharded over 2 ranks: the NCCL-path pieces (all-to-all staged
    # through host memory under gloo) or the fused IPC peer stores; bench.py checks e2e == device
    line = _torchrun_bench(2, "--workload", workload, "--steps", "2", "--warmup", "3", "--no-cpu")
    assert line["n_gpus"] == 2 and line["value"] > 0 and line["scaling"] == "strong"
    assert "2 GPU" in line["config"]["workload"]
