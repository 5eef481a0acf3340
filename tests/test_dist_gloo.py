"""Multi-process plumbing of the N>1 path on CPU (gloo, world_size 2): slice
assignment, MAX of per-rank times, checksum gather, and that the seeded
slices a rank generates are bitwise the same matrices a single process sees
(so outputs are identical across P)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import bqr_dist
import bqr_inputs


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank), WORLD_SIZE=str(world))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        per = 7
        lo, hi = bqr_dist.rank_slice(rank, world, per)
        A = bqr_inputs.random_batch(6, 5, world * per, "f32", seed=11, start=lo, stop=hi)
        t = bqr_dist.max_over_ranks(torch, dist, 1.5 + rank)
        sums = bqr_dist.gather_ints(torch, dist, [bqr_dist.checksum(A), rank])
        bqr_dist.barrier(torch, dist)
        q.put((rank, t, sums, A))
    finally:
        dist.destroy_process_group()


def test_gloo_world2_plumbing():
    world = 2
    port = _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    res.sort(key=lambda x: x[0])
    # MAX over ranks
    assert all(r[1] == 2.5 for r in res)
    # every rank sees every rank's checksum, in rank order
    assert res[0][2] == res[1][2] and [s[1] for s in res[0][2]] == [0, 1]
    # rank slices == the single-process stream
    full = bqr_inputs.random_batch(6, 5, world * 7, "f32", seed=11)
    np.testing.assert_array_equal(np.concatenate([res[0][3], res[1][3]]), full)
    assert res[0][2][0][0] == bqr_dist.checksum(full[:7]) & 0x7FFFFFFFFFFFFFFF


@pytest.mark.parametrize("world", [1, 2, 3, 8])
def test_strong_slices_cover_batch(world):
    total = 1001
    sl = [bqr_dist.rank_slice(r, world, 0, weak=False, total=total) for r in range(world)]
    assert sl[0][0] == 0 and sl[-1][1] == total
    assert all(sl[i][1] == sl[i + 1][0] for i in range(world - 1))


def test_generator_slices_independent_of_chunking():
    """Matrix b's values do not depend on which slice asked for it."""
    full = bqr_inputs.random_batch(4, 4, 300, "c64", seed=3, chunk=64)
    part = bqr_inputs.random_batch(4, 4, 300, "c64", seed=3, start=100, stop=231, chunk=64)
    np.testing.assert_array_equal(full[100:231], part)


def _bench_env():
    env = {k: v for k, v in os.environ.items() if k not in ("RANK", "WORLD_SIZE", "LOCAL_RANK", "MASTER_PORT")}
    env["CUDA_VISIBLE_DEVICES"] = ""
    return env


def test_bench_relaunches_itself_under_torchrun():
    """`python bench.py --gpus 2` (no torchrun environment) starts 2 ranks via
    torch.distributed.run; the ranks agree on the weak and strong slices of
    the C3 batch and rank 0 prints one JSON line (gloo, CPU)."""
    import json
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    r = subprocess.run([sys.executable, os.path.join(root, "bench.py"), "--gpus", "2", "--dry-run"],
                       capture_output=True, text=True, timeout=240, env=_bench_env(), cwd=root)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, r.stdout
    out = json.loads(lines[0])
    assert out["n_gpus"] == 2 and out["max_rank"] == 1.0
    assert out["weak_slices"] == [[0, 5000], [5000, 10000]]
    assert out["strong_slices"] == [[0, 2500], [2500, 5000]]


def test_bench_rejects_world_size_mismatch():
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = _bench_env()
    env.update(WORLD_SIZE="2", RANK="0", LOCAL_RANK="0")
    r = subprocess.run([sys.executable, os.path.join(root, "bench.py"), "--gpus", "4", "--dry-run"],
                       capture_output=True, text=True, timeout=120, env=env, cwd=root)
    assert r.returncode != 0 and "WORLD_SIZE=2" in r.stderr
