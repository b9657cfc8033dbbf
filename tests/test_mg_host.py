"""Host-side logic of the multi-GPU path on CPU (-m "not gpu"): the block-cyclic partition (the Python
bookkeeping and the library's trid_mg_local_cols agree, cover every column once, balance the load) and a
world_size-2 gloo job that exchanges each rank's column set and the 128-byte communicator id the way
comm_nccl() does (broadcast from rank 0 through torch.distributed)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import paper_conf_ppopp_wangdzwzljz25_b200 as trid
import trid_gen


@pytest.mark.parametrize("n,cb,g", [(256, 32, 1), (300, 32, 3), (49152, 64, 8), (1000, 64, 7), (65, 64, 2),
                                    (5, 64, 4)])
def test_partition_cover_and_balance(n, cb, g):
    seen = np.zeros(n, dtype=np.int64)
    sizes = []
    for q in range(g):
        c = trid_gen.block_cyclic_columns(n, cb, g, q)
        assert trid.mg_local_cols(n, cb, g, q) == len(c)
        assert np.all(np.diff(c) > 0)                           # local order = global order
        assert np.all(((c // cb) % g) == q)                     # owner(c) = (c / cb) mod g
        seen[c] += 1
        sizes.append(len(c))
    assert np.all(seen == 1)
    assert max(sizes) - min(sizes) <= cb                        # at most one block apart


def test_mg_bufsize_and_argument_checks():
    L = trid.lib()
    n, b = 1000, 64
    sizes = [trid.sbr_dbbr_mg_bufsize(n, b, 16, 256, 4, q) for q in range(4)]
    assert all(s > 8 * n * 256 * 2 for s in sizes)              # replicated Y and Z (n x k each)
    assert trid.mg_local_cols(10, 0, 1, 0) == -1
    assert L.trid_sbr_dbbr_mg(None, n, None, n, b, b, 16, 256, None, None, 0, None) == -1


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, n, cb, q_out):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        cols = torch.from_numpy(trid_gen.block_cyclic_columns(n, cb, world, rank))
        # every rank learns every rank's column count and set (what the band gather assumes)
        cnt = torch.tensor([cols.numel()], dtype=torch.int64)
        cnts = [torch.zeros(1, dtype=torch.int64) for _ in range(world)]
        dist.all_gather(cnts, cnt)
        mx = int(max(c.item() for c in cnts))
        pad = torch.full((mx,), -1, dtype=torch.int64)
        pad[: cols.numel()] = cols
        allc = [torch.zeros(mx, dtype=torch.int64) for _ in range(world)]
        dist.all_gather(allc, pad)
        union = torch.cat([a[a >= 0] for a in allc]).sort().values
        ok_cover = torch.equal(union, torch.arange(n))
        # the 128-byte id exchange of comm_nccl (rank 0 -> all)
        buf = torch.zeros(128, dtype=torch.uint8)
        if rank == 0:
            buf.copy_(torch.arange(128, dtype=torch.uint8))
        dist.broadcast(buf, src=0)
        ok_id = torch.equal(buf, torch.arange(128, dtype=torch.uint8))
        # max-over-ranks timing reduction used by bench.py
        t = torch.tensor([float(rank + 1)], dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        q_out.put((rank, ok_cover, ok_id, float(t.item()), [int(c.item()) for c in cnts]))
    finally:
        dist.destroy_process_group()


def test_gloo_two_rank_partition_and_id_exchange():
    world, n, cb = 2, 1000, 64
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, n, cb, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for rank, ok_cover, ok_id, tmax, cnts in res:
        assert ok_cover and ok_id and tmax == 2.0
        assert cnts == [trid.mg_local_cols(n, cb, world, r) for r in range(world)]


def test_bench_gpus_flag_spawns_ranks():
    """bench.py --gpus N without a launcher re-runs itself under torch.distributed.run with N ranks (gloo dry run on
    CPU: the rank plumbing the driver's multi-GPU bench uses), and refuses a --gpus / WORLD_SIZE mismatch."""
    import json
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = {k: v for k, v in os.environ.items() if k not in ("WORLD_SIZE", "RANK", "LOCAL_RANK")}
    out = subprocess.run([sys.executable, os.path.join(root, "bench.py"), "--gpus", "2", "--dry-run"],
                         capture_output=True, text=True, timeout=300, env=env)
    assert out.returncode == 0, out.stderr[-2000:]
    line = json.loads([x for x in out.stdout.splitlines() if x.startswith("{")][-1])
    assert line["world_size"] == 2 and sorted(r[0] for r in line["ranks"]) == [0, 1]
    bad = subprocess.run([sys.executable, os.path.join(root, "bench.py"), "--gpus", "2", "--dry-run"],
                         capture_output=True, text=True, timeout=120, env={**env, "WORLD_SIZE": "1"})
    assert bad.returncode == 2
