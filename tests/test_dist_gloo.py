"""N>1 host logic of the driver on CPU: world_size-2 gloo process groups.

The per-shard compute is the oracle (the CUDA path needs a GPU); what is under test
is the driver's sharding arithmetic, its verification reduction (SUM of counts, MAX of
time) and the replica check -- the same code bench.py runs over NCCL."""
import os
import socket

import pytest
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, total, weak, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank),
                      WORLD_SIZE=str(world), LOCAL_RANK=str(rank))
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import oracle
    from paper_conf_cgo_murtovigplls24_b200 import driver
    from xs_workloads import GRID_SEED, LOOKUP_SEED
    R = driver.init(backend="gloo")
    assert R.world == world and R.rank == rank
    first, count = driver.weak_range(total, rank) if weak else driver.shard(total, rank, world)
    P = oracle.Problem(68, 1000, oracle.NUCLIDE, GRID_SEED)
    r = P.run_range(LOOKUP_SEED, first, count, macro=False)
    out = driver.reduce_stats(r["hash"], count, r["pairs"], float(rank + 1))
    same = driver.replicas_identical(12345)
    differ = driver.replicas_identical(12345 + rank)
    big = driver.replicas_identical((1 << 64) - 1)  # u64 checksums above 2^63
    mx = driver.max_over_ranks(float(10 * rank))
    driver.barrier()
    if rank == 0:
        q.put((out, same, differ, big, mx))
    driver.finalize()


@pytest.mark.parametrize("weak", [False, True])
def test_two_rank_reduction_matches_single_rank(weak, oracle_mod):
    from xs_workloads import GRID_SEED, LOOKUP_SEED
    world, total = 2, 30_001
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, total, weak, q)) for r in range(world)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(120)
        assert p.exitcode == 0
    (h, n, pairs, ms), same, differ, big, mx = q.get(timeout=10)
    P = oracle_mod.Problem(68, 1000, oracle_mod.NUCLIDE, GRID_SEED)
    full = P.run_range(LOOKUP_SEED, 0, total * (world if weak else 1), macro=False)
    assert (h, pairs) == (full["hash"], full["pairs"])
    assert n == total * (world if weak else 1)
    assert ms == 2.0 and mx == 10.0
    assert same and not differ and big


def test_shard_arithmetic():
    from paper_conf_cgo_murtovigplls24_b200 import driver
    for total in (0, 1, 7, 17_000_000, 10 ** 9):
        for world in (1, 2, 3, 4, 8):
            parts = [driver.shard(total, r, world) for r in range(world)]
            assert parts[0][0] == 0
            assert all(a + c == b for (a, c), (b, _) in zip(parts, parts[1:]))
            assert sum(c for _, c in parts) == total
            assert max(c for _, c in parts) - min(c for _, c in parts) <= 1
    assert driver.weak_range(100, 3) == (300, 100)
