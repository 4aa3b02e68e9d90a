"""Multi-process (gloo, world size 2, CPU) check of the sharding logic used by
bench.py under torchrun: G-invariant inputs from global instance ids, no data
movement between ranks, per-rank checksums gathered once, and the combined
checksum equal to the single-process whole-problem checksum.  The CPU oracle
stands in for the kernels (this test runs without a GPU)."""
import os
import socket

import numpy as np
import pytest
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, algo, q):
    import sys
    sys.path.insert(0, ROOT)
    import bulkgen
    import oracle
    from paper_conf_ipps_tanitni14_b200 import shard
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        p_total = 37 * world + 3 if algo == "strong" else None
        if algo in ("weak", "tri"):
            h0, h1 = shard.weak_range(25, rank)
        else:
            h0, h1 = shard.strong_range(p_total, rank, world)
        if algo == "tri":
            c = bulkgen.tri_input(9, h1 - h0, seed=3, dtype="int32", h0=h0)
            res = oracle.bulk_opt(c, oracle.ROW_WISE)
            cs = bulkgen.checksum(res, h0=h0)
        else:
            x = bulkgen.prefix_input(40, h1 - h0, seed=2, dtype="float32", layout=bulkgen.COLUMN_WISE, h0=h0)
            res = oracle.bulk_prefix_sums(x, oracle.COLUMN_WISE)
            cs = bulkgen.checksum(res, bulkgen.COLUMN_WISE, h0=h0)
        parts = shard.gather_checksums(cs)
        t = shard.max_over_ranks(float(rank + 1))
        q.put((rank, parts, t))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("algo", ["weak", "strong", "tri"])
def test_two_rank_sharding_matches_single_process(algo):
    import bulkgen
    import oracle
    from paper_conf_ipps_tanitni14_b200 import shard
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, algo, q)) for r in range(world)]
    for pr in procs:
        pr.start()
    results = [q.get(timeout=120) for _ in range(world)]
    for pr in procs:
        pr.join(timeout=60)
        assert pr.exitcode == 0
    results.sort()
    parts = results[0][1]
    assert results[1][1] == parts                 # every rank sees the same gathered list
    assert results[0][2] == results[1][2] == 2.0  # max over ranks
    combined = shard.combine_checksums(parts)
    # the same problem in one process
    if algo == "tri":
        c = bulkgen.tri_input(9, 50, seed=3, dtype="int32")
        whole = bulkgen.checksum(oracle.bulk_opt(c, oracle.ROW_WISE))
    else:
        p = 50 if algo == "weak" else 37 * world + 3
        x = bulkgen.prefix_input(40, p, seed=2, dtype="float32", layout=bulkgen.COLUMN_WISE)
        whole = bulkgen.checksum(oracle.bulk_prefix_sums(x, oracle.COLUMN_WISE), bulkgen.COLUMN_WISE)
    assert combined == whole


def test_ranges():
    from paper_conf_ipps_tanitni14_b200 import shard
    assert shard.weak_range(10, 3) == (30, 40)
    covered = []
    for r in range(3):
        a, b = shard.strong_range(11, r, 3)
        covered += list(range(a, b))
    assert covered == list(range(11))
    assert shard.combine_checksums([2 ** 64 - 1, 2]) == 1
    assert shard.gather_checksums(5) == [5]           # no process group: identity
    np.testing.assert_equal(shard.max_over_ranks(3.5), 3.5)
