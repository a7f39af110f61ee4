"""Multi-process (gloo, CPU) tests of the multi-GPU host logic: shard ranges, max-over-ranks and
the splitter-based exchange of sorted runs (A13), against the oracle's global sort."""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, dist_name, n_total, q):
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    sys.path.insert(0, root)
    import torch
    import torch.distributed as dist

    import hsort_inputs
    import oracle
    from paper_conf_ipps_gowanlockk18a_b200 import dist as hd

    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        A = hsort_inputs.generate(dist_name, n_total, seed=77)
        lo, hi = hd.shard_range(n_total, world, rank)
        # local GPU-sort stand-in on CPU (test side): the oracle's key sort of the shard
        local = oracle.sort_u64(oracle.keys_from_f64(A[lo:hi]))
        mine = hd.exchange_sorted_runs(torch.from_numpy(local.view(np.int64)).view(torch.uint64))
        mx = hd.max_over_ranks(float(rank + 1))
        q.put((rank, mine.numpy().copy(), mx, (lo, hi)))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
@pytest.mark.parametrize("dist_name,n_total", [("uniform_pm1", 50_001), ("zipf_dup", 40_000),
                                               ("all_equal", 5_000), ("special", 3)])
def test_exchange_gives_global_sort(oracle_mod, inputs_mod, world, dist_name, n_total):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, dist_name, n_total, q))
             for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    res.sort(key=lambda x: x[0])
    got = np.concatenate([r[1] for r in res]) if res else np.zeros(0, np.uint64)
    A = inputs_mod.generate(dist_name, n_total, seed=77)
    want = oracle_mod.sort_u64(oracle_mod.keys_from_f64(A))
    assert np.array_equal(got, want)
    assert all(r[2] == float(world) for r in res)          # max over ranks
    cover = sorted(r[3] for r in res)                       # shards tile [0, n)
    assert cover[0][0] == 0 and cover[-1][1] == n_total
    assert all(cover[i][1] == cover[i + 1][0] for i in range(world - 1))


def test_shard_range_balanced():
    from paper_conf_ipps_gowanlockk18a_b200 import dist as hd
    for n in (0, 1, 7, 1000, 10**9 + 7):
        for w in (1, 2, 3, 8):
            sizes = [hd.shard_range(n, w, r)[1] - hd.shard_range(n, w, r)[0] for r in range(w)]
            assert sum(sizes) == n and max(sizes) - min(sizes) <= 1
