"""World-size-2 gloo tests of the multi-GPU host logic (-m "not gpu").

bench.py at N > 1 runs a key-partitioned bank: every rank owns its own
accounts and its own seed (shard-local transactions, no data-path
collective), then ONE all-reduce sums the stats and the balance invariant
and takes the max of the timings.  Here each rank stands in for its GPU with
the CPU oracle's serial run of its shard and calls the same reduction
function bench.py uses.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    import sys
    sys.path.insert(0, ROOT)
    import bench
    import oracle as O
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    accounts, T, K = 1024, 64, 4
    p = O.params("bank", n_words=accounts)
    heap = O.init_heap(p, accounts)
    res, upd = O.serial(p, heap, T, K, bench.shard_seed(rank))
    vec = np.zeros(16)
    vec[0] = upd.sum()
    vec[1] = (~upd).sum()
    t_ms = 10.0 + rank
    out, (tmax, wall) = bench.reduce_over_ranks(vec, float(heap.astype(np.int64).sum()), t_ms, 0.5 * rank,
                                                world, dist, torch.device("cpu"))
    q.put((rank, int(vec[0]), int(vec[1]), out.tolist(), tmax, wall, heap.tobytes()))
    dist.barrier()
    dist.destroy_process_group()


def test_two_rank_reduction_gloo():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    got = [q.get(timeout=120) for _ in range(world)]
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    got.sort()
    commits = sum(g[1] for g in got)
    ro = sum(g[2] for g in got)
    for rank, c, r, out, tmax, wall, _ in got:
        assert out[0] == commits and out[1] == ro                # SUM over shards
        assert out[16] == world * 1024 * 1000                    # global balance invariant
        assert tmax == 11.0 and wall == 0.5                      # MAX over ranks
    assert commits + ro == world * 64 * 4
    # shards use different seeds, so their transactions (and heaps) differ
    assert got[0][6] != got[1][6]


def test_shard_seeds_are_distinct():
    import sys
    sys.path.insert(0, ROOT)
    import bench
    seeds = {bench.shard_seed(r) for r in range(8)}
    assert len(seeds) == 8


def _ht_worker(rank, world, port, q):
    import sys
    sys.path.insert(0, ROOT)
    import bench
    import oracle as O
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    B, T, K, KR = 64, 128, 4, 2048
    M = T * K
    bits = world.bit_length() - 1
    p = O.params("ht", ht_buckets=B, ht_key_range=KR, ht_lookup_pct=50, shard_bits=bits, shard=rank)
    heap = np.zeros(B + 2 * M, dtype=np.uint32)
    res, upd = O.serial(p, heap, T, K, bench.shard_seed(rank))
    nodes, distinct = bench.ht_walk_count(heap, B, M)
    ok = float(nodes == distinct == int(upd.sum()))
    vec = np.zeros(16)
    vec[0] = upd.sum()
    out, _ = bench.reduce_over_ranks(list(vec) + [nodes, ok], 0.0, 1.0, 0.0, world, dist, torch.device("cpu"))
    keys = sorted(int(heap[B + n - 1]) for n in range(1, M + 1) if heap[B + n - 1])
    q.put((rank, out.tolist(), keys))
    dist.barrier()
    dist.destroy_process_group()


def test_two_rank_key_partitioned_ht_gloo():
    """bench.py --workload ht host logic: each rank's shard (here the
    oracle's serial run of it) holds only keys it owns; the one reduction
    sums the key counts and the per-rank invariant flags."""
    import sys
    sys.path.insert(0, ROOT)
    import oracle as O
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_ht_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    got = sorted(q.get(timeout=120) for _ in range(world))
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    total = sum(len(k) for _, _, k in got)
    for rank, out, keys in got:
        assert out[16] == total and out[17] == world             # key count SUM; every rank's invariant held
        assert out[0] == total                                   # update commits = inserted keys
        assert all(O.key_owner(k, 1) == rank for k in keys)
    assert not set(got[0][2]) & set(got[1][2])                   # disjoint shards


def test_bench_roofline_object_is_the_contract_and_the_cost_model():
    """bench.py's `roofline` object (CPU-only arithmetic): contract keys, the
    algorithmic sector model of DESIGN.md §7.2 (paired bank update = 2 pair
    loads + 2 atom.or.b64 + 2 pair stores = 6 x 32 B; read-only = 2 loads;
    split TBV update 10 sectors, + 2 pre-lock VBV loads for HV), and
    achieved = bytes per launch / launch time."""
    import sys
    sys.path.insert(0, ROOT)
    import bench
    tot = {"commits": 1_000_000, "commits_ro": 250_000}
    r = bench.roofline(bench.Variant("hv", "paired"), "hv", tot, t_ms=2.0, steps=2,
                       peaks={"hbm_gbs": 6000.0}, peak_src="test", traffic=123)
    assert {"bound", "achieved", "peak", "unit", "frac", "traffic"} <= set(r)
    assert r["bound"] == "hbm" and r["unit"] == "GB/s" and r["traffic"] == 123
    assert r["bytes_per_unit"] == {"update_tx": 192, "read_only_tx": 64}
    per_launch = (1_000_000 * 192 + 250_000 * 64) / 2
    assert r["algorithmic_bytes_per_launch"] == per_launch
    assert abs(r["achieved"] - per_launch / 1e-3 / 1e9) < 1e-9
    assert abs(r["frac"] - r["achieved"] / 6000.0) < 1e-12
    split_tbv = bench.roofline(bench.Variant("tbv", "split"), "tbv", tot, 2.0, 2, {}, "fallback", traffic=0)
    assert split_tbv["bytes_per_unit"] == {"update_tx": 320, "read_only_tx": 128}
    assert split_tbv["peak"] == 6650.0                  # the profiling guide's fallback
    split_hv = bench.roofline(bench.Variant("hv", "split"), "hv", tot, 2.0, 2, {}, "fallback", traffic=0)
    assert split_hv["bytes_per_unit"]["update_tx"] == 384
