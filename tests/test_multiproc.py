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


def test_bench_roofline_object_is_the_contract():
    """bench.py's `roofline` object (CPU-only arithmetic): the contract keys,
    achieved and peak in algorithmic L2 sector bytes (32 B per access of the
    committed transactions' own op mix), frac = achieved tx/s over the measured
    op-mix roof, and the SURVEY §8(d) max-formula figure beside it."""
    import sys
    sys.path.insert(0, ROOT)
    import bench
    roof = {"roof_tx_per_s": 2.0e10, "threads": 75776, "round_trips_per_tx": 4.0}
    peaks = {"ld": 2.8e11, "atom": 1.25e11, "st": 1.8e11, "clock": 4.9e10}
    ops = {"ld": 2.0, "atom": 2.0, "st": 2.0, "clock": 1.0}
    maxf = bench.max_formula(ops, peaks)
    assert abs(maxf - 1 / max(2 / 2.8e11, 2 / 1.25e11, 2 / 1.8e11, 1 / 4.9e10)) < 1e-3
    r = bench.roofline_object(1.0e10, roof, maxf, 6.0, "test")
    assert {"bound", "achieved", "peak", "unit", "frac", "traffic"} <= set(r)
    assert r["bound"] == "l2" and r["unit"] == "GB/s" and r["traffic"] is None
    assert abs(r["achieved"] - 1.0e10 * 192 / 1e9) < 1e-6 and abs(r["peak"] - 2.0e10 * 192 / 1e9) < 1e-6
    assert abs(r["frac"] - 0.5) < 1e-12 and abs(r["frac"] - r["achieved"] / r["peak"]) < 1e-12
    assert abs(r["frac_max_formula"] - 1.0e10 / maxf) < 1e-9


def test_op_mix_programs_follow_algorithm_3():
    """The op-mix roof's per-transaction programs (roofline.py) issue exactly
    Algorithm 3's memory operations for the committed transactions' log sizes:
    paired bank update = 2 pair loads, 2 atom.or (one pipelined round), the
    clock, 2 pair stores (4 round trips); split TBV RA (4R/4W, 8 locks) = 4 +
    4 loads, 8 sequential atomics (Q15), 4 write-back + 8 release stores, the
    clock; HV adds the pre-lock VBV loads (A3.l71); read-only = reads only."""
    from paper_conf_cgo_xuwglgq14_b200 import roofline as R
    st = dict(commits=900, commits_ro=100, reads_update=1800, reads_ro=200, writes_update=1800, locks_update=1800)
    p = R.programs_from_stats("bank", st, paired=True, mode="hv", prelock=False, pipelined=True)
    ops = R.op_counts(p)
    assert abs(ops["ld"] - 2.0) < 1e-3 and abs(ops["atom"] - 0.9 * 2) < 1e-3
    assert abs(ops["st"] - 0.9 * 2) < 1e-3 and abs(ops["clock"] - 0.9) < 1e-3
    assert abs(R.round_trips(p) - (0.9 * 3 + 0.1 * 1)) < 1e-3       # loads, atomics, clock (stores: no wait)
    st = dict(commits=10, commits_ro=0, reads_update=40, reads_ro=0, writes_update=40, locks_update=80)
    p = R.programs_from_stats("ra", st, paired=False, mode="tbv", prelock=True, pipelined=False)
    ops = R.op_counts(p)
    assert ops == {"ld": 8.0, "atom": 8.0, "st": 12.0, "clock": 1.0}
    assert R.round_trips(p) == 2 + 8 + 1                     # values, lock words; locks one by one; clock
    ph = p[3:3 + p[2]]
    atoms = [c for c in ph if c & 0xff == R.ATOM_L]
    assert [(c >> 8) & 0xff for c in atoms] == [1] * 8 and [c >> 16 for c in atoms] == list(range(8))
    p_hv = R.programs_from_stats("ra", st, paired=False, mode="hv", prelock=True, pipelined=False)
    assert R.op_counts(p_hv)["ld"] == 12.0
    # fractional mean reads (HT chains): two programs reproduce the mean exactly
    st = dict(commits=0, commits_ro=4, reads_update=0, reads_ro=10, writes_update=0, locks_update=0)
    p = R.programs_from_stats("ht", st, paired=False, mode="hv", prelock=False, pipelined=True)
    assert p[0] == 2 and abs(R.op_counts(p)["ld"] - 2 * 2.5) < 1e-3
    # record addressing (k-means: one serial chain per record)
    st = dict(commits=5, commits_ro=0, reads_update=85, reads_ro=0, writes_update=85, locks_update=85)
    p = R.programs_from_stats("km", st, paired=False, mode="hv", prelock=True, pipelined=False, records=(1024, 17))
    assert p[0] == 1 | R.RECORDS and p[1:3] == [1024, 17]
    assert R.op_counts(p)["atom"] == 17.0
    assert R.op_counts(p)["ld"] == 0.0                        # the lock-holding critical section only
    assert p[3 + 2] & 0xff == R.ATOM_L
    # the gated round (lock_pipeline_gated): the lowest lock alone, then the other 16 at once
    p = R.programs_from_stats("km", st, paired=False, mode="hv", prelock=True, pipelined="gated", records=(1024, 17))
    atoms = [c for c in p[5:5 + p[4]] if c & 0xff == R.ATOM_L]
    assert [((c >> 8) & 0xff, c >> 16) for c in atoms] == [(1, 0), (16, 1)]
    assert R.op_counts(p)["atom"] == 17.0


def test_bench_self_launches_n_ranks_with_gloo():
    """`python bench.py --gpus 2` without a torchrun environment re-launches
    itself as 2 ranks (torch.distributed.run); --host-selftest swaps the GPU
    steps for fake counts so the host logic runs here on CPU with gloo: shard
    seeds, barriers, the one SUM/MAX reduction, the aggregate value and the
    communicator size in the JSON line."""
    import json
    import subprocess
    import sys
    env = {k: v for k, v in os.environ.items() if k not in ("WORLD_SIZE", "RANK", "LOCAL_RANK")}
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2", "--host-selftest",
                        "--steps", "4", "--warmup", "3"], capture_output=True, text=True, env=env, timeout=300)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout                          # rank 0 only
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["comm"] == {"backend": "gloo", "nranks": 2} and "selftest" in d
    n = (1 << 20) * 16
    assert d["stats"]["commits"] == 2 * (n - n // 16)         # SUM over ranks
    assert abs(d["ms_per_step"] - 1.5) < 1e-9                 # MAX over ranks (rank 1: 1.5 ms per step)
    assert abs(d["value"] - 2 * n / (4 * 1.5e-3)) < 1.0
    assert d["invariant_total_balance_ok"]
