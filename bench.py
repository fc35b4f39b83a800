#!/usr/bin/env python
"""Benchmark of the GPU-STM hot path (BASELINE.json metric: committed
transactions/sec + abort ratio vs the coarse-lock baseline, 1 B200).

One "step" = one gstm_launch of the whole hot path (TXBegin / TXRead /
TXWrite / TXCommit of every transaction) over one batch of synthetic input:
BASELINE configs[1], bank transfer, 2^20 accounts, 2^20 STM threads x 16
transactions (16M transactions), 2^20 version locks, STM-Optimized mode
(AUTO -> TBV).  The heap is resident in HBM before the timed region;
L2 is flushed (256 MiB write) between timed steps.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl reference]

N > 1 (torchrun, one rank per GPU): key-partitioned bank -- every rank owns
its own 2^20 accounts and runs shard-local transfers (weak scaling); NCCL is
used once, after timing, to reduce the stats and the balance invariant.

Prints ONE JSON line on rank 0.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "committed transactions/sec + abort ratio vs coarse-lock baseline, 1 B200"
UNIT = "tx/s"
ACCOUNTS = 1 << 20
THREADS = 1 << 20
TX_PER_THREAD = 16
BITS = 20
SEED = 20140215


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="native", choices=["native", "reference"])
    ap.add_argument("--mode", default="hv", help="headline STM mode (hv: see DESIGN.md §7.3; auto = the "
                                                 "paper's STM-Optimized rule, also reported)")
    ap.add_argument("--threads", type=int, default=THREADS)
    ap.add_argument("--tx-per-thread", type=int, default=TX_PER_THREAD)
    ap.add_argument("--no-cgl", action="store_true", help="skip the CGL/FGL baselines")
    ap.add_argument("--no-cpu", action="store_true", help="skip the cpu_baseline leg")
    return ap.parse_args()


def shard_seed(rank: int) -> int:
    """Key-partitioned bank: rank r owns its own 2^20 accounts (its own heap
    on its own GPU) and generates shard-local transfers from this seed."""
    return SEED + 1000003 * rank


def reduce_over_ranks(stats_vec, balance, t_ms, wall, world, dist, device):
    """The only collective of the run (after timing): SUM of the per-rank
    stats vector and total balance, MAX of the timed milliseconds and wall
    seconds.  float64 holds every count exactly (< 2^53)."""
    import torch
    vec = torch.tensor(list(stats_vec) + [balance], dtype=torch.float64, device=device)
    tm = torch.tensor([t_ms, wall], dtype=torch.float64, device=device)
    if world > 1:
        dist.all_reduce(vec, op=dist.ReduceOp.SUM)
        dist.all_reduce(tm, op=dist.ReduceOp.MAX)
    return vec.cpu().numpy(), tm.cpu().tolist()


def config(args, mode_used="tbv"):
    return {
        "workload": "bank transfer (BASELINE configs[1]): 2-account transfer tx, total-balance invariant",
        "accounts_per_gpu": ACCOUNTS,
        "threads_per_gpu": args.threads,
        "tx_per_thread": args.tx_per_thread,
        "tx_per_step_per_gpu": args.threads * args.tx_per_thread,
        "lock_table_bits": BITS,
        "mode": f"{args.mode} -> {mode_used}",
        "partition": "key-partitioned shards, shard-local transfers" if args.gpus > 1 else "single shard",
        "l2": "flushed (256 MiB write) between timed steps",
    }


# ---------------------------------------------------------------------------
# reference arm: the CPU oracle as it stands (serial executor), rank 0 only
# ---------------------------------------------------------------------------
def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    import numpy as np
    import oracle as O

    p = O.params("bank", n_words=ACCOUNTS)
    sample_threads = min(args.threads, 1 << 18)          # bounded sample: 4M tx per step
    K = args.tx_per_thread
    heap = O.init_heap(p, ACCOUNTS)
    for _ in range(max(args.warmup, 0) and 1):
        O.serial(p, heap.copy(), sample_threads // 16, K, SEED)
    times = []
    n = sample_threads * K
    for s in range(args.steps):
        t0 = time.perf_counter()
        res, upd = O.serial(p, heap, sample_threads, K, SEED + s)
        times.append(time.perf_counter() - t0)
    tot = sum(times)
    val = n * args.steps / tot
    line = {
        "impl": "reference", "metric": METRIC, "value": val, "unit": UNIT, "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * tot / args.steps,
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u32",
        "data": "synthetic", "config": config(args, "serial"),
        "cpu_baseline": {"value": val, "unit": UNIT, "cores": 1, "kind": "oracle",
                         "sample": f"serial oracle (oracle/serial.c or_serial, gcc -O2, 1 thread) over "
                                   f"{sample_threads} threads x {K} tx = {n} bank transfers per step"},
        "e2e": {"value": val, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


# ---------------------------------------------------------------------------
# clocks sampling during the timed region
# ---------------------------------------------------------------------------
class ClockSampler:
    FIELDS = "clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown," \
             "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap"

    def __init__(self, dev: int):
        self.p = None
        self.dev = dev
        try:
            self.p = subprocess.Popen(["nvidia-smi", "-i", str(dev), f"--query-gpu={self.FIELDS}",
                                       "--format=csv,noheader,nounits", "-lms", "50"],
                                      stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except Exception:
            self.p = None

    def stop(self):
        if not self.p:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.p.terminate()
        out, _ = self.p.communicate(timeout=10)
        sm, mx, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for line in out.strip().splitlines():
            f = [x.strip() for x in line.split(",")]
            if len(f) < 6:
                continue
            try:
                sm.append(float(f[0]))
                mx.append(float(f[1]))
            except ValueError:
                continue
            for nm, v in zip(names, f[2:6]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        sm.sort()
        return {"sm_mhz": sm[len(sm) // 2] if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(sm)}


def measured_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            return json.load(f), "measured (MEASURED_PEAKS.json)"
    except Exception:
        return {"hbm_gbs": 6650.0}, "fallback (B200_PROFILING.md)"


class SM:
    """Stats bookkeeping, baselines and roofline arithmetic."""
    KEYS = ["commits", "commits_ro", "aborts", "aborts_opacity", "aborts_prevbv", "aborts_tbv",
            "aborts_commit_vbv", "aborts_lock", "lock_retries", "postvalidations", "vbv_runs", "spins",
            "attempts", "errors"]

    @staticmethod
    def stats_vector(st):
        import numpy as np
        v = np.zeros(16, dtype=np.float64)
        for i, k in enumerate(SM.KEYS):
            v[i] = getattr(st, k)
        v[14] = st.elapsed_ms
        return v

    @staticmethod
    def from_vector(v):
        d = {k: float(v[i]) for i, k in enumerate(SM.KEYS)}
        d["lib_elapsed_ms"] = float(v[14])
        return d

    # Algorithmic memory accesses of one bank transaction (Algorithm 3 on
    # the bank body, TBV mode, verify off), DESIGN.md §7.1.  Every access is
    # a random 4-byte word, i.e. one 32-byte sector moved between L2 and
    # the SM (and between HBM and L2 when not resident).
    UPD = {"ld": 4, "atom": 2, "st": 4}      # 2 values + 2 lock words; 2 lock atom.or; 2 write-back + 2 release
    UPD_HV = {"ld": 6, "atom": 2, "st": 4}   # + the pre-lock VBV of the 2 values (A3.l71)
    RO = {"ld": 4, "atom": 0, "st": 0}       # skipped transfer: values + lock words
    SECTOR = 32

    @staticmethod
    def upd(mode):
        return SM.UPD_HV if mode == "hv" else SM.UPD

    @staticmethod
    def roofline_bank(tot, t_ms, steps, peaks, peak_src, mode, traffic=None):
        acc_upd = sum(SM.upd(mode).values())
        acc_ro = sum(SM.RO.values())
        bytes_per_launch = (tot["commits"] * acc_upd + tot["commits_ro"] * acc_ro) * SM.SECTOR / steps
        dur_s = t_ms * 1e-3 / steps
        achieved = bytes_per_launch / dur_s / 1e9
        peak = float(peaks.get("hbm_gbs", 6650.0))
        prof = os.path.join(ROOT, "profiles", "r01_bank_ncu_full.json")
        if traffic is None and os.path.exists(prof):
            try:
                traffic = json.load(open(prof)).get("dram_bytes_per_launch")
            except Exception:
                traffic = None
        return {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
                "traffic": traffic, "kernel": f"stm_kernel<BankWL, MODE_{mode.upper()}>",
                "algorithmic_bytes_per_launch": bytes_per_launch,
                "bytes_per_unit": {"update_tx": acc_upd * SM.SECTOR, "read_only_tx": acc_ro * SM.SECTOR},
                "peak_source": peak_src,
                "note": "random 4 B accesses counted as 32 B sectors; launch duration = CUDA events on the "
                        "launching stream, averaged over the timed steps"}

    @staticmethod
    def roofline_l2_bank(G, tot, t_ms, steps, mode):
        """L2-atomic roofline: the same PTX operations, measured on this box by
        gstm_ubench over a table of the heap's size (4 MiB, L2-resident)."""
        upd = SM.upd(mode)
        threads = 148 * 2048
        A = G.gstm_ubench(0, 4 << 20, 1 << 26, threads)[0]      # random atom.or.b32
        L = G.gstm_ubench(2, 4 << 20, 1 << 26, threads)[0]      # random ld.relaxed.gpu
        S = G.gstm_ubench(3, 4 << 20, 1 << 26, threads)[0]      # random st.relaxed.gpu
        Cl = G.gstm_ubench(5, 256, 1 << 24, threads)[0]         # warp-aggregated clock increments
        per = lambda m: m["ld"] / L + m["atom"] / A + m["st"] / S
        roof_s = (tot["commits"] * (per(upd) + 1.0 / Cl) + tot["commits_ro"] * per(SM.RO)) / steps
        dur_s = t_ms * 1e-3 / steps
        return {"bound": "l2_atomic", "frac": roof_s / dur_s,
                "roof_tx_per_s": (tot["commits"] + tot["commits_ro"]) / steps / roof_s,
                "achieved_tx_per_s": (tot["commits"] + tot["commits_ro"]) / steps / dur_s,
                "peaks_ops_per_s": {"atom_or_random_4MiB": A, "ld_relaxed_random_4MiB": L,
                                    "st_relaxed_random_4MiB": S, "clock_increments_warp_aggregated": Cl},
                "ops_per_update_tx": dict(upd, clock=1), "ops_per_read_only_tx": SM.RO,
                "model": "time = sum over op classes of count / measured rate (one shared L2 request pipeline)"}

    @staticmethod
    def baselines(G, stream, accounts, bits, T, seed):
        out = {}
        # CGL: serialised, so its rate does not depend on the batch size; time a
        # bounded sample (same thread count, 1 tx each, fewer threads if slow).
        g = G.Gstm(accounts, bits)
        g.set_workload_defaults("bank", n_words=accounts)
        g.set_mode("cgl")
        g.set_stream(stream)
        g.init_heap("bank")
        # CGL serialises every transaction, so its rate depends on how many
        # threads fight for the one lock, not on the batch size.  Probe the
        # paper's Scheme #3 (backoff 0) and test-and-test-and-set with
        # exponential backoff at several thread counts and divide by the
        # FASTEST (the most favourable baseline), then time it on a bounded
        # sample of ~0.5 s.
        probes = {}
        for Tc in (148 * 32, 1 << 14, 1 << 16, 1 << 18):
            for bo in (0, 256):
                g.set_params(backoff_ns=bo)
                probes[(Tc, bo)] = g.run("bank", Tc, max(1, (1 << 14) // Tc), seed + 11 + bo).tx_per_s
        (Tc, bo) = max(probes, key=probes.get)
        g.set_params(backoff_ns=bo)
        Kc = max(1, int(probes[(Tc, bo)] * 0.5) // Tc)
        st = g.run("bank", Tc, Kc, seed + 12)
        out["cgl"] = {"value": st.tx_per_s, "unit": UNIT, "threads": Tc, "tx_per_thread": Kc, "backoff_ns": bo,
                      "probe_tx_per_s": {f"T={k[0]},backoff={k[1]}": v for k, v in probes.items()},
                      "sample": f"{Tc} threads x {Kc} tx at the fastest probed CGL configuration",
                      "elapsed_ms": st.elapsed_ms, "kernel": "cgl_kernel<BankWL>"}
        g.set_params(backoff_ns=0)
        g.set_mode("fgl")
        g.run("bank", T, 16, seed + 13)
        st = g.run("bank", T, 16, seed + 14)
        out["fgl"] = {"value": st.tx_per_s, "unit": UNIT, "sample": f"{T} threads x 16 tx (full step)",
                      "abort_ratio": 0.0, "lock_retries": st.lock_retries, "kernel": "fgl_kernel<BankWL>"}
        g.close()
        return out

    @staticmethod
    def mode_table(G, stream, flush, accounts, bits, T, K, seed, modes, steps=8, warmup=3):
        """The same timed loop (events per launch, L2 flushed between
        launches, no host sync) for the other concurrency-control modes."""
        import torch
        out = {}
        for mode in modes:
            g = G.Gstm(accounts, bits)
            g.set_workload_defaults("bank", n_words=accounts)
            g.set_mode(mode)
            g.set_stream(stream)
            g.init_heap("bank")
            for w in range(warmup):
                g.launch("bank", T, K, seed + 500 + w)
            torch.cuda.synchronize()
            g.reset_stats_total()
            evs = []
            for k in range(steps):
                flush.fill_(float(k))
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record(stream)
                g.launch("bank", T, K, seed + 600 + k)
                b.record(stream)
                evs.append((a, b))
            torch.cuda.synchronize()
            ms = sum(a.elapsed_time(b) for a, b in evs)
            st, _ = g.stats_total()
            done = st.commits + st.commits_ro
            out[mode] = {"value": done / (ms * 1e-3), "unit": UNIT, "ms_per_step": ms / steps,
                         "abort_ratio": st.aborts / max(1, st.aborts + done),
                         "mode_used": G.MODE_NAMES[st.mode_used]}
            g.close()
        return out

    @staticmethod
    def cpu_baseline(accounts, T, K, seed):
        import oracle as O
        p = O.params("bank", n_words=accounts)
        heap = O.init_heap(p, accounts)
        Ts = T                     # the full step: T x K transfers
        t0 = time.perf_counter()
        O.serial(p, heap, Ts, K, seed)
        dt = time.perf_counter() - t0
        return {"value": Ts * K / dt, "unit": UNIT, "cores": 1, "kind": "oracle",
                "sample": f"serial oracle (oracle/serial.c or_serial, gcc -O2, 1 thread) over one full step: "
                          f"{Ts} threads x {K} tx = {Ts * K} bank transfers, {dt:.2f} s"}


# ---------------------------------------------------------------------------
# native arm
# ---------------------------------------------------------------------------
def run_native(args):
    import numpy as np
    import torch
    import torch.distributed as dist

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world != args.gpus:
        args.gpus = world
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)

    from paper_conf_cgo_xuwglgq14_b200 import build as B
    if rank == 0 or world == 1:
        B.build()
    if world > 1:
        dist.barrier()
    from paper_conf_cgo_xuwglgq14_b200 import gstm as G

    T, K = args.threads, args.tx_per_thread
    # one non-default stream for everything (the library, the L2 flush, the
    # CUDA events): torch's legacy default stream has handle 0, which the C
    # ABI reads as "use the handle's private stream"
    stream = torch.cuda.Stream(device=dev)
    torch.cuda.set_stream(stream)
    g = G.Gstm(ACCOUNTS, BITS)
    g.set_workload_defaults("bank", n_words=ACCOUNTS)
    g.set_mode(args.mode)
    g.set_stream(stream)
    heap = torch.empty(ACCOUNTS, dtype=torch.int32, device=dev)
    g.attach_heap(heap)
    g.init_heap("bank")
    flush = torch.empty(64 << 20, dtype=torch.float32, device=dev)    # 256 MiB > 126 MB L2
    seed0 = shard_seed(rank)

    def step(k):
        g.launch("bank", T, K, seed0 + k)

    for w in range(args.warmup):
        step(100000 + w)
    torch.cuda.synchronize()

    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    g.reset_stats_total()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    sampler = ClockSampler(local)
    time.sleep(0.2)
    wall0 = time.perf_counter()
    # K steps enqueued back to back (no host sync inside the timed region);
    # each step bracketed by events, the L2 flush between steps outside them
    for k in range(args.steps):
        flush.fill_(float(k))
        e0, e1 = evs[k]
        e0.record(stream)
        step(k)
        e1.record(stream)
    torch.cuda.synchronize()
    wall = time.perf_counter() - wall0
    st_tot, n_launch = g.stats_total()
    assert n_launch == args.steps
    agg = SM.stats_vector(st_tot)
    if world > 1:
        dist.barrier()
    clocks = sampler.stop()
    step_ms = [a.elapsed_time(b) for a, b in evs]
    t_ms = float(sum(step_ms))
    mode_used = G.MODE_NAMES[g.stats().mode_used]

    # NCCL: one all-reduce of the stats and invariants (SUM), one of the time (MAX)
    bal = float(heap.to(torch.int64).sum().item())
    vec, (t_ms, wall) = reduce_over_ranks(agg, bal, t_ms, wall, world, dist, dev)
    tot = SM.from_vector(vec[:16])
    balance_ok = int(vec[16]) == world * ACCOUNTS * 1000

    extra = {}
    if rank == 0:
        # e2e through the C ABI with HOST buffers (H2D + launch + D2H timed)
        pin_in = torch.full((ACCOUNTS,), 1000, dtype=torch.int32).pin_memory()
        pin_out = torch.empty(ACCOUNTS, dtype=torch.int32).pin_memory()
        h_in = pin_in.numpy().view(np.uint32)
        h_out = pin_out.numpy().view(np.uint32)
        g2 = G.Gstm(ACCOUNTS, BITS)
        g2.set_workload_defaults("bank", n_words=ACCOUNTS)
        g2.set_mode(args.mode)
        g2.set_stream(stream)
        g2.run_host("bank", h_in, h_out, T, K, seed0)        # warm-up
        e2e_ms, e2e_done = 0.0, 0
        n_e2e = max(3, min(args.steps, 10))
        for k in range(n_e2e):
            flush.fill_(float(k))
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(stream)
            st2 = g2.run_host("bank", h_in, h_out, T, K, seed0 + 7 + k)
            b.record(stream)
            b.synchronize()
            e2e_ms += a.elapsed_time(b)
            e2e_done += st2.commits + st2.commits_ro
        extra["e2e"] = {"value": e2e_done / (e2e_ms * 1e-3), "unit": UNIT,
                        "h2d_bytes_per_step": ACCOUNTS * 4, "d2h_bytes_per_step": ACCOUNTS * 4 + 184}
        g2.close()
        if not args.no_cgl:
            extra.update(SM.baselines(G, stream, ACCOUNTS, BITS, T, seed0))
            extra["modes"] = SM.mode_table(G, stream, flush, ACCOUNTS, BITS, T, K, seed0,
                                           [m for m in ("auto", "tbv", "hv", "fgl") if m != args.mode])
        # roofline of the dominant kernel (stm_kernel<BankWL, TBV>)
        peaks, peak_src = measured_peaks()
        extra["roofline"] = SM.roofline_bank(tot, t_ms, args.steps, peaks, peak_src, mode_used)
        extra["roofline_l2"] = SM.roofline_l2_bank(G, tot, t_ms, args.steps, mode_used)
        if world == 1 and not args.no_cpu:
            extra["cpu_baseline"] = SM.cpu_baseline(ACCOUNTS, T, K, SEED)

    done = tot["commits"] + tot["commits_ro"]
    if rank == 0:
        value = done / (t_ms * 1e-3)
        line = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": t_ms / args.steps, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
            "config": config(args, mode_used),
            "abort_ratio": tot["aborts"] / max(1.0, tot["aborts"] + done),
            "stats": {k: int(v) for k, v in tot.items()},
            "invariant_total_balance_ok": bool(balance_ok),
            "clocks": clocks,
            "gpu_launches": 3 * args.steps,
            "wall_s_timed_region": wall,
        }
        if "cgl" in extra:
            line["speedup_vs_cgl"] = value / world / extra["cgl"]["value"]
        line.update(extra)
        print(json.dumps(line), flush=True)
    g.close()
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    return 0


def main():
    args = parse()
    if args.impl == "reference":
        return run_reference(args)
    return run_native(args)


if __name__ == "__main__":
    sys.exit(main())
