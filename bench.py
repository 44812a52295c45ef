#!/usr/bin/env python3
"""bench.py — records/s and HBM GB/s of the SASSI handler fold on B200 (BASELINE.json metric).

N = 1 (default): config c3 of BASELINE.json (the largest configuration that fits one GPU): an
SGEMM/stencil-shaped trace of 10^8 warp-instruction records (~19 GB in HBM, >> the 126 MB L2, so
no flush is needed between steps), all four handlers attached. One step = the whole hot path:
sassi_reset (CUPTI launch-callback analogue) + sassi_consume (fused fold) + sassi_sample_sites
(1,000 injection sites, L629).

N > 1: config c5, the configuration the metric quotes for 8 GPUs: ~4x10^9 records in 8 warp shards,
strong scaling (the total is fixed; rank r folds shards r, r+N, ...), the per-rank tables merged
by sassi_merge (one NCCL allreduce) before the 1,000 draws. The line carries c5's 1-GPU time T_1
(rank 0 alone folds all 8 shards afterwards, same protocol) so E_N = T_1 / (N T_N) can be formed,
and a weak-scaling secondary (every rank folds its own c3-shaped 10^8-record shard + the merge).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl reference] [--workload c2|c3|c4|c5]

--gpus N without torchrun re-launches this script under torch.distributed.run with N ranks (one
per GPU, rendezvous on 127.0.0.1). --impl reference times the oracle (plain single-threaded C++,
oracle/) on the host cores on a bounded sample of the same workload — the only reference
implementation this tier has.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "warp-instr records/sec & HBM GB/s (% peak) at 1/2/4/8 B200; instrumented slowdown"
SPEC_HBM_GBS = 8000.0
N_DRAWS = 1000


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--workload", default=None, choices=["c2", "c3", "c4", "c5"],
                    help="default: c3 at N = 1, c5 at N > 1")
    ap.add_argument("--selftest-dist", action="store_true",
                    help="launch / rendezvous / max-over-ranks plumbing only (gloo without a GPU)")
    ap.add_argument("--merge", default="nccl", choices=["nccl", "p2p"],
                    help="N > 1: sassi_merge over NCCL after the fold, or the fused fold + merge over "
                         "peer memory (every rank's fold also updates the other ranks' images)")
    ap.add_argument("--share-gpu", action="store_true",
                    help="N > 1 ranks all on cuda:0 (gloo process group, --merge p2p; c2 / c3 / c4): "
                         "the multi-rank code path on a one-GPU box, not a scaling measurement")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-slowdown", action="store_true")
    ap.add_argument("--no-injection", action="store_true")
    return ap.parse_args()


def dist_env():
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return rank, world, local


def self_launch(n):
    """`--gpus N` outside torchrun: run this script under torch.distributed.run with N ranks on this
    node (rendezvous on 127.0.0.1, a free port); returns its exit code. Rank 0 prints the line."""
    import socket
    import subprocess
    with socket.socket() as so:
        so.bind(("127.0.0.1", 0))
        port = so.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=%d" % n,
           "--master-addr=127.0.0.1", "--master-port=%d" % port, os.path.abspath(__file__)] + sys.argv[1:]
    return subprocess.call(cmd)


def max_over_ranks(x, dev=None):
    """Maximum of a float over all ranks (device timing rule: the job time is the slowest rank's)."""
    import torch
    import torch.distributed as dist
    if not (dist.is_available() and dist.is_initialized()):
        return x
    t = torch.tensor([float(x)], dtype=torch.float64, device=dev)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def sum_over_ranks(x, dev=None):
    import torch
    import torch.distributed as dist
    if not (dist.is_available() and dist.is_initialized()):
        return x
    t = torch.tensor([int(x)], dtype=torch.int64, device=dev)
    dist.all_reduce(t)
    return int(t.item())


def host_info():
    """nproc and the CPU model of the box the oracle baseline runs on."""
    model = None
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                model = line.split(":", 1)[1].strip()
                break
    except OSError:
        pass
    return {"nproc": os.cpu_count(), "cpu_model": model}


def run_selftest_dist(args, rank, world):
    """The multi-rank plumbing of this script without a GPU: process group (nccl with CUDA, else
    gloo), barrier, a per-rank timing reduced as the maximum over ranks, one line from rank 0."""
    import torch
    import torch.distributed as dist
    backend = "nccl" if torch.cuda.is_available() else "gloo"
    dev = None
    if backend == "nccl":
        torch.cuda.set_device(int(os.environ.get("LOCAL_RANK", "0")))
        dev = torch.device("cuda", torch.cuda.current_device())
    if world > 1:
        dist.init_process_group(backend)
        dist.barrier()
    t0 = time.perf_counter()
    time.sleep(0.01 * (rank + 1))
    el = max_over_ranks(time.perf_counter() - t0, dev)
    ranks = sum_over_ranks(1, dev)
    if rank == 0:
        print(json.dumps({"selftest": "dist", "n_gpus": world, "ranks_reporting": ranks,
                          "backend": backend if world > 1 else "none", "max_over_ranks_s": el}),
              flush=True)
    if world > 1:
        dist.destroy_process_group()


def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md, 6.65 TB/s)"


def ncu_traffic(workload):
    """dram read+write bytes per consume launch from the committed ncu --set full capture."""
    p = os.path.join(ROOT, "profiles", "ncu_consume_%s.json" % workload)
    if os.path.exists(p):
        try:
            return float(json.load(open(p))["dram_bytes_per_launch"])
        except Exception:
            return None
    return None


class ClockSampler:
    """Samples SM clock + throttle reasons with NVML during the timed region."""

    REASONS = {0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap",
               0x8: "hw_slowdown", 0x10: "sync_boost", 0x20: "sw_thermal_slowdown",
               0x40: "hw_thermal_slowdown", 0x80: "hw_power_brake_slowdown",
               0x100: "display_clock_setting"}

    def __init__(self, index):
        self.samples, self.reasons, self.stop_ev = [], 0, threading.Event()
        self.max_mhz = None
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
        except Exception:
            self.nv = None

    def _run(self):
        while not self.stop_ev.is_set():
            try:
                self.samples.append(self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM))
                self.reasons |= int(self.nv.nvmlDeviceGetCurrentClocksEventReasons(self.h))
            except Exception:
                pass
            time.sleep(0.005)

    def __enter__(self):
        if self.nv:
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        return self

    def __exit__(self, *a):
        self.stop_ev.set()
        if self.nv:
            self.t.join()

    def result(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": ["unavailable"]}
        names = [n for b, n in self.REASONS.items() if self.reasons & b and n != "gpu_idle"]
        return {"sm_mhz": statistics.median(self.samples), "sm_max_mhz": self.max_mhz,
                "reasons": names, "samples": len(self.samples)}


def workload_program(name, world):
    from paper_conf_isca_stephensonhlejn15_b200 import gen
    P, limit, _, desc = gen.preset(name)
    P.total_warps = P.total_warps * world  # weak scaling: each rank owns one shard of warps
    return P, limit, desc


def algorithmic_bytes(rec, handlers):
    """16 B per header + 256 B per addr row of a GLOBAL memory site (memdiv attached) + 128 B per
    val row (value attached) — counted from the stream."""
    import torch
    from paper_conf_isca_stephensonhlejn15_b200 import gen
    sites = rec["sites"]
    glob = [int(s["pc"]) for s in sites if (int(s["flags"]) & gen.F_MEM) and int(s["domain"]) == 0]
    pcs = rec["hdr"][:, 0]
    n_glob = int(torch.isin(pcs, torch.tensor(np.array(glob, np.int64).astype(np.int32),
                                              device=pcs.device)).sum().item()) if glob else 0
    b = 16 * rec["n"]
    if handlers & 2:
        b += 256 * n_glob
    if handlers & 4:
        b += 128 * rec["n_val_rows"]
    return b, n_glob


def run_reference(args, rank, world, workload):
    """Oracle on the host cores, on a bounded sample of the same workload (rank 0 only; under
    torchrun the other ranks exit without work)."""
    if rank != 0:
        return
    import oracle
    from paper_conf_isca_stephensonhlejn15_b200 import gen
    P, limit, desc = workload_program(workload, 1)
    mask = gen.PRESETS[workload][2]
    sample_n = 1 << 21
    rec = gen.generate_host(P, sample_n, 0, 1024)
    times = []
    for i in range(args.warmup + args.steps):
        t0 = time.perf_counter()
        oracle.run(rec["sites"], P.total_warps, mask, rec["hdr"], rec["addr"], rec["val"])
        if i >= args.warmup:
            times.append(time.perf_counter() - t0)
    tmax = max(sum(times), 1e-9)
    v = args.steps * rec["n"] / tmax
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": "records/s",
            "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": 1e3 * tmax / args.steps, "higher_is_better": True,
            "scaling": "weak" if world == 1 else "strong", "vs_baseline": None, "dtype": "u32",
            "data": "synthetic",
            "config": {"workload": workload + ": " + desc, "sample_records": rec["n"]},
            "cpu_baseline": dict({"value": v, "unit": "records/s", "cores": 1, "threads": 1,
                                  "kind": "oracle",
                                  "sample": "first %d records (warps 0..1023) of %s per step" %
                                            (rec["n"], workload)}, **host_info()),
            "e2e": {"value": v, "unit": "records/s", "h2d_bytes_per_step": 0,
                    "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def cpu_baseline(args, d_rec, mask, P):
    """The oracle as it stands, single-threaded, timed for ~10 s on a bounded sample (rank 0, N=1):
    the first 2^23 records of the same stream, copied to the host, folded repeatedly."""
    import oracle
    from paper_conf_isca_stephensonhlejn15_b200 import gen
    n = min(1 << 23, d_rec["n"] // 256 * 256)
    pre_cb = d_rec["chunk_base"][n // 256].cpu().numpy().view(np.uint64)
    pre = dict(d_rec, hdr=d_rec["hdr"][:n], addr=d_rec["addr"][: int(pre_cb[0])],
               val=d_rec["val"][: int(pre_cb[1])], n=n, n_addr_rows=int(pre_cb[0]),
               n_val_rows=int(pre_cb[1]))
    h = gen.to_host(pre)
    t0 = time.perf_counter()
    reps = 0
    while True:
        oracle.run(h["sites"], P.total_warps, mask, h["hdr"], h["addr"], h["val"])
        reps += 1
        el = time.perf_counter() - t0
        if el > 10.0 or reps >= 30:
            break
    return dict({"value": reps * n / el, "unit": "records/s", "cores": 1, "threads": 1,
                 "kind": "oracle",
                 "sample": "first %d records of the %s stream, %d repetition(s), %.1f s" %
                           (n, args.workload, reps, el)}, **host_info())


def nccl_comm(world, rank, local, dev):
    """A communicator of libsassi's own (its NCCL), the unique id broadcast over torch.distributed."""
    import torch
    import torch.distributed as dist
    from paper_conf_isca_stephensonhlejn15_b200 import sassi
    uid = torch.zeros(128, dtype=torch.uint8, device=dev)
    if rank == 0:
        uid.copy_(torch.frombuffer(bytearray(sassi.sassi_nccl_get_unique_id()), dtype=torch.uint8))
    if dist.is_initialized():
        dist.broadcast(uid, 0)
    return sassi.sassi_nccl_comm_create(world, rank, bytes(uid.cpu().numpy()), local)


def fold_c5_shards(args, shards, P, mask, dev, local, job=None):
    """Fold c5 warp shards one by one into `job` (a Context, created if None): each shard is
    generated in HBM (untimed), warmed up, timed over --steps passes of reset + consume on a scratch
    context (CUDA events on the launching stream), then folded once more into the job.
    -> (job, per-shard mean consume ms, records, algorithmic bytes, records of the first shard)."""
    import torch
    from paper_conf_isca_stephensonhlejn15_b200 import gen, sassi
    stream = torch.cuda.current_stream(dev)
    scratch = None
    consume_ms, n_total, alg_total, n_first = [], 0, 0, None
    for shard in shards:
        rec = gen.generate_device(P, None, shard * 16384, 16384, device=dev)
        if job is None:
            job = sassi.Context(rec["sites"], P.total_warps, mask, device=local)
        if scratch is None:
            scratch = sassi.Context(rec["sites"], P.total_warps, mask, device=local)
        b, _ = algorithmic_bytes(rec, mask)
        for _ in range(args.warmup):
            scratch.reset(stream)
            scratch.consume(rec, stream=stream)
        evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
               for _ in range(args.steps)]
        for a, e in evs:
            scratch.reset(stream)
            a.record(stream)
            scratch.consume(rec, stream=stream)
            e.record(stream)
        job.consume(rec, stream=stream)
        torch.cuda.synchronize(dev)
        consume_ms.append(statistics.mean(a.elapsed_time(e) for a, e in evs))
        n_total += rec["n"]
        alg_total += b
        n_first = rec["n"] if n_first is None else n_first
        del rec
        torch.cuda.empty_cache()
    scratch.close()
    return job, consume_ms, n_total, alg_total, n_first


def run_c5(args, rank, world, local):
    """Config c5 as the metric quotes it: ~4x10^9 records in 8 warp shards of 16,384 warps. Rank r
    folds shards r, r+N, ... (strong scaling: the total is fixed); the job time is the sum over the
    rank's shards of the timed fold + the NCCL merge (N > 1) + the final 1,000-site sampling, max
    over ranks. At N > 1 rank 0 then folds all 8 shards alone (same protocol: T_1) and every rank
    runs the c3 weak-scaling measurement (secondary key)."""
    import torch
    import torch.distributed as dist
    from paper_conf_isca_stephensonhlejn15_b200 import gen
    dev = torch.device("cuda", local)
    P, limit, mask, desc = gen.preset("c5")
    stream = torch.cuda.current_stream(dev)
    # the N > 1 parts (merge, T_1, weak scaling) also run at N = 1 with SASSI_BENCH_SCALING_EXTRAS=1
    # (a 1-rank communicator), so the multi-GPU code path is exercised on a one-GPU box
    multi = world > 1 or os.environ.get("SASSI_BENCH_SCALING_EXTRAS") == "1"
    comm = nccl_comm(world, rank, local, dev) if multi else None

    def barrier():
        if dist.is_initialized():
            dist.barrier()

    draws = torch.empty(N_DRAWS * 32, dtype=torch.uint8, device=dev)
    status = torch.zeros(1, dtype=torch.int32, device=dev)
    # the job's context, set up untimed: a merge of its empty tables (the identity: every rank
    # keeps empty tables) allocates the packed image and runs the one host-checked checksum
    # comparison; a sampling call on zero counts allocates the scan buffers (status 1, no draws)
    from paper_conf_isca_stephensonhlejn15_b200 import sassi
    job = sassi.Context(P.sites(), P.total_warps, mask, device=local)
    if comm is not None:
        job.merge(comm, stream)
    job.sample_device(draws, status, N_DRAWS, 20150617, stream)
    torch.cuda.synchronize(dev)
    with ClockSampler(local) as clk:
        job, consume_ms, n_total, alg_total, n_first = fold_c5_shards(args, range(rank, 8, world), P,
                                                                      mask, dev, local, job=job)
        barrier()
        t0, t1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        t0.record(stream)
        if comm is not None:
            job.merge(comm, stream)
        job.sample_device(draws, status, N_DRAWS, 20150617, stream)
        t1.record(stream)
        torch.cuda.synchronize(dev)
    assert int(status.item()) == 0, "c5: nothing to sample"
    t_tail = t0.elapsed_time(t1) / 1e3
    t_shards = sum(consume_ms) / 1e3
    t_job = max_over_ranks(t_shards + t_tail, dev)
    # weak scaling at a fixed ~5x10^8 records per GPU: every rank's first shard
    # (shard r) + the merge and the draws, max over ranks
    t_weak = max_over_ranks(consume_ms[0] / 1e3 + t_tail, dev)
    n_weak = sum_over_ranks(n_first, dev)
    n_total = sum_over_ranks(n_total, dev)
    alg_total = sum_over_ranks(alg_total, dev)
    launches = job.kernel_launches()
    n_sites = len(job.sites)
    job.close()
    t1_job = t1_shard_ms = None
    weak = None
    if multi:
        barrier()
        if rank == 0:  # T_1: the same job on one GPU (all 8 shards, no merge)
            j1 = sassi.Context(P.sites(), P.total_warps, mask, device=local)
            j1.sample_device(draws, status, N_DRAWS, 20150617, stream)  # scan buffers, untimed
            j1, ms1, _, _, _ = fold_c5_shards(args, range(8), P, mask, dev, local, job=j1)
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(stream)
            j1.sample_device(draws, status, N_DRAWS, 20150617, stream)
            b.record(stream)
            torch.cuda.synchronize(dev)
            t1_job = sum(ms1) / 1e3 + a.elapsed_time(b) / 1e3
            t1_shard_ms = ms1
            j1.close()
        barrier()
        weak = run_weak(args, rank, world, local, "c3", extras=False, comm=comm,
                        steps=min(args.steps, 10))
    if comm is not None:
        from paper_conf_isca_stephensonhlejn15_b200 import sassi
        sassi.sassi_nccl_comm_destroy(comm)
    if rank == 0:
        peak, peak_src = measured_peaks()
        per_gpu_alg = alg_total / world
        line = {"metric": METRIC, "value": n_total / t_job, "unit": "records/s", "n_gpus": world,
                "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * t_job,
                "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "u32",
                "data": "synthetic",
                "config": {"workload": "c5: " + desc + " (8 warp shards of 16,384 warps, folded "
                           "shard by shard; step = all shards + merge + 1000-site sampling)",
                           "records": n_total, "sites": n_sites,
                           "threads": 32 * P.total_warps, "handlers": mask,
                           "algorithmic_bytes": alg_total,
                           "l2": "each shard is ~90 GB >> 126 MB L2; no flush",
                           "parallelism": "dp%d over warp shards%s" % (
                               world, ", NCCL allreduce merge" if world > 1 else "")},
                "hbm_gbs": alg_total / t_job / 1e9,
                "hbm_frac_of_spec_8tbs": per_gpu_alg / t_job / 1e9 / SPEC_HBM_GBS,
                "roofline": {"bound": "hbm", "kernel": "consume_kernel<%d>" % mask,
                             "achieved": per_gpu_alg / t_shards / 1e9, "peak": peak, "unit": "GB/s",
                             "frac": per_gpu_alg / t_shards / 1e9 / peak, "peak_source": peak_src,
                             "traffic": ncu_traffic("c5"), "consume_ms_per_shard": consume_ms},
                "gpu_launches": launches, "clocks": clk.result()}
        if multi:
            line["strong_scaling"] = {
                "t1_ms": 1e3 * t1_job, "tN_ms": 1e3 * t_job, "t1_consume_ms_per_shard": t1_shard_ms,
                "note": "T_1 = rank 0 alone folding all 8 shards + sampling, same protocol, same run; "
                        "E_N = T_1 / (N T_N) (north_star target >= 0.85)"}
        line["weak_scaling_c5"] = {
            "value": n_weak / t_weak, "unit": "records/s", "records_per_gpu": n_weak // world,
            "ms": 1e3 * t_weak,
            "note": "one c5 shard (~5x10^8 records) per GPU: each rank's first shard + merge + draws, "
                    "max over ranks (SURVEY §8d weak scaling at a fixed 5x10^8 records per GPU)"}
        if weak:
            line["weak_scaling"] = weak
            if "e2e" in weak:
                line["e2e"] = dict(weak["e2e"], note=weak["e2e"]["note"] + " (c3-shaped shard per rank: "
                                   "c5's records never exist in host memory at once)")
        print(json.dumps(line), flush=True)


def run_weak(args, rank, world, local, workload, extras=True, comm=None, steps=None):
    """`workload` (c2 / c3 / c4), each rank folding its own shard of the preset's size (weak scaling:
    warp ids offset by rank), + the NCCL merge when N > 1, + 1,000 draws. Returns the JSON line on
    rank 0 (None elsewhere); extras = e2e, cpu_baseline, slowdown, online trace, injection."""
    import torch
    import torch.distributed as dist
    from paper_conf_isca_stephensonhlejn15_b200 import gen, sassi

    dev = torch.device("cuda", local)
    steps = args.steps if steps is None else steps
    launched = dist.is_initialized()
    merge_on = world > 1 or comm is not None or os.environ.get("SASSI_BENCH_FORCE_MERGE") == "1"
    P, limit, desc = workload_program(workload, world)
    mask = gen.PRESETS[workload][2]
    per = P.total_warps // world
    rec = gen.generate_device(P, limit, rank * per, per, device=dev)
    n = rec["n"]
    alg_bytes, n_glob = algorithmic_bytes(rec, mask)
    ctx = sassi.Context(rec["sites"], P.total_warps, mask, device=local)
    own_comm = None
    p2p = getattr(args, "merge", "nccl") == "p2p" and world > 1
    if p2p:  # fused fold + merge: every rank's flush also updates the other ranks' images
        handles = [None] * world
        dist.all_gather_object(handles, ctx.ipc_table_handle())
        for j in range(world):
            if j != rank:
                ctx.add_peer_table(handles[j])
    elif merge_on and comm is None:
        comm = own_comm = nccl_comm(world, rank, local, dev)
    stream = torch.cuda.current_stream(dev)
    sample = bool(mask & 8)
    # draws stay on the device inside the timed steps (stream-ordered, no host round trip per step)
    draws = torch.empty(N_DRAWS * 32, dtype=torch.uint8, device=dev)
    draw_status = torch.zeros(1, dtype=torch.int32, device=dev)

    def step(ev_c0=None, ev_c1=None):
        ctx.reset(stream)
        if p2p:  # every image reset before any rank folds into it
            torch.cuda.synchronize(dev)
            dist.barrier()
        if ev_c0 is not None:
            ev_c0.record(stream)
        ctx.consume(rec, stream=stream)
        if ev_c1 is not None:
            ev_c1.record(stream)
        if p2p:  # every rank's fold (and its flush into the peers) done before the draws
            torch.cuda.synchronize(dev)
            dist.barrier()
        if comm is not None:
            ctx.merge(comm, stream)
        if sample:
            ctx.sample_device(draws, draw_status, N_DRAWS, 20150616, stream)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    if launched:
        dist.barrier()
    torch.cuda.synchronize()
    launches0 = ctx.kernel_launches()
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
           for _ in range(steps)]
    t_start, t_end = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with ClockSampler(local) as clk:
        t_start.record(stream)
        for k in range(steps):
            step(*evs[k])
        t_end.record(stream)
        torch.cuda.synchronize()
    if launched:
        dist.barrier()
    torch.cuda.synchronize()
    launches = ctx.kernel_launches() - launches0
    if sample:   # the device-side draws of the last step == the host-output API on the same tables
        assert int(draw_status.item()) == 0, "sampling: no eligible dynamic instruction"
        host_draws = ctx.sample(N_DRAWS, 20150616, stream)
        assert draws.cpu().numpy().tobytes() == host_draws.tobytes(), "device draws differ"
    ms = t_start.elapsed_time(t_end)
    consume_ms = [a.elapsed_time(b) for a, b in evs]
    if p2p:  # the step is the fused fold + merge; the host barriers around it are not device time
        ms = sum(consume_ms)
    ms = max_over_ranks(ms, dev)
    sec = ms / 1e3
    value = world * n * steps / sec
    consume_avg_s = statistics.mean(consume_ms) / 1e3
    peak, peak_src = measured_peaks()
    achieved = alg_bytes / consume_avg_s / 1e9

    # end-to-end through the public API with HOST buffers (pinned), copies inside the timed region
    e2e = None
    if not args.no_e2e and not p2p:  # every rank at once on its own shard; the merge is inside the step at N > 1
        e2e = measure_e2e(rec, P, mask, min(n, 1 << 24), dev, comm=comm, world=world,
                          launched=launched)
        if extras and mask & 2:  # the same with the non-GLOBAL address rows split off
            e2e["global_rows_only"] = measure_e2e(rec, P, mask, min(n, 1 << 24), dev, comm=comm,
                                                  world=world, launched=launched, global_rows=True)

    cpu = slow = online = inj = None
    if extras and not args.no_cpu_baseline and rank == 0 and world == 1:
        cpu = cpu_baseline(args, rec, mask, P)
    if extras and not args.no_slowdown and rank == 0:
        slow = measure_slowdown(dev)
        online = measure_online_trace(dev, slow)
    if extras and not args.no_injection and rank == 0:
        inj = measure_injection(dev)
    if own_comm is not None:
        sassi.sassi_nccl_comm_destroy(own_comm)
    if p2p:  # (the p2p protocol's parity: tests/test_gpu_p2p.py)
        ctx.clear_peer_tables()
        dist.barrier()  # every handle to this image is closed before it is freed
    ctx.close()
    if rank != 0:
        return None
    stored = 16 * n + 256 * rec["n_addr_rows"] + 128 * rec["n_val_rows"]
    line = {
        "metric": METRIC, "value": value, "unit": "records/s", "n_gpus": world,
        "steps": steps, "warmup": args.warmup, "ms_per_step": ms / steps,
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u32",
        "data": "synthetic",
        "config": {"workload": workload + ": " + desc + (", all four handlers + %d-site sampling" %
                                                         N_DRAWS if sample else ""),
                   "records_per_gpu": n, "sites": len(rec["sites"]),
                   "threads": 32 * P.total_warps, "handlers": mask,
                   "stored_bytes_per_gpu": stored, "algorithmic_bytes_per_gpu": alg_bytes,
                   "l2": "inputs (%.1f GB) exceed the 126 MB L2; no flush" % (stored / 1e9),
                   "parallelism": "dp%d (warp-id shards%s)" % (
                       world, ", fused fold + merge over peer memory" if p2p else
                       (", NCCL allreduce merge per step" if merge_on else "")),
                   "shared_gpu": bool(getattr(args, "share_gpu", False))},
        "hbm_gbs": world * alg_bytes * steps / sec / 1e9,
        "hbm_frac_of_spec_8tbs": alg_bytes * steps / sec / 1e9 / SPEC_HBM_GBS,
        "roofline": {"bound": "hbm", "kernel": "consume_kernel<%d>" % mask,
                     "achieved": achieved, "peak": peak, "unit": "GB/s",
                     "frac": achieved / peak, "peak_source": peak_src,
                     "traffic": ncu_traffic(workload),
                     "algorithmic_bytes_per_launch": alg_bytes,
                     "consume_ms_avg": consume_avg_s * 1e3,
                     "consume_share_of_step": (consume_avg_s * 1e3) / (ms / steps)},
        "gpu_launches": launches,
        "clocks": clk.result(),
    }
    for k, v in (("e2e", e2e), ("cpu_baseline", cpu), ("instrumented_slowdown", slow),
                 ("online_trace", online), ("error_injection", inj)):
        if v:
            line[k] = v
    return line


def main():
    args = parse()
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        sys.exit(self_launch(args.gpus))
    rank, world, local = dist_env()
    if world != args.gpus:
        sys.exit("bench.py: --gpus %d but WORLD_SIZE=%d (launch one rank per GPU)" % (args.gpus, world))
    if args.selftest_dist:
        run_selftest_dist(args, rank, world)
        return
    args.workload = args.workload or ("c3" if world == 1 else "c5")
    if args.impl == "reference":
        run_reference(args, rank, world, args.workload)
        return
    import torch
    import torch.distributed as dist
    if args.share_gpu:
        if args.merge != "p2p" or args.workload == "c5":
            sys.exit("bench.py: --share-gpu needs --merge p2p and c2 / c3 / c4 (NCCL refuses two ranks "
                     "on one GPU; c5 shards do not fit twice)")
        local = 0
    torch.cuda.set_device(local)
    if "RANK" in os.environ:  # under torchrun (any world size)
        if args.share_gpu:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    try:
        if args.workload == "c5":
            run_c5(args, rank, world, local)
        else:
            line = run_weak(args, rank, world, local, args.workload)
            if line is not None:
                print(json.dumps(line), flush=True)
    finally:
        if dist.is_initialized():
            dist.destroy_process_group()


def measure_injection(dev, k=1000):
    """§8.1's error-injection study on the four instrumented kernels (the Fig.10 analogue,
    L637-L667): profile, draw k sites (L629), one run per site; % of runs per outcome and the
    campaign's rate (runs/s, wall clock around the k runs: each run synchronises)."""
    import torch
    from paper_conf_isca_stephensonhlejn15_b200 import sassi
    out = {}
    for name in ("vecadd", "bfs", "sgemm", "stencil"):
        ik = sassi.InstrumentedKernel(name, 0, device=dev.index)
        ctx = ik.context(sassi.SASSI_H_INSTCOUNT)
        ik.run(sassi.SASSI_H_INSTCOUNT, ctx)
        sites = ctx.sample(k, 20150616)
        ctx.close()
        torch.cuda.synchronize(dev)
        t0 = time.perf_counter()
        outs = ik.inject(sites)
        dt = time.perf_counter() - t0
        r = {"runs": k, "runs_per_s": k / dt}
        for code, nm in enumerate(sassi.INJ_OUTCOME_NAMES):
            r[nm + "_pct"] = 100.0 * float((outs["outcome"] == code).sum()) / k
        out[name] = r
        ik.close()
    return out


def measure_slowdown(dev):
    """Instrumented-kernel slowdown K = t_instrumented / t_uninstrumented (the K column of the
    paper's Table 3), median of 5 runs each (L679), per handler, for the four synthetic
    kernels at their timing sizes; `null_abi` is the paper's stubbed-handler control (L687);
    `instmix` is Fig.3's handler (L193-L199), `all` the four case studies, `every` all five;
    `*_smem` the same with the opt-in per-CTA shared-memory tables (the default uses none, L741)."""
    import torch
    from paper_conf_isca_stephensonhlejn15_b200 import sassi
    modes = {"null_abi": sassi.SASSI_IK_NULL_ABI, "branch": 1, "memdiv": 2, "value": 4,
             "instcount": 8, "instmix": 16, "all": 15, "every": 31}
    # the same handlers with the opt-in per-CTA shared-memory tables (SASSI_IK_SMEM)
    modes.update({k + "_smem": m | sassi.SASSI_IK_SMEM for k, m in list(modes.items())
                  if 0 < m <= sassi.SASSI_H_EVERY})
    out = {}
    stream = torch.cuda.current_stream(dev)
    for name in ("vecadd", "bfs", "sgemm", "stencil"):
        ik = sassi.InstrumentedKernel(name, 0, device=dev.index)
        ctx = ik.context(sassi.SASSI_H_EVERY)

        def timed(mode):
            ts = []
            for rep in range(6):
                if mode & sassi.SASSI_H_EVERY:
                    ctx.reset(stream)
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record(stream)
                ik.run(mode, ctx if mode & sassi.SASSI_H_EVERY else None, stream)
                b.record(stream)
                b.synchronize()
                if rep:
                    ts.append(a.elapsed_time(b))
            return statistics.median(ts)

        base = timed(sassi.SASSI_IK_NONE)
        r = {"base_ms": base}
        for k, m in modes.items():
            r[k] = timed(m) / base
        out[name] = r
        ctx.close()
        ik.close()
    # harmonic mean over the kernels per handler set (the statistic of the paper's Table 3)
    keys = [k for k in next(iter(out.values())) if k != "base_ms"]
    out["hmean"] = {k: len(out) / sum(1.0 / out[n][k] for n in out) for k in keys}
    return out


# online-trace sizes: the timing sizes, except SGEMM at 1024 (2048's trace is ~1.2e9 records)
ONLINE_SIZES = {"vecadd": 0, "bfs": 0, "sgemm": 1024, "stencil": 0}


def measure_online_trace(dev, slow=None):
    """The trace-driven alternative to inline handlers (L747): each kernel traced
    segment by segment into a two-slot ring while the previous segment is folded by the consume
    kernel on a second stream (sassi_ik_trace_fold), all five handlers. Median of 3 (CUDA events on
    the caller's stream around the blocking call); K = t / t_uninstrumented of the same size;
    `serial_ms` = the same with the overlap disabled."""
    import torch
    from paper_conf_isca_stephensonhlejn15_b200 import sassi
    out = {}
    stream = torch.cuda.current_stream(dev)
    for name, size in ONLINE_SIZES.items():
        ik = sassi.InstrumentedKernel(name, size, device=dev.index)
        ctx = ik.context(sassi.SASSI_H_EVERY)

        def timed(fn, reps=4):
            ts = []
            for rep in range(reps):
                ctx.reset(stream)
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record(stream)
                r = fn()
                b.record(stream)
                b.synchronize()
                if rep:
                    ts.append(a.elapsed_time(b))
            return statistics.median(ts), r

        base, _ = timed(lambda: ik.run(sassi.SASSI_IK_NONE, None, stream), 6)
        t_on, st = timed(lambda: ik.trace_fold(ctx, stream=stream))
        t_ser, _ = timed(lambda: ik.trace_fold(ctx, serial=True, stream=stream))
        traced = 16 * st["n_records"] + 256 * st["n_addr_rows"] + 128 * st["n_val_rows"]
        out[name] = {"size": size or "timing", "base_ms": base, "online_ms": t_on, "serial_ms": t_ser,
                     "K_online": t_on / base, "records": st["n_records"],
                     "records_per_s": st["n_records"] / (t_on * 1e-3), "trace_bytes": traced,
                     "segments": st["segments"], "ring_bytes": st["ring_bytes"]}
        if slow and name in slow and not size:
            out[name]["K_inline_every"] = slow[name]["every"]
        ctx.close()
        ik.close()
    return out


def measure_e2e(rec, P, mask, n_e2e, dev, comm=None, world=1, launched=False, global_rows=False):
    """records/s through sassi_consume_host: pinned host buffers of the first n_e2e records, the
    H2D copies (double-buffered inside the library) and the table read-back inside the timing.
    At N > 1 every rank does the same on its own shard at the same time (after a barrier), the
    step includes the NCCL merge, and the time is the maximum over ranks. global_rows: the producer
    split off the address rows of non-GLOBAL memory sites (SASSI_ADDR_ROWS_GLOBAL), which no
    handler reads, so they never cross PCIe."""
    import torch
    import torch.distributed as dist
    from paper_conf_isca_stephensonhlejn15_b200 import gen, sassi
    n_e2e = (n_e2e // 256) * 256
    cb = rec["chunk_base"][: n_e2e // 256 + 1]
    tail = cb[-1].cpu().numpy().view(np.uint64)
    na, nv = int(tail[0]), int(tail[1])
    src = dict(rec, hdr=rec["hdr"][:n_e2e], addr=rec["addr"][:na], val=rec["val"][:nv],
               chunk_base=cb, n=n_e2e, n_addr_rows=na, n_val_rows=nv)
    if global_rows:  # producer-side split (input preparation, untimed)
        src = gen.split_global_rows(src)
        na = src["n_addr_rows"]
    h = dict(hdr=src["hdr"].cpu().pin_memory(), addr=src["addr"].cpu().pin_memory(),
             val=src["val"].cpu().pin_memory(), chunk_base=src["chunk_base"].cpu().pin_memory(),
             n=n_e2e, n_addr_rows=na, n_val_rows=nv)
    ctx = sassi.Context(rec["sites"], P.total_warps, mask, device=dev.index)
    if global_rows:
        ctx.set_addr_rows(sassi.SASSI_ADDR_ROWS_GLOBAL)
    stream = torch.cuda.current_stream(dev)
    out = np.zeros(ctx.layout["total"], np.uint64)
    cm = None
    if comm is not None:  # a communicator of its own for this context
        uid = torch.zeros(128, dtype=torch.uint8, device=dev)
        if not launched or dist.get_rank() == 0:
            uid.copy_(torch.frombuffer(bytearray(sassi.sassi_nccl_get_unique_id()), dtype=torch.uint8))
        if launched:
            dist.broadcast(uid, 0)
        cm = sassi.sassi_nccl_comm_create(world, dist.get_rank() if launched else 0,
                                          bytes(uid.cpu().numpy()), dev.index)

    def one():
        ctx.reset(stream)
        ctx.consume_host(h, stream=stream)
        if cm is not None:
            ctx.merge(cm, stream)
        sassi.sassi_read_tables(ctx.handle, out.size, stream, out)

    for _ in range(2):
        one()
    reps = 3
    torch.cuda.synchronize()
    if launched:
        dist.barrier()
    t0 = time.perf_counter()
    for _ in range(reps):
        one()
    el = time.perf_counter() - t0
    if launched:
        t = torch.tensor([el], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        el = float(t.item())
    if cm is not None:
        sassi.sassi_nccl_comm_destroy(cm)
    ctx.close()
    # what sassi_consume_host copies: rows only for the handlers that read them (sassi.h)
    h2d = (16 * n_e2e + (256 * na if mask & 2 else 0) + (128 * nv if mask & 4 else 0) +
           (16 * (n_e2e // 256 + 1) if mask & 6 else 0))
    return {"value": world * reps * n_e2e / el, "unit": "records/s", "h2d_bytes_per_step": world * h2d,
            "d2h_bytes_per_step": world * 8 * ctx.layout["total"], "records_per_step": world * n_e2e,
            "h2d_gbs": world * reps * h2d / el / 1e9,
            "note": "pinned host buffers, first %d records of each rank's shard%s; wall clock "
                    "around consume_host%s + read_tables (which synchronise), max over ranks" % (
                        n_e2e, ", address rows of GLOBAL memory sites only (SASSI_ADDR_ROWS_GLOBAL)"
                        if global_rows else "", " + merge" if cm is not None else "")}


if __name__ == "__main__":
    main()
