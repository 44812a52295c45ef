"""The oracle over a full-size configuration, sharded by warp across host processes (test
infrastructure: the tables are commutative folds, so the oracle's own merge of per-shard tables is
the single-pass fold; that identity is itself pinned in test_oracle.py::test_merge_equals_single_pass).

Each worker regenerates its warps with the host build of the seeded generator (the same C source
as the device generator; their byte equality is a GPU test), folds them with the plain
single-threaded oracle, and returns its table; the parent merges the tables with oracle.merge.
A limit (the preset's record count) cuts the stream exactly where the device stream is cut."""
from __future__ import annotations

import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def _work(job):
    import oracle
    from paper_conf_isca_stephensonhlejn15_b200 import gen
    name, warp_base, n_warps, limit, mask, pcs = job
    P, _, _, _ = gen.preset(name)
    r = gen.generate_host(P, limit, warp_base, n_warps)
    if r["n"] == 0:
        return None
    return oracle.run(r["sites"], P.total_warps, mask, r["hdr"], r["addr"], r["val"], pcs=pcs)


def oracle_full(name, mask, warp_base=0, n_warps=None, limit=None, pcs=(), warps_per_job=2048,
                workers=None):
    """Oracle table of warps [warp_base, warp_base + n_warps) of preset `name` cut at `limit`
    records (None: the whole range), computed in parallel warp shards and merged."""
    import multiprocessing as mp
    import oracle
    from paper_conf_isca_stephensonhlejn15_b200 import gen
    P, _, _, _ = gen.preset(name)
    n_warps = P.total_warps - warp_base if n_warps is None else n_warps
    counts = gen.count_host(P, warp_base, n_warps)[:, 0].astype(np.int64)
    first = np.concatenate([[0], np.cumsum(counts)])
    total = int(first[-1]) if limit is None else min(int(limit), int(first[-1]))
    jobs = []
    for w0 in range(0, n_warps, warps_per_job):
        if first[w0] >= total:
            break
        nw = min(warps_per_job, n_warps - w0)
        lim = min(int(first[w0 + nw] - first[w0]), total - int(first[w0]))
        jobs.append((name, warp_base + w0, nw, lim, mask, tuple(pcs)))
    workers = workers or max(1, min(8, os.cpu_count() or 1, len(jobs)))
    S = len(P.sites())
    acc = oracle.table_init(S, P.total_warps, mask, pcs)
    with mp.get_context("spawn").Pool(workers) as pool:
        for t in pool.imap_unordered(_work, jobs):
            if t is not None:
                oracle.merge(acc, t, S, P.total_warps)
    return acc, total
