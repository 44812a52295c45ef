"""c5 in full (all 8 warp shards, ~4x10^9 records, ~680 GB generated shard by shard): the GPU folds
every shard (bench.py's launch configuration) into a per-shard context and into one job context;
each shard's table and the job's table must equal the oracle (tests/oracle_shards.py: host warp
sub-shards in parallel processes, merged). Prints one line per shard and a summary; exit 1 on any
difference. usage: python tools/parity_c5_full.py [N_SHARDS]"""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
from gpu_helpers import diff_tables  # noqa: E402
from oracle_shards import oracle_full  # noqa: E402
from paper_conf_isca_stephensonhlejn15_b200 import gen, sassi  # noqa: E402

if __name__ == "__main__":
    n_shards = int(sys.argv[1]) if len(sys.argv) > 1 else 8
    P, _, mask, _ = gen.preset("c5")
    W = P.total_warps
    job, acc, fails, total = None, None, 0, 0
    for shard in range(n_shards):
        t0 = time.time()
        d = gen.generate_device(P, None, shard * 16384, 16384)
        S = len(d["sites"])
        if job is None:
            job = sassi.Context(d["sites"], W, mask)
        ctx = sassi.Context(d["sites"], W, mask)
        ctx.consume(d)
        job.consume(d)
        t = ctx.read_tables()
        ctx.close()
        n = d["n"]
        del d
        torch.cuda.empty_cache()
        o, no = oracle_full("c5", mask, warp_base=shard * 16384, n_warps=16384, warps_per_job=512)
        msg = diff_tables(t, o, S, W) if no == n else "record counts differ"
        acc = o if acc is None else oracle.merge(acc, o, S, W)
        fails += msg is not None
        total += n
        print("shard %d: %d records, %s (%.0f s)" % (shard, n, "bit-exact" if msg is None else msg,
                                                   time.time() - t0), flush=True)
    tj = job.read_tables()
    msg = diff_tables(tj, acc, S, W)
    fails += msg is not None
    print("job (all %d shards folded into one context, %d records): %s" % (
        n_shards, total, "bit-exact vs the oracle's merge" if msg is None else msg), flush=True)
    job.close()
    sys.exit(1 if fails else 0)
