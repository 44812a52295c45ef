"""Worker for test_gpu_p2p.py (run under torchrun, gloo group, every rank on a GPU of this node —
all on cuda:0 when the node has one): the fused fold + merge over peer memory. Each rank folds its
part of a record stream straight into every rank's table image (sassi_add_peer_table); after the
barrier every image must equal the oracle's tables of the whole stream, bit for bit."""
import os
import sys

import numpy as np
import torch
import torch.distributed as dist

HERE = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, HERE)
sys.path.insert(0, os.path.dirname(HERE))
import oracle  # noqa: E402
from gpu_helpers import to_device  # noqa: E402
from test_oracle import random_trace  # noqa: E402
from paper_conf_isca_stephensonhlejn15_b200 import gen, sassi  # noqa: E402


def split(d, rank, world):
    """Chunk-aligned record range of this rank (rows addressed absolutely by the chunk index)."""
    n = d["n"]
    cuts = [min(n, (n * r // world) // 256 * 256) for r in range(world)] + [n]
    a, b = cuts[rank], cuts[rank + 1]
    return dict(d, hdr=d["hdr"][a:b], chunk_base=d["chunk_base"][a // 256: (b + 255) // 256 + 1], n=b - a)


def run_case(name, sites, W, mask, d, want, rank, world):
    ctx = sassi.Context(sites, W, mask)
    handles = [None] * world
    dist.all_gather_object(handles, ctx.ipc_table_handle())
    for j in range(world):
        if j != rank:
            ctx.add_peer_table(handles[j])
    # while peers fold into this image its layout is fixed: another handler set or pc selection
    # is refused
    for bad in (lambda: sassi.sassi_attach_handler(ctx.handle, sassi.SASSI_H_BRANCH),
                lambda: ctx.select_memdiv_pcs([])):
        try:
            bad()
            raise AssertionError("layout change accepted with peer tables attached")
        except sassi.SassiError as e:
            assert e.status == sassi.SASSI_ESTATE
    for rep in range(2):  # twice: reset between rounds works with peers attached
        ctx.reset()
        torch.cuda.synchronize()
        dist.barrier()
        part = split(d, rank, world)
        if part["n"]:
            ctx.consume(part)
        torch.cuda.synchronize()
        dist.barrier()
        t = ctx.read_tables()
        assert np.array_equal(t, want), "%s: rank %d round %d differs from the oracle" % (name, rank, rep)
        dist.barrier()  # nobody resets before everyone has read
    ctx.clear_peer_tables()
    dist.barrier()      # every handle to this image is closed before it is freed
    ctx.close()


def main():
    dist.init_process_group("gloo")
    rank, world = dist.get_rank(), dist.get_world_size()
    torch.cuda.set_device(int(os.environ.get("LOCAL_RANK", 0)) % torch.cuda.device_count())
    # a random edge-case trace, every handler
    s, W, hdr, addr, val = random_trace(2718, n=30000)
    want = oracle.run(s, W, sassi.SASSI_H_ALL | sassi.SASSI_H_INSTMIX, hdr, addr, val)
    run_case("random", s, W, sassi.SASSI_H_EVERY, to_device(s, hdr, addr, val), want, rank, world)
    # the BFS-shaped config c2 (first 10^6 records)
    P, lim, mask, _ = gen.preset("c2")
    d = gen.generate_device(P, 1_000_000)
    h = gen.to_host(d)
    want = oracle.run(h["sites"], P.total_warps, mask, h["hdr"], h["addr"], h["val"])
    run_case("c2", d["sites"], P.total_warps, mask, d, want, rank, world)
    print("p2p ok rank %d of %d" % (rank, world), flush=True)
    dist.destroy_process_group()


if __name__ == "__main__":
    main()
