/* gen_host.c — host build of the seeded record generator (sassi_gen.h). Input generation only. */
#include <stdlib.h>
#include <string.h>
#include "sassi_gen.h"

/* Per-warp record / addr-row / val-row counts of warps [0, P->n_warps). out: [n_warps][3]. */
int sassi_gen_count_host(const gen_prog* P, const gen_op* ops, uint64_t* out) {
  for (uint32_t wl = 0; wl < P->n_warps; ++wl) {
    gen_out o;
    memset(&o, 0, sizeof(o));
    gen_walk(P, ops, wl, &o, 0);
    out[3 * wl + 0] = o.n_rec;
    out[3 * wl + 1] = o.n_arow;
    out[3 * wl + 2] = o.n_vrow;
  }
  return 0;
}

/* Emit records with index < limit. offs: [n_warps][3] exclusive prefixes of the counts. The
 * caller writes the chunk_base sentinel when limit equals the total record count. */
int sassi_gen_emit_host(const gen_prog* P, const gen_op* ops, const uint64_t* offs, uint64_t limit,
                        uint32_t* hdr, uint64_t* addr, uint32_t* val, uint64_t* chunk_base) {
  for (uint32_t wl = 0; wl < P->n_warps; ++wl) {
    if (offs[3 * wl] > limit) break;
    gen_out o;
    memset(&o, 0, sizeof(o));
    o.hdr = hdr; o.addr = addr; o.val = val; o.chunk_base = chunk_base;
    o.rec0 = offs[3 * wl]; o.arow0 = offs[3 * wl + 1]; o.vrow0 = offs[3 * wl + 2];
    o.limit = limit;
    gen_walk(P, ops, wl, &o, 1);
  }
  return 0;
}

uint64_t sassi_gen_hash_host(uint64_t seed, uint32_t gw, uint32_t it, uint32_t op, uint32_t lane,
                             uint32_t salt) {
  return gen_hash(seed, gw, it, op, lane, salt);
}
int sassi_gen_sizeof_op(void) { return (int)sizeof(gen_op); }
int sassi_gen_sizeof_prog(void) { return (int)sizeof(gen_prog); }
