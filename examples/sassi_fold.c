/*
 * sassi_fold.c — a plain C99 user of the C ABI (include/sassi.h): folds a record stream read from
 * binary files and writes the table image (and, optionally, injection-site draws).
 *
 *   sassi_fold SITES HDR ADDR VAL N_WARPS HANDLER_MASK OUT_TABLE [K SEED OUT_DRAWS]
 *
 * SITES: sassi_site[], HDR: sassi_hdr[], ADDR: uint64_t[rows][32], VAL: uint32_t[rows][32]
 * (SRF1, little-endian, no headers; ADDR / VAL may be empty files). The chunk index is built on the
 * device with sassi_index_records. Exit status 0 on success, 1 on a usage / IO error, 2 on a
 * library error (message on stderr). Device memory comes from the CUDA runtime; nothing else.
 */
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>

#include <cuda_runtime_api.h>

#include "sassi.h"

static void* read_file(const char* path, size_t* bytes) {
  FILE* f = fopen(path, "rb");
  if (!f) return NULL;
  fseek(f, 0, SEEK_END);
  long n = ftell(f);
  fseek(f, 0, SEEK_SET);
  void* p = malloc(n > 0 ? (size_t)n : 1);
  if (p && n > 0 && fread(p, 1, (size_t)n, f) != (size_t)n) {
    free(p);
    p = NULL;
  }
  fclose(f);
  *bytes = n > 0 ? (size_t)n : 0;
  return p;
}

static void* to_device(const void* host, size_t bytes) {
  void* d = NULL;
  if (cudaMalloc(&d, bytes ? bytes : 16) != cudaSuccess) return NULL;
  if (host && bytes && cudaMemcpy(d, host, bytes, cudaMemcpyHostToDevice) != cudaSuccess) return NULL;
  return d;
}

#define CHECK(call)                                                                   \
  do {                                                                                \
    int rc_ = (call);                                                                 \
    if (rc_ != SASSI_OK) {                                                            \
      fprintf(stderr, "%s: %s (%s)\n", #call, sassi_strerror(rc_), sassi_last_error()); \
      return 2;                                                                       \
    }                                                                                 \
  } while (0)

int main(int argc, char** argv) {
  if (argc != 8 && argc != 11) {
    fprintf(stderr, "usage: %s SITES HDR ADDR VAL N_WARPS HANDLER_MASK OUT_TABLE [K SEED OUT_DRAWS]\n",
            argv[0]);
    return 1;
  }
  size_t bs, bh, ba, bv;
  sassi_site* sites = (sassi_site*)read_file(argv[1], &bs);
  sassi_hdr* hdr = (sassi_hdr*)read_file(argv[2], &bh);
  uint64_t* addr = (uint64_t*)read_file(argv[3], &ba);
  uint32_t* val = (uint32_t*)read_file(argv[4], &bv);
  if (!sites || !hdr || !addr || !val) {
    fprintf(stderr, "cannot read an input file\n");
    return 1;
  }
  const uint32_t n_sites = (uint32_t)(bs / sizeof(sassi_site)), n_warps = (uint32_t)strtoul(argv[5], NULL, 0);
  const uint32_t mask = (uint32_t)strtoul(argv[6], NULL, 0);
  const uint64_t n = bh / sizeof(sassi_hdr);

  struct sassi_ctx* ctx = NULL;
  CHECK(sassi_ctx_create(&ctx, 0, sites, n_sites, n_warps));
  CHECK(sassi_attach_handler(ctx, mask));

  sassi_records r;
  r.hdr = (const sassi_hdr*)to_device(hdr, bh);
  r.addr = (const uint64_t*)to_device(addr, ba);
  r.val = (const uint32_t*)to_device(val, bv);
  r.n_addr_rows = ba / 256;
  r.n_val_rows = bv / 128;
  sassi_chunk_base* cb = (sassi_chunk_base*)to_device(NULL, 16 * ((n + SASSI_CHUNK - 1) / SASSI_CHUNK + 1));
  if (!r.hdr || !r.addr || !r.val || !cb) {
    fprintf(stderr, "device allocation failed\n");
    return 2;
  }
  r.chunk_base = cb;
  CHECK(sassi_index_records(ctx, r.hdr, n, cb, NULL));
  CHECK(sassi_consume(ctx, &r, n, NULL));

  sassi_layout L;
  CHECK(sassi_table_layout(n_sites, n_warps, &L));
  uint64_t* table = (uint64_t*)malloc(8 * L.total);
  CHECK(sassi_read_tables(ctx, table, L.total, NULL));
  FILE* f = fopen(argv[7], "wb");
  if (!f || fwrite(table, 8, L.total, f) != L.total) return 1;
  fclose(f);
  printf("records %llu  invalid %llu  unknown pc %llu  sites %u  warps %u\n",
         (unsigned long long)table[0], (unsigned long long)table[1], (unsigned long long)table[2],
         n_sites, n_warps);

  if (argc == 11) {  /* error-injection site sampling (L629) */
    const uint32_t k = (uint32_t)strtoul(argv[8], NULL, 0);
    const uint64_t seed = strtoull(argv[9], NULL, 0);
    sassi_inj_site* draws = (sassi_inj_site*)malloc(sizeof(sassi_inj_site) * (k ? k : 1));
    CHECK(sassi_sample_sites(ctx, k, seed, draws, NULL));
    FILE* g = fopen(argv[10], "wb");
    if (!g || fwrite(draws, sizeof(sassi_inj_site), k, g) != k) return 1;
    fclose(g);
    free(draws);
  }
  sassi_ctx_destroy(ctx);
  cudaFree((void*)r.hdr);
  cudaFree((void*)r.addr);
  cudaFree((void*)r.val);
  cudaFree(cb);
  free(table);
  free(sites);
  free(hdr);
  free(addr);
  free(val);
  return 0;
}
