// tables.cu — table image layout and (re)initialisation (the CUPTI launch-callback analogue, L217).
#include "common.cuh"

namespace sassi {

Offsets layout_offsets(uint32_t S, uint32_t W) {
  Offsets o;
  o.br = 8;
  o.mem = o.br + 5ull * S;
  o.val = o.mem + 4ull * S;
  o.ones = o.val + 2ull * S;
  o.zeros = o.ones + 4ull * S;
  o.scalar = o.zeros + 4ull * S;
  o.h32 = o.scalar + 4ull * S;
  o.h128 = o.h32 + 1024;
  o.counts = o.h128 + 1024;
  o.mix = o.counts + 32ull * W;
  o.imix = o.mix + S;
  o.pcsel = o.imix + 8;
  o.pcmat = o.pcsel + 4;
  o.total = o.pcmat + 4ull * 1024;
  return o;
}

namespace {

// Sums start at 0; constantOnes / constantZeros start all-ones and isScalar starts 1 (the AND
// identities, Fig.9);
// diag[4..7] describe the image.
__global__ void init_tables_kernel(uint64_t* t, Offsets o, uint32_t S, uint32_t W, uint32_t mask,
                                   uint4 pcsel) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < o.total; i += stride) {
    uint64_t v = 0;
    if (i >= o.ones && i < o.scalar) v = 0xFFFFFFFFull;
    else if (i >= o.scalar && i < o.h32) v = 1;
    else if (i == 4) v = S;
    else if (i == 5) v = W;
    else if (i == 6) v = mask;
    else if (i == 7) v = SASSI_ABI_VERSION;
    else if (i == o.pcsel) v = pcsel.x;
    else if (i == o.pcsel + 1) v = pcsel.y;
    else if (i == o.pcsel + 2) v = pcsel.z;
    else if (i == o.pcsel + 3) v = pcsel.w;
    t[i] = v;
  }
}

}  // namespace

int launch_init_tables(sassi_ctx* c, cudaStream_t s) {
  uint64_t blocks = (c->off.total + 255) / 256;
  if (blocks > 4096) blocks = 4096;
  const uint4 sel = make_uint4(c->pcsel[0], c->pcsel[1], c->pcsel[2], c->pcsel[3]);
  init_tables_kernel<<<(unsigned)blocks, 256, 0, s>>>(c->d_table, c->off, c->S, c->W, c->mask, sel);
  SASSI_CUDA(cudaGetLastError());
  c->launches += 1;
  return SASSI_OK;
}

}  // namespace sassi

extern "C" int sassi_table_layout(uint32_t n_sites, uint32_t n_warps, sassi_layout* out) {
  if (!out) return sassi::set_error(SASSI_EINVAL, "sassi_table_layout: null out");
  sassi::Offsets o = sassi::layout_offsets(n_sites, n_warps);
  out->diag = 0;
  out->br = o.br;
  out->mem = o.mem;
  out->val = o.val;
  out->ones = o.ones;
  out->zeros = o.zeros;
  out->scalar = o.scalar;
  out->h32 = o.h32;
  out->h128 = o.h128;
  out->counts = o.counts;
  out->mix = o.mix;
  out->imix = o.imix;
  out->pcsel = o.pcsel;
  out->pcmat = o.pcmat;
  out->total = o.total;
  return SASSI_OK;
}
