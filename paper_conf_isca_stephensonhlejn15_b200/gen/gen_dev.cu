// gen_dev.cu — device build of the seeded record generator (sassi_gen.h): one CUDA warp walks one
// trace warp. Input generation only (untimed); none of the handler arithmetic lives here.
#include <cuda_runtime.h>
#include <cstdio>
#include "sassi_gen.h"

namespace {

__global__ void __launch_bounds__(128) gen_count_kernel(const gen_prog* __restrict__ P,
                                                        const gen_op* __restrict__ ops,
                                                        uint64_t* __restrict__ out) {
  const uint32_t wl = blockIdx.x * 4 + (threadIdx.x >> 5);
  if (wl >= P->n_warps) return;
  gen_out o = {};
  gen_walk(P, ops, wl, &o, 0);
  if ((threadIdx.x & 31) == 0) {
    out[3 * wl + 0] = o.n_rec;
    out[3 * wl + 1] = o.n_arow;
    out[3 * wl + 2] = o.n_vrow;
  }
}

__global__ void __launch_bounds__(128) gen_emit_kernel(const gen_prog* __restrict__ P,
                                                       const gen_op* __restrict__ ops,
                                                       const uint64_t* __restrict__ offs,
                                                       uint64_t limit, uint32_t* hdr,
                                                       uint64_t* addr, uint32_t* val,
                                                       uint64_t* chunk_base) {
  const uint32_t wl = blockIdx.x * 4 + (threadIdx.x >> 5);
  if (wl >= P->n_warps) return;
  if (offs[3 * wl] > limit) return;
  gen_out o = {};
  o.hdr = hdr; o.addr = addr; o.val = val; o.chunk_base = chunk_base;
  o.rec0 = offs[3 * wl]; o.arow0 = offs[3 * wl + 1]; o.vrow0 = offs[3 * wl + 2];
  o.limit = limit;
  gen_walk(P, ops, wl, &o, 1);
}

int upload(const gen_prog* P, const gen_op* ops, gen_prog** dP, gen_op** dops, cudaStream_t s) {
  const size_t nops = (size_t)P->n_pro + P->n_body + P->n_epi;
  if (cudaMallocAsync((void**)dP, sizeof(gen_prog), s) != cudaSuccess) return -2;
  if (cudaMallocAsync((void**)dops, sizeof(gen_op) * (nops ? nops : 1), s) != cudaSuccess) return -2;
  if (cudaMemcpyAsync(*dP, P, sizeof(gen_prog), cudaMemcpyHostToDevice, s) != cudaSuccess) return -2;
  if (nops && cudaMemcpyAsync(*dops, ops, sizeof(gen_op) * nops, cudaMemcpyHostToDevice, s) != cudaSuccess)
    return -2;
  return 0;
}

int finish(gen_prog* dP, gen_op* dops, cudaStream_t s) {
  cudaFreeAsync(dP, s);
  cudaFreeAsync(dops, s);
  cudaError_t e = cudaStreamSynchronize(s);
  if (e == cudaSuccess) e = cudaGetLastError();
  if (e != cudaSuccess) {
    fprintf(stderr, "sassi_gen: %s\n", cudaGetErrorString(e));
    return -2;
  }
  return 0;
}

}  // namespace

extern "C" {

// host P/ops; device out [n_warps][3]. Synchronous.
int sassi_gen_count(const gen_prog* P, const gen_op* ops, uint64_t* out, void* stream) {
  cudaStream_t s = (cudaStream_t)stream;
  gen_prog* dP = nullptr;
  gen_op* dops = nullptr;
  if (upload(P, ops, &dP, &dops, s)) return -2;
  if (P->n_warps) gen_count_kernel<<<(P->n_warps + 3) / 4, 128, 0, s>>>(dP, dops, out);
  return finish(dP, dops, s);
}

// host P/ops; device offs and outputs. Synchronous.
int sassi_gen_emit(const gen_prog* P, const gen_op* ops, const uint64_t* offs, uint64_t limit,
                   uint32_t* hdr, uint64_t* addr, uint32_t* val, uint64_t* chunk_base,
                   void* stream) {
  cudaStream_t s = (cudaStream_t)stream;
  gen_prog* dP = nullptr;
  gen_op* dops = nullptr;
  if (upload(P, ops, &dP, &dops, s)) return -2;
  if (P->n_warps)
    gen_emit_kernel<<<(P->n_warps + 3) / 4, 128, 0, s>>>(dP, dops, offs, limit, hdr, addr, val,
                                                         chunk_base);
  return finish(dP, dops, s);
}

}  // extern "C"
