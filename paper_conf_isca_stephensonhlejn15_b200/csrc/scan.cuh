// scan.cuh — exclusive prefix sum of a u64 array on the device (two kernels: per-block sums, then
// apply: each block adds up the sums of the blocks before it itself, so no third launch). Used by sampling (per-thread counts) and by
// sassi_index_records (per-chunk row counts). Included by one .cu each (internal linkage).
#pragma once
#include "common.cuh"

namespace sassi {
namespace {
namespace scan_detail {

constexpr int kScanThreads = 1024;
constexpr int kScanPerThread = 4;
constexpr uint64_t kScanBlock = kScanThreads * kScanPerThread;

__device__ __forceinline__ uint64_t warp_incl_scan(uint64_t v, uint32_t lane) {
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint64_t y = __shfl_up_sync(FULL, v, o);
    if (lane >= (uint32_t)o) v += y;
  }
  return v;
}

// block-wide exclusive scan of one value per thread; returns the exclusive prefix, *total = sum
__device__ uint64_t block_excl_scan(uint64_t v, uint64_t* total) {
  __shared__ uint64_t warp_sums[32];
  const uint32_t lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const uint64_t inc = warp_incl_scan(v, lane);
  if (lane == 31) warp_sums[w] = inc;
  __syncthreads();
  if (w == 0) {
    const uint64_t x = lane < blockDim.x / 32 ? warp_sums[lane] : 0;
    const uint64_t xi = warp_incl_scan(x, lane);
    warp_sums[lane] = xi - x;
    if (lane == 31) *total = xi;
  }
  __syncthreads();
  const uint64_t r = warp_sums[w] + inc - v;
  __syncthreads();
  return r;
}

__global__ void __launch_bounds__(kScanThreads) block_sums_kernel(const uint64_t* __restrict__ c,
                                                                  uint64_t n, uint64_t* bsum) {
  __shared__ uint64_t tot;
  const uint64_t i0 = blockIdx.x * kScanBlock + threadIdx.x * kScanPerThread;
  uint64_t s = 0;
#pragma unroll
  for (int k = 0; k < kScanPerThread; ++k)
    if (i0 + k < n) s += c[i0 + k];
  block_excl_scan(s, &tot);
  if (threadIdx.x == 0) bsum[blockIdx.x] = tot;
}

__global__ void __launch_bounds__(kScanThreads) scan_apply_kernel(const uint64_t* __restrict__ c,
                                                                  uint64_t n,
                                                                  const uint64_t* __restrict__ bsum,
                                                                  uint64_t* P) {
  __shared__ uint64_t tot, base;
  // this block's offset: the sum of the block sums before it (a few thousand at most)
  uint64_t part = 0;
  for (uint64_t b = threadIdx.x; b < blockIdx.x; b += blockDim.x) part += bsum[b];
  block_excl_scan(part, &tot);
  if (threadIdx.x == 0) base = tot;
  __syncthreads();
  const uint64_t i0 = blockIdx.x * kScanBlock + threadIdx.x * kScanPerThread;
  uint64_t x[kScanPerThread];
  uint64_t s = 0;
#pragma unroll
  for (int k = 0; k < kScanPerThread; ++k) {
    x[k] = i0 + k < n ? c[i0 + k] : 0;
    s += x[k];
  }
  uint64_t run = base + block_excl_scan(s, &tot);
#pragma unroll
  for (int k = 0; k < kScanPerThread; ++k) {
    if (i0 + k < n) P[i0 + k] = run;
    run += x[k];
  }
  if (blockIdx.x == gridDim.x - 1 && threadIdx.x == 0) P[n] = base + tot;
}

}  // namespace scan_detail
}  // namespace

// P[0..n] = exclusive prefix of in[0..n) (P[n] = total); scratch >= scan_scratch_words(n) words.
static inline uint64_t scan_scratch_words(uint64_t n) {
  return (n + scan_detail::kScanBlock - 1) / scan_detail::kScanBlock;
}
static inline int scan_u64(const uint64_t* in, uint64_t n, uint64_t* P, uint64_t* scratch,
                           cudaStream_t s) {
  using namespace scan_detail;
  const uint64_t nb = (n + kScanBlock - 1) / kScanBlock;
  if (nb == 0) {
    SASSI_CUDA(cudaMemsetAsync(P, 0, 8, s));
    return SASSI_OK;
  }
  block_sums_kernel<<<(unsigned)nb, kScanThreads, 0, s>>>(in, n, scratch);
  scan_apply_kernel<<<(unsigned)nb, kScanThreads, 0, s>>>(in, n, scratch, P);
  SASSI_CUDA(cudaGetLastError());
  return SASSI_OK;
}

}  // namespace sassi
