// sample.cu — error-injection site selection (§8.1): exclusive scan of the per-thread
// eligible dynamic-instruction counts, then k draws uniform over all eligible dynamic
// thread-instructions (reading R14: splitmix64(seed + j), k = floor(u * total / 2^64), thread =
// upper_bound(P, k) - 1, dynamic index = k - P[thread]).
#include "scan.cuh"

namespace sassi {
namespace {

__device__ __forceinline__ uint64_t splitmix64(uint64_t x) {
  uint64_t z = x + 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

__global__ void draw_kernel(const uint64_t* __restrict__ P, uint64_t n, uint32_t k, uint64_t seed,
                            sassi_inj_site* out) {
  const uint32_t j = blockIdx.x * blockDim.x + threadIdx.x;
  if (j >= k) return;
  const uint64_t total = P[n];
  const uint64_t u = splitmix64(seed + j);
  const uint64_t kk = __umul64hi(u, total);
  // upper_bound over P[0..n]: first index with P[idx] > kk; thread = idx - 1
  uint64_t lo = 0, hi = n + 1;
  while (lo < hi) {
    const uint64_t mid = (lo + hi) >> 1;
    if (P[mid] <= kk) lo = mid + 1;
    else hi = mid;
  }
  const uint64_t t = lo - 1;
  const uint64_t r = splitmix64((seed ^ 0xD1B54A32D192ED03ull) + j);
  sassi_inj_site o;
  o.kernel = 0;
  o.invocation = 0;
  o.thread = (uint32_t)t;
  o.reg_seed = (uint32_t)r;
  o.bit_seed = (uint32_t)(r >> 32);
  o.reserved = 0;
  o.dyn_index = kk - P[t];
  out[j] = o;
}

}  // namespace

int launch_sample(sassi_ctx* c, uint32_t k, uint64_t seed, sassi_inj_site* host_out,
                  cudaStream_t s) {
  const uint64_t n = 32ull * c->W;
  const uint64_t sw = scan_scratch_words(n);
  const uint64_t words = (n + 1) + sw + (4ull * k + 4);
  if (words > c->scan_words) {
    cudaFree(c->d_scan);
    c->d_scan = nullptr;
    c->scan_words = 0;
    SASSI_CUDA(cudaMalloc(&c->d_scan, 8 * words));
    c->scan_words = words;
  }
  uint64_t* P = c->d_scan;
  uint64_t* scratch = P + n + 1;
  sassi_inj_site* d_out = reinterpret_cast<sassi_inj_site*>(scratch + sw);
  const uint64_t* counts = c->d_table + c->off.counts;
  int rc = scan_u64(counts, n, P, scratch, s);
  if (rc) return rc;
  c->launches += 3;
  uint64_t h_total = 0;
  SASSI_CUDA(cudaMemcpyAsync(&h_total, P + n, 8, cudaMemcpyDeviceToHost, s));
  SASSI_CUDA(cudaStreamSynchronize(s));
  if (h_total == 0)
    return set_error(SASSI_ESTATE, "no eligible dynamic instruction was counted: nothing to sample");
  if (k == 0) return SASSI_OK;
  draw_kernel<<<(k + 255) / 256, 256, 0, s>>>(P, n, k, seed, d_out);
  c->launches += 1;
  SASSI_CUDA(cudaGetLastError());
  SASSI_CUDA(cudaMemcpyAsync(host_out, d_out, sizeof(sassi_inj_site) * k, cudaMemcpyDeviceToHost, s));
  SASSI_CUDA(cudaStreamSynchronize(s));
  return SASSI_OK;
}

}  // namespace sassi
