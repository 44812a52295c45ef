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

// One warp per draw. upper_bound over P[0..n] as a 32-ary search: each round the lanes probe the
// last element of 32 equal segments of [lo, hi) and one ballot picks the first segment that ends
// above kk (about 4 rounds of one coalesced load for 10^6 threads, not 20 dependent loads).
// Invariant: the answer (first idx with P[idx] > kk) lies in [lo, hi], = hi iff no P[lo..hi) > kk.
// A zero total (nothing eligible) is reported in *flag instead of drawing.
__global__ void draw_kernel(const uint64_t* __restrict__ P, uint64_t n, uint32_t k, uint64_t seed,
                            sassi_inj_site* out, uint32_t* flag) {
  const uint32_t lane = threadIdx.x & 31u;
  const uint32_t j = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const uint64_t total = P[n];
  if (j == 0 && lane == 0) *flag = total == 0 ? 1u : 0u;
  if (total == 0 || j >= k) return;
  const uint64_t u = splitmix64(seed + j);
  const uint64_t kk = __umul64hi(u, total);  // < total = P[n], and P[0] = 0 <= kk
  uint64_t lo = 0, hi = n + 1;
  while (hi - lo > 32) {
    const uint64_t step = (hi - lo + 31) / 32;
    const uint64_t end = min(lo + (lane + 1) * step, hi);  // one past segment `lane`
    const bool above = end > lo + lane * step && P[end - 1] > kk;
    const uint32_t b = __ballot_sync(FULL, above);
    if (b == 0) {  // every probed element <= kk: the answer is hi
      lo = hi;
      break;
    }
    const uint32_t i = __ffs(b) - 1;
    const uint64_t nlo = lo + i * step;
    hi = min(lo + (i + 1) * step, hi) - 1;
    lo = nlo;
  }
  if (lo < hi) {
    const uint32_t b = __ballot_sync(FULL, lo + lane < hi && P[lo + lane] > kk);
    lo = b ? lo + __ffs(b) - 1 : hi;
  }
  if (lane != 0) return;
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

// scan + draws, stream-ordered, no host synchronisation: draws to dev_out[k], *dev_status = 1 when
// the total is 0 (nothing to sample), else 0
int launch_sample_device(sassi_ctx* c, uint32_t k, uint64_t seed, sassi_inj_site* dev_out,
                         uint32_t* dev_status, cudaStream_t s) {
  const uint64_t n = 32ull * c->W;
  const uint64_t sw = scan_scratch_words(n);
  const uint64_t words = (n + 1) + sw;
  if (words > c->scan_words) {
    cudaFree(c->d_scan);
    c->d_scan = nullptr;
    c->scan_words = 0;
    SASSI_CUDA(cudaMalloc(&c->d_scan, 8 * words));
    c->scan_words = words;
  }
  uint64_t* P = c->d_scan;
  uint64_t* scratch = P + n + 1;
  const uint64_t* counts = c->d_table + c->off.counts;
  int rc = scan_u64(counts, n, P, scratch, s);
  if (rc) return rc;
  c->launches += 2;
  const uint32_t warps = k ? k : 1u;
  draw_kernel<<<(warps + 7) / 8, 256, 0, s>>>(P, n, k, seed, dev_out, dev_status);
  c->launches += 1;
  SASSI_CUDA(cudaGetLastError());
  return SASSI_OK;
}

// host-output form: the draws and the status come back in one copy, one synchronisation
int launch_sample(sassi_ctx* c, uint32_t k, uint64_t seed, sassi_inj_site* host_out,
                  cudaStream_t s) {
  const uint64_t bytes = sizeof(sassi_inj_site) * ((uint64_t)k + 1);  // + the status word
  if (bytes > c->sample_bytes) {
    cudaFree(c->d_sample);
    c->d_sample = nullptr;
    c->sample_bytes = 0;
    SASSI_CUDA(cudaMalloc(&c->d_sample, bytes));
    c->sample_bytes = bytes;
  }
  sassi_inj_site* d_out = reinterpret_cast<sassi_inj_site*>(c->d_sample);
  uint32_t* d_flag = reinterpret_cast<uint32_t*>(d_out + k);
  int rc = launch_sample_device(c, k, seed, d_out, d_flag, s);
  if (rc) return rc;
  uint32_t h_flag = 0;
  SASSI_CUDA(cudaMemcpyAsync(&h_flag, d_flag, 4, cudaMemcpyDeviceToHost, s));
  if (k) SASSI_CUDA(cudaMemcpyAsync(host_out, d_out, sizeof(sassi_inj_site) * k, cudaMemcpyDeviceToHost, s));
  SASSI_CUDA(cudaStreamSynchronize(s));
  if (h_flag)
    return set_error(SASSI_ESTATE, "no eligible dynamic instruction was counted: nothing to sample");
  return SASSI_OK;
}

}  // namespace sassi
