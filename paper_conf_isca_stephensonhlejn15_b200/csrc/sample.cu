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

// One profile of a sampling campaign: a kernel invocation's per-thread prefix P[0..n] (P[n] = its
// total) and the ids its tuples carry.
struct Prof {
  const uint64_t* P;
  uint64_t n;
  uint32_t kernel, invocation;
};

// One warp per draw, over the concatenation of the profiles' eligible dynamic thread-instructions
// (a single profile is sassi_sample_sites). The grand total and the draw's profile come from the
// profiles' totals (32 at a time: one load per lane, an inclusive warp scan, one ballot); within the
// profile, upper_bound over P[0..n] as a 32-ary search: each round the lanes probe the last element
// of 32 equal segments of [lo, hi) and one ballot picks the first segment that ends above kk (about
// 4 rounds of one coalesced load for 10^6 threads, not 20 dependent loads). Invariant: the answer
// (first idx with P[idx] > kk) lies in [lo, hi], = hi iff no P[lo..hi) > kk.
// A zero total (nothing eligible) is reported in *flag instead of drawing. prof == nullptr: the one
// profile `one` (sassi_sample_sites: no table to upload).
__global__ void draw_kernel(const Prof* __restrict__ prof, uint32_t n_prof, Prof one, uint32_t k,
                            uint64_t seed, sassi_inj_site* out, uint32_t* flag) {
  const uint32_t lane = threadIdx.x & 31u;
  const uint32_t j = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  auto get = [&](uint32_t q) -> Prof { return prof ? prof[q] : one; };
  uint64_t total = 0;
  for (uint32_t q = lane; q < n_prof; q += 32) {
    const Prof pq = get(q);
    total += pq.P[pq.n];
  }
  for (uint32_t o = 16; o; o >>= 1) total += __shfl_xor_sync(FULL, total, o);
  if (j == 0 && lane == 0) *flag = total == 0 ? 1u : 0u;
  if (total == 0 || j >= k) return;
  const uint64_t u = splitmix64(seed + j);
  uint64_t kk = __umul64hi(u, total);  // < total
  // the profile holding kk: first q with (sum of totals up to q) > kk
  uint32_t q = 0;
  for (uint32_t q0 = 0;; q0 += 32) {
    const uint32_t qq = q0 + lane;
    uint64_t t = 0;
    if (qq < n_prof) {
      const Prof pq = get(qq);
      t = pq.P[pq.n];
    }
    uint64_t inc = t;
    for (uint32_t o = 1; o < 32; o <<= 1) {
      const uint64_t y = __shfl_up_sync(FULL, inc, o);
      if (lane >= o) inc += y;
    }
    const uint32_t b = __ballot_sync(FULL, qq < n_prof && inc > kk);
    if (b) {
      const uint32_t i = __ffs(b) - 1;
      kk -= __shfl_sync(FULL, inc - t, i);  // the totals of the profiles before it
      q = q0 + i;
      break;
    }
    kk -= __shfl_sync(FULL, inc, 31);
  }
  const Prof pr = get(q);
  const uint64_t* const P = pr.P;
  const uint64_t n = pr.n;
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
  o.kernel = pr.kernel;
  o.invocation = pr.invocation;
  o.thread = (uint32_t)t;
  o.reg_seed = (uint32_t)r;
  o.bit_seed = (uint32_t)(r >> 32);
  o.reserved = 0;
  o.dyn_index = kk - P[t];
  out[j] = o;
}

// exclusive scan of a context's per-thread counts into its scan buffer -> the prefix P[0..32W]
int scan_counts(sassi_ctx* c, cudaStream_t s, const uint64_t** P_out) {
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
  int rc = scan_u64(c->d_table + c->off.counts, n, P, P + n + 1, s);
  if (rc) return rc;
  c->launches += 2;
  *P_out = P;
  return SASSI_OK;
}

}  // namespace

// scan + draws, stream-ordered, no host synchronisation: draws to dev_out[k], *dev_status = 1 when
// the total is 0 (nothing to sample), else 0
int launch_sample_device(sassi_ctx* c, uint32_t k, uint64_t seed, sassi_inj_site* dev_out,
                         uint32_t* dev_status, cudaStream_t s) {
  const uint64_t* P = nullptr;
  int rc = scan_counts(c, s, &P);
  if (rc) return rc;
  const uint32_t warps = k ? k : 1u;
  draw_kernel<<<(warps + 7) / 8, 256, 0, s>>>(nullptr, 1u, Prof{P, 32ull * c->W, 0u, 0u}, k, seed,
                                               dev_out, dev_status);
  c->launches += 1;
  SASSI_CUDA(cudaGetLastError());
  return SASSI_OK;
}

// several profiles (kernel invocations, one context each, one device): scans, then the draws over
// their concatenation; the host-output tuples and status come back with one synchronisation
int launch_sample_multi(sassi_ctx* const* ctxs, const uint32_t* kernel, const uint32_t* invocation,
                        uint32_t n, uint32_t k, uint64_t seed, sassi_inj_site* host_out, cudaStream_t s) {
  std::vector<Prof> prof(n);
  for (uint32_t i = 0; i < n; ++i) {
    const uint64_t* P = nullptr;
    int rc = scan_counts(ctxs[i], s, &P);
    if (rc) return rc;
    prof[i] = Prof{P, 32ull * ctxs[i]->W, kernel[i], invocation[i]};
  }
  char* buf = nullptr;
  const size_t pb = ((sizeof(Prof) * n + 255) & ~size_t(255));
  SASSI_CUDA(cudaMallocAsync(reinterpret_cast<void**>(&buf), pb + sizeof(sassi_inj_site) * ((size_t)k + 1), s));
  Prof* d_prof = reinterpret_cast<Prof*>(buf);
  sassi_inj_site* d_out = reinterpret_cast<sassi_inj_site*>(buf + pb);
  uint32_t* d_flag = reinterpret_cast<uint32_t*>(d_out + k);
  SASSI_CUDA(cudaMemcpyAsync(d_prof, prof.data(), sizeof(Prof) * n, cudaMemcpyHostToDevice, s));
  const uint32_t warps = k ? k : 1u;
  draw_kernel<<<(warps + 7) / 8, 256, 0, s>>>(d_prof, n, Prof{}, k, seed, d_out, d_flag);
  SASSI_CUDA(cudaGetLastError());
  ctxs[0]->launches += 1;
  uint32_t h_flag = 0;
  SASSI_CUDA(cudaMemcpyAsync(&h_flag, d_flag, 4, cudaMemcpyDeviceToHost, s));
  if (k) SASSI_CUDA(cudaMemcpyAsync(host_out, d_out, sizeof(sassi_inj_site) * k, cudaMemcpyDeviceToHost, s));
  SASSI_CUDA(cudaFreeAsync(buf, s));
  SASSI_CUDA(cudaStreamSynchronize(s));
  if (h_flag)
    return set_error(SASSI_ESTATE, "no eligible dynamic instruction was counted: nothing to sample");
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
