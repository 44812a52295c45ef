// index.cu — sassi_index_records: build the chunk index (first addr / val row of every 256-record
// chunk) from device headers when the record producer did not emit it. Rows per record follow
// from the site of its pc (SRF1, include/sassi.h); unregistered pcs carry no rows.
#include "scan.cuh"

namespace sassi {
namespace {

// one warp per chunk: per-chunk addr-row and val-row counts
__global__ void __launch_bounds__(256) chunk_counts_kernel(const uint4* __restrict__ hdr, uint64_t n,
                                                           const uint4* __restrict__ hash,
                                                           uint32_t cap, uint32_t hmul, uint32_t hshr,
                                                           uint32_t arow_bit, uint64_t* na, uint64_t* nv) {
  const uint64_t c = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const uint32_t lane = threadIdx.x & 31;
  const uint64_t nch = (n + SASSI_CHUNK - 1) / SASSI_CHUNK;
  if (c >= nch) return;
  uint32_t a = 0, v = 0;
  for (uint32_t k = lane; k < SASSI_CHUNK; k += 32) {
    const uint64_t i = c * SASSI_CHUNK + k;
    if (i >= n) break;
    const uint32_t pc = hdr[i].x;
    uint32_t slot = pc_slot(pc, hmul, hshr, cap);
    for (;;) {
      const uint4 e = hash[slot];
      const uint32_t key = e.x;
      if (key == pc) {
        const uint32_t inf = e.y;
        a += (inf & arow_bit) ? 1u : 0u;  // I_ADDR_ROW, or I_MEMDIV for GLOBAL-only address rows
        v += (inf >> I_NDST_SHIFT) & 7u;
        break;
      }
      if (key == EMPTY_KEY) break;
      slot = (slot + 1) & (cap - 1);
    }
  }
  a = __reduce_add_sync(FULL, a);
  v = __reduce_add_sync(FULL, v);
  if (lane == 0) {
    na[c] = a;
    nv[c] = v;
  }
}

__global__ void interleave_kernel(const uint64_t* __restrict__ Pa, const uint64_t* __restrict__ Pv,
                                  uint64_t m, ulonglong2* out) {
  const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < m) out[i] = make_ulonglong2(Pa[i], Pv[i]);
}

}  // namespace

int launch_index(sassi_ctx* c, const sassi_hdr* hdr, uint64_t n, sassi_chunk_base* out,
                 cudaStream_t s) {
  const uint64_t nch = (n + SASSI_CHUNK - 1) / SASSI_CHUNK;
  const uint64_t sw = scan_scratch_words(nch);
  uint64_t* buf = nullptr;
  const uint64_t words = 2 * nch + 2 * (nch + 1) + sw;
  SASSI_CUDA(cudaMallocAsync(&buf, 8 * (words ? words : 1), s));
  uint64_t *na = buf, *nv = buf + nch, *Pa = nv + nch, *Pv = Pa + nch + 1, *scratch = Pv + nch + 1;
  if (nch) {
    chunk_counts_kernel<<<(unsigned)((nch * 32 + 255) / 256), 256, 0, s>>>(
        reinterpret_cast<const uint4*>(hdr), n, c->d_hash, c->cap, c->hmul, c->hshr,
        c->addr_global_only ? I_MEMDIV : I_ADDR_ROW, na, nv);
    SASSI_CUDA(cudaGetLastError());
  }
  int rc = scan_u64(na, nch, Pa, scratch, s);
  if (!rc) rc = scan_u64(nv, nch, Pv, scratch, s);
  if (!rc) {
    interleave_kernel<<<(unsigned)((nch + 1 + 255) / 256), 256, 0, s>>>(
        Pa, Pv, nch + 1, reinterpret_cast<ulonglong2*>(out));
    SASSI_CUDA(cudaGetLastError());
  }
  cudaFreeAsync(buf, s);
  c->launches += nch ? 6 : 1;  // counts + 2 scans x 2 + interleave
  return rc;
}

}  // namespace sassi
