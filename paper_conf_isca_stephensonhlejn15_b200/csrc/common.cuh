// common.cuh — internals shared by the libsassi.so translation units (never by the oracle).
#pragma once

#include <nvtx3/nvToolsExt.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include <string>
#include <vector>

#include "sassi.h"

namespace sassi {

// NVTX range around a public call (header-only nvtx3: no cost unless a profiler is attached)
struct NvtxRange {
  explicit NvtxRange(const char* m) { nvtxRangePushA(m); }
  ~NvtxRange() { nvtxRangePop(); }
  NvtxRange(const NvtxRange&) = delete;
  NvtxRange& operator=(const NvtxRange&) = delete;
};

constexpr uint32_t FULL = 0xFFFFFFFFu;
constexpr uint32_t EMPTY_KEY = 0xFFFFFFFFu;
constexpr int kConsumeThreads = 1024;         // 32 warps: one CTA per SM (see DESIGN 6.1)
constexpr int kWarpsPerCta = kConsumeThreads / 32;
constexpr uint64_t kMaxRecordsPerLaunch = 1ull << 29;  // 32-bit record / row indices in a launch
constexpr uint32_t kDynLocalLg = 9, kDynLocal = 1u << kDynLocalLg;  // per-CTA dynamic-pc cache slots
constexpr uint32_t kDynLocalWords = 4 * kDynLocal;                  // key + count (u32) + threads (u64)
constexpr uint32_t kMaxPeers = 7;   // fused merge over peer memory: up to 8 GPUs of one node
// error-flag bits (ctx->d_err, reported by sassi_read_tables): 4 = rows of a batch run past its
// chunk's rows or the index disagrees with the rows, 8 = chunk index outside the row buffers
// (both SASSI_EFORMAT); kMergeMismatch = a merge found other site tables (SASSI_EMISMATCH)
constexpr uint32_t kErrRows = 4u, kErrIndex = 8u, kMergeMismatch = 1u << 16;
// the context's error word, then kSchedSlots chunk schedulers of 2 words; consecutive fold launches
// take consecutive slots, so folds of one context on unordered streams (up to kSchedSlots in
// flight) never share one
constexpr uint32_t kSchedSlots = 64, kErrWords = 4 + 2 * kSchedSlots;

// Packed per-site info word in the hash (bit layout). The companion cidx word holds the
// site's compact branch-or-memdiv slot (low 16 bits) and compact value-site slot (high 16 bits).
constexpr uint32_t I_BRANCH = 1u << 0;        // COND_BRANCH site
constexpr uint32_t I_ADDR_ROW = 1u << 1;      // record carries an addr row (MEM, any domain)
constexpr uint32_t I_MEMDIV = 1u << 2;        // MEM && GLOBAL: folded by the memdiv handler
constexpr uint32_t I_ELIGIBLE = 1u << 3;      // instcount-eligible (R12)
constexpr uint32_t I_NDST_SHIFT = 4;          // 3 bits: n_gpr_dst
constexpr uint32_t I_VD0_SHIFT = 8;           // 16 bits: first value-destination state slot
constexpr uint32_t I_PCM = 1u << 24;          // memdiv site with a per-PC matrix ...
constexpr uint32_t I_PCM_SHIFT = 25;          // ... in slot (info >> 25) & 3

// Home slot of a pc in the site hash: multiplicative hash ((pc * mul) >> shr) & (cap - 1), its
// parameters chosen per site table at attach time (capi.cu choose_hash): for the dense pcs of a
// real kernel (one SASS instruction every 16 B) mul = 1, shr = 4 is collision-free.
__host__ __device__ __forceinline__ uint32_t pc_slot(uint32_t pc, uint32_t mul, uint32_t shr,
                                                     uint32_t cap) {
  return ((pc * mul) >> shr) & (cap - 1);
}

// Table image offsets (u64 words), same formulas as sassi_table_layout().
struct Offsets {
  uint64_t br, mem, val, ones, zeros, scalar, h32, h128, counts, mix, imix, pcsel, pcmat, total;
};

// Kernel parameter block of the fused consume kernel.
struct ConsumeParams {
  const uint4* hdr;                 // [n] headers (16 B each), this launch's first record first
  const uint64_t* addr;             // addr rows; row r at addr + 32 * (r - arow_base)
  const uint32_t* val;              // val rows;  row r at val + 32 * (r - vrow_base)
  const ulonglong2* cb;             // chunk index for the records of this launch
  uint32_t n;                       // records in this launch (hdr[0] starts a chunk)
  uint64_t arow_base, vrow_base;    // row index of addr[0] / val[0]
  uint64_t arow_end, vrow_end;      // one past the last valid row index (bounds check)
  const uint4* hash;                // [cap] {key, info, cidx, 0}
  uint32_t cap;                     // power of two
  uint32_t hmul, hshr;              // pc_slot parameters
  uint32_t nb, nm, nv, nvd;         // branch sites, memdiv sites, value sites, value (site,dst)s
  uint32_t pw;                      // private counter words per warp (16 B multiple)
  uint32_t priv;                    // 1: per-warp private counters; 0: one shared set + atomics
  uint32_t n_warps;                 // per-thread count coverage (32 * n_warps threads)
  const uint32_t* flush_b;          // [nb] site index of branch compact slot
  const uint32_t* flush_m;          // [nm] site index of memdiv compact slot
  const uint32_t* flush_v;          // [nv][3] site index, first value-dst slot, n_dst
  const uint32_t* flush_x;          // [S] Fig.3 category bits of each site (instruction mix)
  uint32_t S;                       // registered sites
  uint32_t px;                      // first private word of the per-site mix counters
  uint32_t npcm;                    // per-PC memdiv matrices kept (shared-memory copies)
  uint64_t* table;                  // device table image
  Offsets off;
  uint32_t* err;                    // error bits (bit 0: row index out of range ...)
  uint32_t* sched;                  // this launch's chunk scheduler {next claimed item, CTAs done}:
                                    // zero at launch, back to zero when the launch's last CTA exits
  uint32_t* dyn_keys;               // insert-on-miss table of unregistered pcs (0: disabled) ...
  unsigned long long* dyn_vals;     // ... [cap][2] warp / thread executions, then dropped records
  uint32_t dyn_cap, dyn_lg;         // slots (power of two) and log2
  unsigned long long* peers[kMaxPeers];  // fused merge: peers' table images (same layout) ...
  uint32_t n_peers;                 // ... that every flush atomic also goes to
  uint32_t gmode;                   // 1: global mode (site table beyond shared memory)
  uint32_t arow_bit;                // info bit of records with an address row in the stream:
                                    // I_ADDR_ROW (every MEM site), I_MEMDIV (GLOBAL-only rows)
};

// home slot of an unregistered pc in the dynamic table (Fibonacci hashing: dense pcs spread)
__host__ __device__ __forceinline__ uint32_t dyn_slot(uint32_t pc, uint32_t lg) {
  return (pc * 0x9E3779B1u) >> (32u - lg);
}

// Fig.4 l.21-23 "Create a new entry if one does not exist" for an unregistered pc: claim its slot
// with a CAS (linear probing), then add the counts; a full table (or the reserved pc) counts the
// records as dropped. (Not inlined: the consume kernel calls it only on the rare miss path.)
static __device__ __forceinline__ void dyn_insert(uint32_t pc, uint64_t nrec, uint64_t nthr, uint32_t* keys,
                                        unsigned long long* vals, uint32_t cap, uint32_t lg) {
  if (pc != EMPTY_KEY) {
    uint32_t slot = dyn_slot(pc, lg);
    for (uint32_t probe = 0; probe < cap; ++probe) {
      uint32_t k = *reinterpret_cast<volatile uint32_t*>(keys + slot);
      if (k == EMPTY_KEY) {
        k = atomicCAS(keys + slot, EMPTY_KEY, pc);
        if (k == EMPTY_KEY) k = pc;
      }
      if (k == pc) {
        atomicAdd(vals + 2 * slot, (unsigned long long)nrec);
        if (nthr) atomicAdd(vals + 2 * slot + 1, (unsigned long long)nthr);
        return;
      }
      slot = (slot + 1) & (cap - 1);
    }
  }
  atomicAdd(vals + 2 * cap, (unsigned long long)nrec);  // reserved pc or a full table: dropped
}


}  // namespace sassi

struct sassi_ctx {
  int device = 0;
  uint32_t S = 0, W = 0;
  uint32_t mask = 0;
  bool consumed = false;
  std::vector<sassi_site> sites;
  sassi::Offsets off{};
  uint64_t checksum = 0;
  // device state
  uint64_t* d_table = nullptr;
  uint4* d_hash = nullptr;          // [cap] {key, info, cidx, 0}
  std::vector<uint4> entries;       // per registered site {pc, info, cidx, 0} (host copy)
  uint32_t cap_base = 0;            // pow2 >= 2 * n_sites
  uint32_t hash_cap = 0;            // capacity of the table on the device
  uint32_t cap = 0;
  uint32_t hmul = 1, hshr = 4;      // pc_slot parameters of the table on the device
  uint32_t nb = 0, nm = 0, nv = 0, nvd = 0, pw = 0, priv = 1;
  uint32_t gmode = 0;               // site table beyond shared memory: hash / state / counters global
  uint32_t addr_global_only = 0;    // address row streams carry GLOBAL memory sites' rows only
  uint32_t pw_base = 0;             // private words of the branch / memdiv / value counters
  std::vector<uint32_t> mix_cat;    // per site: Fig.3 category bits (bit c = dynamic_instr_counts[c])
  uint32_t pcsel[4] = {0, 0, 0, 0}; // per-PC memdiv matrices: site index + 1 (0 = unused)
  uint32_t npcm = 0;
  uint64_t site_checksum = 0;       // of the registered sites (checksum adds the selection)
  uint32_t* d_flush = nullptr;      // flush_b | flush_m | flush_v
  uint32_t* d_err = nullptr;          // [kErrWords]: error bits, chunk schedulers
  uint64_t sched_seq = 0;             // fold launches so far (scheduler slot rotation)
  uint64_t* d_scan = nullptr;       // sampling: prefix [32W+1] + block sums
  uint64_t scan_words = 0;
  void* d_sample = nullptr;         // sampling: draws + status word of the host-output form
  uint64_t sample_bytes = 0;
  int num_sms = 0;
  int ctas_per_sm = 0;
  size_t smem_bytes = 0;
  void* launch_fn = nullptr;        // consume kernel last configured (attribute + occupancy) ...
  size_t launch_smem = 0;           // ... for this shared-memory size
  uint64_t launches = 0;
  uint64_t max_launch = 0;          // records per consume launch (kMaxRecordsPerLaunch unless lowered)
  // host-consume staging (lazily allocated)
  void* stage[2] = {nullptr, nullptr};
  size_t stage_bytes = 0;
  cudaStream_t copy_stream = nullptr;
  cudaEvent_t ev_copied[2] = {nullptr, nullptr};
  cudaEvent_t ev_used[2] = {nullptr, nullptr};
  // merge scratch
  uint64_t* d_pack = nullptr;
  uint64_t pack_words = 0;
  void* verified_comm = nullptr;     // communicator whose ranks were proven to hold this layout ...
  uint64_t verified_checksum = 0;   // ... for this checksum (sassi_merge's host-synchronised check)
  // dynamic sites: insert-on-miss table of unregistered pcs (sassi_enable_dynamic_pcs)
  uint32_t dyn_cap = 0, dyn_lg = 0;
  uint32_t* d_dyn_keys = nullptr;           // [dyn_cap]
  unsigned long long* d_dyn_vals = nullptr; // [2 dyn_cap + 1]
  void* d_dyn_gather = nullptr;             // merge: all ranks' keys and values
  size_t dyn_gather_bytes = 0;
  // fused merge over peer memory: peers' table images opened from CUDA IPC handles
  unsigned long long* peer_tables[sassi::kMaxPeers] = {};
  uint32_t n_peers = 0;
};

namespace sassi {

// error plumbing (capi.cu)
int set_error(int status, const std::string& msg);
int cuda_check(cudaError_t e, const char* what);
#define SASSI_CUDA(call)                                       \
  do {                                                         \
    cudaError_t _e = (call);                                   \
    if (_e != cudaSuccess) return ::sassi::cuda_check(_e, #call); \
  } while (0)

Offsets layout_offsets(uint32_t S, uint32_t W);

// kernels' host launchers
int launch_init_tables(sassi_ctx* c, cudaStream_t s);
int launch_consume(sassi_ctx* c, const ConsumeParams& p, cudaStream_t s);
int launch_index(sassi_ctx* c, const sassi_hdr* hdr, uint64_t n, sassi_chunk_base* out,
                 cudaStream_t s);
int launch_sample(sassi_ctx* c, uint32_t k, uint64_t seed, sassi_inj_site* host_out,
                  cudaStream_t s);
int launch_sample_device(sassi_ctx* c, uint32_t k, uint64_t seed, sassi_inj_site* dev_out,
                         uint32_t* dev_status, cudaStream_t s);
int launch_sample_multi(sassi_ctx* const* ctxs, const uint32_t* kernel, const uint32_t* invocation,
                        uint32_t n, uint32_t k, uint64_t seed, sassi_inj_site* host_out, cudaStream_t s);
int launch_merge(sassi_ctx* c, void* comm, cudaStream_t s);
int launch_merge_local(sassi_ctx* const* ctxs, uint32_t n, cudaStream_t s);
int consume_smem_bytes(const sassi_ctx* c, size_t* bytes);
int launch_dyn_reset(sassi_ctx* c, cudaStream_t s);

}  // namespace sassi
