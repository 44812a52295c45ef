// consume.cu — the fused SASSI handler fold over warp-instruction records (sm_100a).
//
// One launch streams headers (16 B) + only the payload rows the attached handlers need, and folds
// them into per-CTA shared-memory partial tables keyed by an open-addressed per-PC hash, flushed
// to the global u64 table image at CTA exit. Handlers (PAPER.md = /root/reference/PAPER.md):
//   branch     Fig.4 (L237-L243)   lane-per-record: popc of active / taken masks
//   memdiv     Fig.6 (L361-L369)   warp-per-row: distinct 32 B sectors and 128 B lines among the
//                                  guard-true lanes; window-bitmap REDUX fast path, warp sort otherwise
//   value      Fig.9 (L549-L563)   row-per-lane: a batch's contiguous value rows are bulk-copied
//                                  (TMA, cp.async.bulk + mbarrier) into the warp's shared-memory
//                                  buffer; lane j folds row j's 32 values (AND / OR of the written
//                                  lanes) -> constantOnes / constantZeros / isScalar
//   instcount  §8.1 (L625-L627)    lane-per-record: 32x32 bit-matrix transpose + popc gives the
//                                  per-lane count of 32 records; register accumulator per trace warp
//   instmix    Fig.3 (L193-L199)   lane-per-record: popc(active) into a per-site counter; the seven
//                                  category totals are formed at the flush
// Work split: a warp owns one 256-record chunk at a time (chunk_base gives its row offsets) and walks
// it in 8 batches of 32 records; row indices inside a batch come from ballot prefix sums.
#include <map>
#include <mutex>
#include <utility>

#include "common.cuh"

#ifndef SASSI_HDR_DEPTH
#define SASSI_HDR_DEPTH 3  // header batches in flight per warp (header-only handler sets)
#endif
#ifndef SASSI_ROW_GROUP
#define SASSI_ROW_GROUP 3  // memdiv address rows loaded per group (measured: 3 beats 2, 4, 6)
#endif
#ifndef SASSI_HASH_LG
#define SASSI_HASH_LG 12     // memdiv distinctness check: 2^12 bit buckets per warp (512 B)
#endif
#ifndef SASSI_PREF_ROWS
#define SASSI_PREF_ROWS 6  // memdiv: address rows of the next batch prefetched into L2 (0: off)
#endif
#ifndef SASSI_SPLIT_PARTS
#define SASSI_SPLIT_PARTS 2  // the launch's last chunks are folded in this many parts
#endif
#ifndef SASSI_DYN_ROUNDS
#define SASSI_DYN_ROUNDS 16  // payload folds: the last 16 rounds of chunks claimed dynamically
#endif
#ifndef SASSI_HASH_ROUNDS
#define SASSI_HASH_ROUNDS 2  // hash rounds (different multipliers) before the exact sort
#endif

#ifdef SASSI_TIMELINE  // development builds: per-warp %globaltimer stamps of the last launch
__device__ unsigned long long g_timeline[4 * 148 * 32 * 4];
extern "C" int sassi_debug_timeline(void* host, size_t bytes) {
  return (int)cudaMemcpyFromSymbol(host, g_timeline, bytes);
}
#define SASSI_STAMP(k, v)                                                                      \
  if ((tid & 31u) == 0 && blockIdx.x * 32 + (tid >> 5) < 4 * 148 * 32)                            \
    g_timeline[4 * (blockIdx.x * 32 + (tid >> 5)) + (k)] = (v);
__device__ __forceinline__ unsigned long long gtime() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}
#else
#define SASSI_STAMP(k, v)
#endif

namespace sassi {
namespace {

__device__ __forceinline__ uint4 ld_nc_v4(const uint4* p) {
  uint4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0, %1, %2, %3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
               : "l"(p));
  return r;
}
__device__ __forceinline__ uint64_t ld_nc_u64(const uint64_t* p) {
  uint64_t r;
  asm volatile("ld.global.nc.L1::no_allocate.u64 %0, [%1];" : "=l"(r) : "l"(p));
  return r;
}
// 32x32 bit-matrix transpose across the warp: in, lane i holds row i; out, lane l holds the word
// whose bit i is bit l of row i. Five butterfly stages swapping off-diagonal blocks: per stage the
// lane keeps its own half (mask `keep`) and takes the partner's other half, brought into place by
// one rotate (right by J in the upper lane of a pair, left by J in the lower: the wrapped bits fall
// outside the taken half). The rotate form issues fewer instructions but holds more registers: the
// header-only kernels use it, the payload kernels (register-capped at 64) the shift form.
template <bool kRotate>
__device__ __forceinline__ uint32_t transpose32(uint32_t x, uint32_t lane) {
  const uint32_t m16 = 0x0000FFFFu, m8 = 0x00FF00FFu, m4 = 0x0F0F0F0Fu, m2 = 0x33333333u,
                 m1 = 0x55555555u;
#define SASSI_TSTAGE(J, M)                                                           \
  {                                                                                  \
    const uint32_t y = __shfl_xor_sync(FULL, x, J);                                  \
    const bool hi = (lane & J) != 0;                                                 \
    if (kRotate) {                                                                   \
      const uint32_t keep = hi ? ~M : M;                                             \
      x = (x & keep) | (__funnelshift_r(y, y, hi ? J : 32u - J) & ~keep);            \
    } else {                                                                         \
      x = hi ? ((x & ~M) | ((y >> J) & M)) : ((x & M) | ((y << J) & ~M));            \
    }                                                                                \
  }
  SASSI_TSTAGE(16, m16)
  SASSI_TSTAGE(8, m8)
  SASSI_TSTAGE(4, m4)
  SASSI_TSTAGE(2, m2)
  SASSI_TSTAGE(1, m1)
#undef SASSI_TSTAGE
  return x;
}

// Bitonic sort of one key per lane across the warp (ascending in lane order), in the "flip" form:
// each merge of blocks of k starts by comparing lane i with lane i ^ (k - 1) (the reversed partner)
// and continues with i ^ j; in every step the lower lane of a pair keeps the minimum, so a lane's
// direction is one of its five index bits (no per-step direction arithmetic: 2 ALU ops a step).
template <typename T>
__device__ __forceinline__ T warp_sort(T v, uint32_t lane) {
#pragma unroll
  for (uint32_t k = 2; k <= 32; k <<= 1) {
    {
      const T o = __shfl_xor_sync(FULL, v, k - 1);
      const bool lower = (lane & (k >> 1)) == 0;
      v = lower ? (o < v ? o : v) : (o > v ? o : v);
    }
#pragma unroll
    for (uint32_t j = k >> 2; j > 0; j >>= 1) {
      const T o = __shfl_xor_sync(FULL, v, j);
      const bool lower = (lane & j) == 0;
      v = lower ? (o < v ? o : v) : (o > v ? o : v);
    }
  }
  return v;
}

// {distinct sectors, distinct lines} of one row from its sorted sector keys (lanes outside G sort
// last): the positions < n whose key differs from the previous one.
template <typename T>
__device__ __forceinline__ void count_sorted(T v, uint32_t n, uint32_t lane, uint32_t* out_s,
                                             uint32_t* out_l) {
  const T pv = __shfl_up_sync(FULL, v, 1);
  const bool new_s = lane < n && (lane == 0 || v != pv);
  const bool new_l = lane < n && (lane == 0 || (v >> 2) != (pv >> 2));
  *out_s = __popc(__ballot_sync(FULL, new_s));
  *out_l = __popc(__ballot_sync(FULL, new_l));
}

// One round of the distinctness check of a gather row: every lane of G sets bit h(line) of the
// warp's 2^SASSI_HASH_LG-bit shared-memory bitmap with an atomic OR that returns the old word. If
// no lane finds its bit already set, the lines of G hash to pairwise different buckets, so they
// are pairwise distinct (equal lines hash alike). The lanes then clear their words again.
__device__ __forceinline__ bool lines_distinct(uint32_t line, bool in, uint32_t* bm, uint32_t mul) {
  const uint32_t h = (line * mul) >> (32 - SASSI_HASH_LG);
  const uint32_t w = (uint32_t)__cvta_generic_to_shared(bm) + 4u * (h >> 5);
  const uint32_t bit = 1u << (h & 31u);
  uint32_t old;
  // predicated shared atomic / store (no branch around them)
  asm volatile("{ .reg .pred q; setp.ne.u32 q, %1, 0; mov.u32 %0, 0; @q atom.shared.or.b32 %0, [%2], %3; }"
               : "=r"(old) : "r"((uint32_t)in), "r"(w), "r"(bit) : "memory");
  const bool ok = !__any_sync(FULL, (old & bit) != 0u);
  __syncwarp();
  asm volatile("{ .reg .pred q; setp.ne.u32 q, %0, 0; @q st.shared.u32 [%1], %2; }"
               :: "r"((uint32_t)in), "r"(w), "r"(0u) : "memory");
  __syncwarp();
  return ok;
}

// Fig.6 for one warp-wide address row: n = |G|, s = distinct (addr >> 5), L = distinct (addr >> 7)
// over the lanes of G (the count of Fig.6's leader-election loop, l.16-26).
//  - window path: every sector of G within the 32-sector (1 KB, 8-line) window that starts at the
//    line holding the lowest sector (same high word): the window bitmap is OR-reduced across the
//    warp (REDUX), s = its popcount, L = the popcount of its nibbles OR-folded (a nibble = a line).
//  - otherwise (gathers): if a hashed bitmap shows the lines of G to be pairwise distinct,
//    s = L = |G| (lines_distinct, two rounds); else, when all high words agree, sort the 32-bit
//    keys across the warp (bitonic) with the
//    lanes outside G padded to the maximum so they sort last, and count positions < n whose key
//    differs from the previous one; lines come from the same sorted sectors (>> 2 keeps order).
//  - rows whose sectors differ in the high word return false and go to memdiv_row64 (64-bit keys),
//    called once per such row outside the unrolled row loop to keep that loop's code small.
__device__ __forceinline__ bool memdiv_row32(uint64_t a, uint32_t G, uint32_t lane, uint32_t* bm,
                                             uint32_t* out_s, uint32_t* out_l) {
  const bool in = (G >> lane) & 1u;
  const uint64_t sec = a >> 5;
  const uint32_t slo = (uint32_t)sec, shi = (uint32_t)(sec >> 32);
  const uint32_t bhi = __reduce_max_sync(FULL, in ? shi : 0u);
  const uint32_t base = __reduce_min_sync(FULL, in ? slo : FULL) & ~3u;  // line-aligned
  const uint32_t e = slo - base;  // window position, valid when < 32 and high words agree
  const bool same_hi = !in || shi == bhi;
  if (__all_sync(FULL, same_hi && (!in || e < 32u))) {
    const uint32_t m = __reduce_or_sync(FULL, in ? (1u << e) : 0u);
    *out_s = __popc(m);
    const uint32_t t = m | (m >> 2);
    *out_l = __popc((t | (t >> 1)) & 0x11111111u);
    return true;
  }
  // scattered rows (gathers): if the lines of G are pairwise distinct, so are the sectors, and
  // s = L = |G| with no sort; a hash collision or a repeated line falls through to the sort. The
  // keys are the lines' low 30 bits: equal lines give equal keys, so distinct keys prove distinct
  // lines whatever the high words (no uniformity check needed before the hash)
  if (SASSI_HASH_ROUNDS >= 1 && lines_distinct(slo >> 2, in, bm, 0x9E3779B1u)) {
    *out_s = *out_l = __popc(G);
    return true;
  }
  if (SASSI_HASH_ROUNDS >= 2 && lines_distinct(slo >> 2, in, bm, 0x85EBCA6Bu)) {
    *out_s = *out_l = __popc(G);
    return true;
  }
  if (!__all_sync(FULL, same_hi)) return false;
  count_sorted(warp_sort<uint32_t>(in ? slo : FULL, lane), __popc(G), lane, out_s, out_l);
  return true;
}

__device__ __forceinline__ void memdiv_row64(uint64_t a, uint32_t G, uint32_t lane, uint32_t* out_s,
                                             uint32_t* out_l) {
  const bool in = (G >> lane) & 1u;
  count_sorted(warp_sort<uint64_t>(in ? (a >> 5) : ~0ull, lane), __popc(G), lane, out_s, out_l);
}

// ---- TMA bulk copy global -> shared with an mbarrier (cp.async.bulk, SASS UBLKCP) ----
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}
__device__ __forceinline__ void bulk_load(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // prior generic reads of dst done
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)),
               "r"(bytes) : "memory");
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}
// Wait for phase `parity` of the barrier; bounded so a broken stream traps instead of hanging.
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  uint32_t done = 0;
  for (uint32_t spin = 0;; ++spin) {
    asm volatile(
        "{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
        : "=r"(done)
        : "r"(smem_u32(bar)), "r"(parity)
        : "memory");
    if (done) return;
    if (spin > (1u << 28)) __trap();
  }
}

// Per-record counter update into the warp's private counter words: shared-memory atomics
// (lanes whose records hit the same site in one batch — short loop bodies — add correctly, and
// no duplicate detection is needed; a MATCH.ANY-guarded plain read-modify-write measured slower).
__device__ __forceinline__ void add_counters4(bool pred, uint32_t off, uint4 v, uint32_t* region) {
  if (pred) {
    atomicAdd(region + off, v.x);
    atomicAdd(region + off + 1, v.y);
    atomicAdd(region + off + 2, v.z);
    if (v.w) atomicAdd(region + off + 3, v.w);
  }
}

__device__ __forceinline__ void add_counters2(bool pred, uint32_t off, uint2 v, uint32_t* region) {
  if (pred) {
    atomicAdd(region + off, v.x);
    atomicAdd(region + off + 1, v.y);
  }
}

// Shared-memory layout (u32 words) for handler set H: only the regions the attached handlers use,
// fixed-size regions first so their offsets are compile-time constants.
constexpr uint32_t kVbufWords = 1024;  // 4 KB of value rows per warp
template <uint32_t H>
struct SmLayout {
  static constexpr bool kMem = (H & SASSI_H_MEMDIV) != 0, kVal = (H & SASSI_H_VALUE) != 0;
  static constexpr uint32_t kDiag = 0;                                  // 8 u32
  static constexpr uint32_t kImix = 8;                                  // 8 u64 (instmix totals)
  static constexpr uint32_t kSlot = 24;                                 // [warps] u32 (claimed items)
  static constexpr uint32_t kH32 = kSlot + kWarpsPerCta;                // [32][32] u32 (memdiv)
  static constexpr uint32_t kH128 = kH32 + 1024;                        // [32][32] u32 (memdiv)
  static constexpr uint32_t kHbm = kH128 + 1024;  // [warps][2^LG / 32] distinctness bitmaps
  static constexpr uint32_t kHbmWords = SASSI_HASH_ROUNDS ? (1u << SASSI_HASH_LG) / 32 : 0u;
  static constexpr uint32_t kBar = kMem ? kHbm + kWarpsPerCta * kHbmWords : kH32;
  static constexpr uint32_t kVbuf = kVal ? ((kBar + 2 * kWarpsPerCta + 31) & ~31u) : kBar;
  static constexpr uint32_t kVar = kVbuf + (kVal ? kWarpsPerCta * kVbufWords : 0u);  // hash, ...
  static_assert(kVbuf % 32 == 0 || !kVal, "value buffers must be 128 B aligned");
  static_assert(kVar % 4 == 0 && kBar % 2 == 0, "alignment");
};
// host mirror of SmLayout<H>::kVar
uint32_t sm_var_words(uint32_t H) {
  const bool mem = H & SASSI_H_MEMDIV, val = H & SASSI_H_VALUE;
  const uint32_t hbm = SASSI_HASH_ROUNDS ? (1u << SASSI_HASH_LG) / 32 : 0u;
  const uint32_t bar = mem ? 24 + kWarpsPerCta + 2048 + kWarpsPerCta * hbm : 24 + kWarpsPerCta;
  const uint32_t vbuf = val ? ((bar + 2 * kWarpsPerCta + 31) & ~31u) : bar;
  return vbuf + (val ? kWarpsPerCta * kVbufWords : 0u);
}

// Row offsets at record r0 of a chunk (the start of one of its parts, r0 a multiple of 32 below
// the chunk's record count): the address / value rows of records [0, r0), from their pcs' info
// words (no handler runs on them). Out of line: it runs only for the launch's last items.
__device__ __noinline__ uint2 part_offsets(const uint4* hchunk, uint32_t r0, uint32_t lane,
                                           const uint4* tbl, uint32_t cap, uint32_t hmul, uint32_t hshr,
                                           uint32_t arow_bit) {
  uint32_t arow = 0, vrow = 0;
  for (uint32_t i = lane; i < r0; i += 32) {
    const uint4 h = ld_nc_v4(hchunk + i);
    uint32_t slot = pc_slot(h.x, hmul, hshr, cap);
    uint4 e = tbl[slot];
    while (e.x != h.x && e.x != EMPTY_KEY) {
      slot = (slot + 1) & (cap - 1);
      e = tbl[slot];
    }
    const uint32_t info = (e.x == h.x && h.x != EMPTY_KEY) ? e.y : 0u;
    arow += __popc(__ballot_sync(FULL, info & arow_bit));
    vrow += __reduce_add_sync(FULL, (info >> I_NDST_SHIFT) & 7u);
  }
  return make_uint2(arow, vrow);
}

// kExt: the extended instantiation, used when the insert-on-miss table of unregistered pcs is
// enabled (p.dyn_cap), the flush also updates peers' images (p.n_peers), and / or the site table
// does not fit shared memory (p.gmode: the "global mode" below); the plain kernels carry none of it.
// Global mode (site tables beyond one SM's shared memory, up to SASSI_MAX_SITES): the pc hash is
// read from global memory (L1 / L2 resident), each record's counters are added straight to the u64
// table image with device atomics (Fig.4 / Fig.9's own atomicAdd / atomicAnd into a device-global
// table, L239 / L595), and the value state is ANDed into the image's constantOnes / constantZeros /
// isScalar words when a bit changes; only the 32x32 matrices stay in shared memory.
template <uint32_t H, bool kExt>
__global__ void __launch_bounds__(kConsumeThreads, 1) consume_kernel(const ConsumeParams p) {
  extern __shared__ __align__(128) uint32_t sm[];
  using Ly = SmLayout<H>;
  constexpr uint32_t kSmDiag = Ly::kDiag, kSmImix = Ly::kImix, kSmH32 = Ly::kH32, kSmH128 = Ly::kH128,
                     kSmBar = Ly::kBar, kSmVbuf = Ly::kVbuf, kSmVar = Ly::kVar;
  constexpr uint32_t kCounters = SASSI_H_BRANCH | SASSI_H_MEMDIV | SASSI_H_VALUE | SASSI_H_INSTMIX;
  const uint32_t cap = p.cap;
  const bool gm = kExt && p.gmode;  // global mode: no hash, value state or counters in smem
  const uint32_t scap = gm ? 0u : cap;
  uint4* s_hash = reinterpret_cast<uint4*>(sm + kSmVar);            // [cap] {key, info, cidx, -}
  uint4* s_vstate = s_hash + scap;                                  // [nvd] ones, zeros, isScalar
  uint32_t* s_priv = reinterpret_cast<uint32_t*>(s_vstate + (Ly::kVal && !gm ? p.nvd : 0u));  // counters
  // [npcm][32][32] per-PC matrices (the private counters exist only for handler sets that count)
  uint32_t* s_pcm = s_priv + ((H & kCounters) && !gm ? (p.priv ? kWarpsPerCta : 1u) * p.pw : 0u);
  // dynamic sites: a per-CTA insert-on-miss cache of unregistered pcs (keys, record counts, thread
  // counts), flushed into the global table at CTA exit
  uint32_t* const s_dkey = s_pcm + 1024 * p.npcm;
  uint32_t* const s_dcnt = s_dkey + kDynLocal;
  unsigned long long* const s_dthr = reinterpret_cast<unsigned long long*>(s_dcnt + kDynLocal);
  const uint32_t n_regions = p.priv ? kWarpsPerCta : 1u;

  const uint32_t tid = threadIdx.x;
  SASSI_STAMP(0, gtime())
  for (uint32_t i = tid; i < scap; i += blockDim.x) s_hash[i] = p.hash[i];
  if (Ly::kVal && !gm)
    for (uint32_t i = tid; i < p.nvd; i += blockDim.x) s_vstate[i] = make_uint4(FULL, FULL, 1u, 0u);
  if ((H & kCounters) && !gm)
    for (uint32_t i = tid; i < n_regions * p.pw; i += blockDim.x) s_priv[i] = 0;
  for (uint32_t i = tid; i < kSmBar; i += blockDim.x) sm[i] = 0;  // diag (+ matrices)
  if (H & SASSI_H_MEMDIV)
    for (uint32_t i = tid; i < 1024 * p.npcm; i += blockDim.x) s_pcm[i] = 0;
  if (kExt && p.dyn_cap)
    for (uint32_t i = tid; i < kDynLocal; i += blockDim.x) {
      s_dkey[i] = EMPTY_KEY;
      s_dcnt[i] = 0;
      s_dthr[i] = 0;
    }
  if (Ly::kVal && tid < kWarpsPerCta) mbar_init(reinterpret_cast<uint64_t*>(sm + kSmBar) + tid, 1);
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  __syncthreads();

  SASSI_STAMP(1, gtime())
  const uint32_t lane = tid & 31u, wib = tid >> 5;
  const uint32_t lt = (1u << lane) - 1u;
  uint32_t* const wpriv = s_priv + (p.priv ? wib * p.pw : 0u);
  uint4* const vbuf = reinterpret_cast<uint4*>(sm + kSmVbuf + wib * kVbufWords);
  uint64_t* const vbar = reinterpret_cast<uint64_t*>(sm + kSmBar) + wib;
  uint32_t* const hbm = sm + Ly::kHbm + wib * Ly::kHbmWords;  // this warp's distinctness bitmap
  uint32_t vphase = 0;
  const uint32_t PB = 4 * p.nb, PV = 4 * p.nb + 4 * p.nm;
  const uint32_t n_units = (p.n + SASSI_CHUNK - 1) / SASSI_CHUNK;
  const uint32_t nw = gridDim.x * kWarpsPerCta;
  uint32_t c_rec = 0, c_inv = 0, c_unk = 0, c_bad = 0;
  uint32_t acc = 0, acc_w = FULL;  // per-thread-count accumulator of trace warp acc_w, lane = lane
  // vertical (bit-sliced) counters: lane r's bit l of plane k is bit k of the number of batches in
  // which lane r's record had lane l eligible (records of trace warp acc_w only); transposed and
  // folded into acc every 15 batches, so most batches cost 7 LOPs instead of a 32x32 transpose.
  // Only for handler sets without payload rows: with them, the 4 extra registers cost more than
  // the transposes they save (measured: c3 2.90 -> 3.06 ms)
  constexpr bool kVertical = !(H & (SASSI_H_MEMDIV | SASSI_H_VALUE));
  // (flushed every 5 iterations of the 3-batch header loop, and whenever the accumulator moves)
  uint32_t vp0 = 0, vp1 = 0, vp2 = 0, vp3 = 0;
  auto flush_planes = [&]() {
    if (__any_sync(FULL, (vp0 | vp1 | vp2 | vp3) != 0)) {
      acc += __popc(transpose32<true>(vp0, lane)) + 2 * __popc(transpose32<true>(vp1, lane)) +
             4 * __popc(transpose32<true>(vp2, lane)) + 8 * __popc(transpose32<true>(vp3, lane));
      vp0 = vp1 = vp2 = vp3 = 0;
    }
  };
  uint32_t err = 0;
  unsigned long long* const table = reinterpret_cast<unsigned long long*>(p.table);
  // every table update goes to this context's image and to the peers' (fused merge: the atomics
  // travel over NVLink to the other GPUs' images, so no collective runs after the fold)
  // (peer images live on other GPUs: system-scope atomics, atom.sys, so that updates from several
  // GPUs to one word are atomic with each other; the own image keeps device scope)
  auto gadd = [&](uint64_t off, unsigned long long v) {
    atomicAdd(table + off, v);
    if (kExt)
      for (uint32_t j = 0; j < p.n_peers; ++j) atomicAdd_system(p.peers[j] + off, v);
  };
  auto gand = [&](uint64_t off, unsigned long long v) {
    atomicAnd(table + off, v);
    if (kExt)
      for (uint32_t j = 0; j < p.n_peers; ++j) atomicAnd_system(p.peers[j] + off, v);
  };

  // global mode: this lane's record adds v.x.. to the u64 words base + 0.. of the image
  auto gcount4 = [&](bool pred, uint64_t base, uint4 v) {
    if (pred) {
      gadd(base, (unsigned long long)v.x);
      if (v.y) gadd(base + 1, (unsigned long long)v.y);
      if (v.z) gadd(base + 2, (unsigned long long)v.z);
      if (v.w) gadd(base + 3, (unsigned long long)v.w);
    }
  };
  unsigned long long g_imix[7] = {0, 0, 0, 0, 0, 0, 0};  // global mode: Fig.3 totals of this warp

  // ---- find(pc): open-addressed, linear probing, one 16-byte slot per probe (L239). Returns the
  // slot {key, info, cidx, site}; `known` = a registered site (0xFFFFFFFF is never registered) ----
  // h is always a real header of the stream (loads are clamped), so the probe needs no guard;
  // records are counted per chunk / range (c_rec), not here
  auto lookup = [&](const uint4& h, bool valid, bool& known) -> uint4 {
    uint32_t slot = pc_slot(h.x, p.hmul, p.hshr, cap);
    uint4 e = gm ? __ldg(p.hash + slot) : s_hash[slot];
    while (e.x != h.x && e.x != EMPTY_KEY) {  // collision: linear probing (load <= 1/2, rare)
      slot = (slot + 1) & (cap - 1);
      e = gm ? __ldg(p.hash + slot) : s_hash[slot];
    }
    known = valid && e.x == h.x && h.x != EMPTY_KEY;
    c_unk += valid && !known;
    c_inv += known && h.z == 0;
    if (kExt && p.dyn_cap) {  // dynamic sites: each lane adds its own unregistered record to the CTA's cache
      if (valid && !known) {
        bool done = false;
        if (h.x != EMPTY_KEY) {
          uint32_t slot = dyn_slot(h.x, kDynLocalLg);
          for (uint32_t probe = 0; probe < 8 && !done; ++probe) {
            uint32_t k = *reinterpret_cast<volatile uint32_t*>(s_dkey + slot);
            if (k == EMPTY_KEY) {
              k = atomicCAS(s_dkey + slot, EMPTY_KEY, h.x);
              if (k == EMPTY_KEY) k = h.x;
            }
            if (k == h.x) {
              atomicAdd(s_dcnt + slot, 1u);
              if (h.z) atomicAdd(s_dthr + slot, (unsigned long long)__popc(h.z));
              done = true;
            }
            slot = (slot + 1) & (kDynLocal - 1);
          }
        }
        // a long probe or the reserved pc: the global table (Fig.4 l.21-23's device-wide table)
        if (!done) dyn_insert(h.x, 1, (uint32_t)__popc(h.z), p.dyn_keys, p.dyn_vals, p.dyn_cap, p.dyn_lg);
      }
    }
    return e;
  };
  // ---- the handlers that read only the header: branch (Fig.4), instruction mix (Fig.3),
  // per-thread counts (§8.1) ----
  auto header_handlers = [&](const uint4& h, uint32_t info, uint32_t cidx, uint32_t site, bool live,
                             uint32_t G) {
    const uint32_t act = h.z;
    // ---- Case study I: branch divergence (Fig.4) ----
    if (H & SASSI_H_BRANCH) {
      const bool isb = live && (info & I_BRANCH);
      const uint32_t na = __popc(act), nt = __popc(G);
      const uint32_t dv = (G != 0 && G != act) ? 1u : 0u;
      if (gm) {
        if (isb) {
          gadd(p.off.br + 5ull * site, 1ull);
          gadd(p.off.br + 5ull * site + 1, (unsigned long long)na);
          if (nt) gadd(p.off.br + 5ull * site + 2, (unsigned long long)nt);
          if (na - nt) gadd(p.off.br + 5ull * site + 3, (unsigned long long)(na - nt));
          if (dv) gadd(p.off.br + 5ull * site + 4, 1ull);
        }
      } else {
        add_counters4(isb, 4 * (cidx & 0xFFFFu), make_uint4(1u, na, nt, dv), wpriv);
      }
    }
    // ---- Fig.3 instruction mix (L193-L199): every active thread counts; per-site thread
    // executions here, the seven category totals at the flush (R22) ----
    if ((H & SASSI_H_INSTMIX) && !gm && live) atomicAdd(wpriv + p.px + site, (uint32_t)__popc(act));
    if ((H & SASSI_H_INSTMIX) && gm) {  // global mode: the site's word and the categories per batch
      const uint32_t np = live ? (uint32_t)__popc(act) : 0u;
      if (np) gadd(p.off.mix + site, (unsigned long long)np);
      const uint32_t cat = live ? __ldg(p.flush_x + site) : 0u;
#pragma unroll
      for (uint32_t k = 0; k < 7; ++k) g_imix[k] += __reduce_add_sync(FULL, ((cat >> k) & 1u) ? np : 0u);
    }
    // ---- Case study IV: per-thread eligible dynamic-instruction counts (§8.1) ----
    if (H & SASSI_H_INSTCOUNT) {
      uint32_t E = (live && (info & I_ELIGIBLE)) ? G : 0u;
      auto drop_bad_warps = [&]() {  // records of warps outside the counts (n_bad_warp)
        if (E != 0 && h.y >= p.n_warps) {
          ++c_bad;
          E = 0;
        }
      };
      uint32_t pend;
      if (kVertical) {
        // the usual case in a warp-major stream: every eligible lane is on the accumulator's trace
        // warp (a checked one: acc_w != FULL) -> add E into the vertical counters; one vote decides
        // it, and only the other path needs the warp-range check
        if (acc_w != FULL && !__any_sync(FULL, E != 0 && h.y != acc_w)) {
          const uint32_t k0 = vp0 & E;
          vp0 ^= E;
          const uint32_t k1 = vp1 & k0;
          vp1 ^= k0;
          const uint32_t k2 = vp2 & k1;
          vp2 ^= k1;
          vp3 ^= k2;  // at most 15 additions between flushes: no carry out of plane 3
          pend = 0;
        } else {
          drop_bad_warps();
          flush_planes();
          pend = __ballot_sync(FULL, E != 0);
        }
      } else {
        drop_bad_warps();
        pend = __ballot_sync(FULL, E != 0);
      }
      while (pend) {
        const uint32_t w0 = __shfl_sync(FULL, h.y, __ffs(pend) - 1);
        const bool mine = E != 0 && h.y == w0;
        const uint32_t cnt = __popc(transpose32<kVertical>(mine ? E : 0u, lane));
        if (w0 != acc_w) {
          if (acc_w != FULL && acc)
            gadd(p.off.counts + 32ull * acc_w + lane, (unsigned long long)acc);
          acc_w = w0;
          acc = 0;
        }
        acc += cnt;
        pend &= ~__ballot_sync(FULL, mine);
        if (mine) E = 0;
      }
    }
  };

  constexpr bool kUnitRows = (H & (SASSI_H_MEMDIV | SASSI_H_VALUE)) != 0;
  if (!kUnitRows) {
    // ---- header-only handler sets: each warp takes one contiguous range of records (so its
    // per-thread-count accumulator stays on one trace warp for thousands of records) and walks it
    // in 32-record batches, headers loaded kDepth batches ahead ----
    constexpr uint32_t kDepth = SASSI_HDR_DEPTH;
    const uint32_t per = (p.n + 32u * nw - 1u) / (32u * nw) * 32u;  // records per warp
    const uint32_t R0 = min((blockIdx.x * kWarpsPerCta + wib) * per, p.n), R1 = min(R0 + per, p.n);
    if (lane == 0) c_rec += R1 - R0;
    auto first_rec = [&](uint32_t t) -> uint32_t { return R0 + 32u * t; };
    auto hload = [&](uint32_t r0) -> uint4 {
      return r0 < R1 ? ld_nc_v4(p.hdr + min(r0 + lane, R1 - 1u)) : make_uint4(0u, 0u, 0u, 0u);
    };
    uint4 q[kDepth];
#pragma unroll
    for (uint32_t k = 0; k < kDepth; ++k) q[k] = hload(first_rec(k));
    uint32_t it = 0;  // iterations since the vertical counters were last folded
    for (uint32_t t = 0;; t += kDepth) {
      // fold every floor(15 / kDepth) iterations: <= 15 additions between folds
      if ((H & SASSI_H_INSTCOUNT) && kVertical && ++it == 15 / kDepth + 1) {
        flush_planes();
        it = 1;
      }
      bool done = false;
#pragma unroll
      for (uint32_t k = 0; k < kDepth; ++k) {
        const uint32_t r0 = first_rec(t + k);
        if (r0 >= R1) {
          done = true;
          break;
        }
        const uint4 h = q[k];
        q[k] = hload(first_rec(t + k + kDepth));
        bool known;
        const uint4 e = lookup(h, r0 + lane < R1, known);
        const bool live = known && h.z != 0;
        header_handlers(h, known ? e.y : 0u, e.z, e.w, live, h.z & h.w);
      }
      if (done) break;
    }
  }
  // payload handler sets: work items are chunks; the launch's last nw chunks are split into
  // SASSI_SPLIT_PARTS parts (128 records each) so that the items still running at the end are
  // short. Items below
  // n_static go round-robin over the warps (SM-interleaved ids); the last SASSI_DYN_ROUNDS rounds
  // are claimed from a launch-wide counter (p.sched[0]; back to zero when the launch's last CTA
  // exits), so warps whose items were cheaper take more (c2: every warp had ~8 chunks of uneven
  // cost; measured 0.510 -> 0.480 ms). A warp claims its next item when one ends.
  uint32_t* const sched = p.sched;
  const uint32_t n_split = min(n_units, nw);
  constexpr uint32_t kParts = SASSI_SPLIT_PARTS, kPartRec = SASSI_CHUNK / kParts;
  static_assert(kPartRec % 32 == 0 && kPartRec * kParts == SASSI_CHUNK, "parts of whole batches");
  const uint32_t n_whole = n_units - n_split, n_items = n_whole + kParts * n_split;
  const uint32_t n_static = n_whole > SASSI_DYN_ROUNDS * nw ? n_whole - SASSI_DYN_ROUNDS * nw : 0u;
  // the claimed id reaches the warp through its shared-memory slot, read with a plain load: a loop
  // whose exit depends on an atomic's return value (or on a volatile load) looks like a spin loop
  // to ptxas, which then puts YIELDs into every loop nested in it (measured: c3 +1.3 %, c5 +2 %)
  uint32_t* const s_slot = sm + Ly::kSlot + wib;
  auto next_item = [&](uint32_t it) -> uint32_t {
    if (it < n_static) return it;
    if (lane == 0) *s_slot = atomicAdd(sched, 1u);
    __syncwarp();
    const uint32_t v = *s_slot;
    __syncwarp();
    return n_static + v;
  };
  for (uint32_t it = kUnitRows ? next_item(wib * gridDim.x + blockIdx.x) : n_items; it < n_items;
       it = next_item(it + nw)) {
    // item -> chunk u, whole or one of its kParts parts (records [part * kPartRec, + kPartRec));
    // a part is folded as a chunk of its own (its own record count and row bases), so the batch
    // loop below is the same for every item
    uint32_t u = it, part = 0;
    if (it >= n_whole) {
      u = n_whole + (it - n_whole) / kParts;
      part = (it - n_whole) % kParts;
    }
    const ulonglong2 cb0 = kUnitRows ? p.cb[u] : make_ulonglong2(p.arow_base, p.vrow_base);
    const ulonglong2 cb1 = kUnitRows ? p.cb[u + 1] : cb0;
    if (kUnitRows && !(cb0.x >= p.arow_base && cb0.x <= cb1.x && cb1.x <= p.arow_end &&
                       cb0.y >= p.vrow_base && cb0.y <= cb1.y && cb1.y <= p.vrow_end)) {
      err |= kErrIndex;  // chunk index outside the row buffers
      continue;
    }
    const uint4* hchunk = p.hdr + u * SASSI_CHUNK;
    uint32_t nrec = min(p.n - u * SASSI_CHUNK, (uint32_t)SASSI_CHUNK);
    uint32_t aend = (uint32_t)(cb1.x - cb0.x), vend = (uint32_t)(cb1.y - cb0.y);
    uint32_t a0 = 0, v0 = 0;  // rows before the item's first record (parts after the first)
    if (it >= n_whole) {
      const uint32_t r0 = part * kPartRec;
      if (nrec <= r0) continue;  // a short last chunk: its earlier parts cover it
      if (r0) {
        const uint2 r = part_offsets(hchunk, r0, lane, gm ? p.hash : s_hash, cap, p.hmul, p.hshr,
                                     p.arow_bit);
        if (r.x > aend || r.y > vend) {
          err |= kErrRows;  // the earlier parts' rows run past the chunk's rows
          continue;
        }
        a0 = r.x;
        v0 = r.y;
        aend -= a0;
        vend -= v0;
        hchunk += r0;
      }
      nrec = min(nrec - r0, kPartRec);  // bounded by the chunk's rows; the end checked by the last part
    }
    // rows are addressed relative to this item: 32-bit offsets from here on
    const uint64_t* const achunk = p.addr + ((cb0.x - p.arow_base + a0) << 5);
    const uint32_t* const vchunk = p.val + ((cb0.y - p.vrow_base + v0) << 5);
    uint32_t arow = 0, vrow = 0;
    const uint32_t nbat = (nrec + 31) >> 5;
    if (lane == 0) c_rec += nrec;
    // header loads are clamped to the item's last record (always in bounds) and masked by `valid`
    const uint32_t ilast = nrec - 1;
    uint4 hnext = ld_nc_v4(hchunk + min(lane, ilast));
    uint32_t b = 0;
    for (; b < nbat; ++b) {
      const uint32_t ib = 32 * b + lane;
      const bool valid = ib < nrec;
      const uint4 h = hnext;
      if (b + 1 < nbat) hnext = ld_nc_v4(hchunk + min(ib + 32, ilast));
      bool known;
      const uint4 e = lookup(h, valid, known);
      const uint32_t info = known ? e.y : 0u, cidx = e.z;
      // ---- row indices of this batch (rows follow their records); only handlers that read
      // payload rows need them, header-only handler sets skip the bookkeeping ----
      constexpr bool kRows = (H & (SASSI_H_MEMDIV | SASSI_H_VALUE)) != 0;
      const uint32_t ma = kRows ? __ballot_sync(FULL, info & p.arow_bit) : 0u;
      const uint32_t nd = (info >> I_NDST_SHIFT) & 7u;
      uint32_t vpre = 0, vtot = 0;
      if (kRows) {
#pragma unroll
        for (int k = 0; k < 3; ++k) {
          const uint32_t mk = __ballot_sync(FULL, (nd >> k) & 1u);
          vpre += __popc(mk & lt) << k;
          vtot += __popc(mk) << k;
        }
      }
      const uint32_t arow_b = arow, vrow_b = vrow;
      if (kRows) {
        arow += __popc(ma);
        vrow += vtot;
        if (arow > aend || vrow > vend) {
          err |= kErrRows;  // rows of this batch run past the chunk's rows: stream inconsistent
          break;
        }
#if SASSI_PREF_ROWS
        // the next batch's address rows (about a batch's worth: SASSI_PREF_ROWS) into L2 now, so
        // that its row loads wait on L2 instead of DRAM (measured: c3 2.476 -> 2.425 ms, c2 0.477 ->
        // 0.470; 8+ rows or deduplicated deeper windows are slower, value-row prefetch too). In the
        // default row layout the window also covers rows of non-GLOBAL sites that memdiv skips:
        // c3 DRAM reads 15.70 -> 16.26 GB (GLOBAL-only streams: none)
        if ((H & SASSI_H_MEMDIV) && lane == 0 && arow < aend)
          asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(achunk + 32 * arow),
                       "r"(256u * min(aend - arow, (uint32_t)SASSI_PREF_ROWS)) : "memory");
#endif
      }
      const uint32_t act = h.z;
      const bool live = known && act != 0;
      const uint32_t G = act & h.w;  // guard-true (or taken) active lanes
      // value rows of this batch are contiguous: start the first bulk copy now, so it lands while
      // the other handlers work on the batch
      const uint32_t* const vsrc = vchunk + 32 * vrow_b;
      if ((H & SASSI_H_VALUE) && vtot && lane == 0) bulk_load(vbuf, vsrc, 128u * min(vtot, 32u), vbar);

      header_handlers(h, info, cidx, e.w, live, G);
      // ---- Case study II: memory address divergence (Fig.6), one warp per address row ----
      if (H & SASSI_H_MEMDIV) {
        const bool selm_l = live && (info & I_MEMDIV) && G != 0;
        uint32_t selm = __ballot_sync(FULL, selm_l);
        if (selm) {
          const uint64_t* const abase = achunk + 32 * arow_b + lane;
          const uint32_t arel = __popc(ma & lt);
          uint32_t my_s = 0, my_l = 0;  // results of this lane's own record
          uint32_t slow = 0;            // rows whose sectors differ in the high word
          do {
            uint64_t a[SASSI_ROW_GROUP];
            uint32_t g[SASSI_ROW_GROUP], jj[SASSI_ROW_GROUP];
#pragma unroll
            for (int k = 0; k < SASSI_ROW_GROUP; ++k) {
              g[k] = 0;
              if (selm) {
                const int j = __ffs(selm) - 1;
                selm &= selm - 1;
                jj[k] = j;
                g[k] = __shfl_sync(FULL, G, j);
                a[k] = ld_nc_u64(abase + 32 * __shfl_sync(FULL, arel, j));
              }
            }
#pragma unroll
            for (int k = 0; k < SASSI_ROW_GROUP; ++k) {
              if (g[k]) {
                uint32_t s, L;
                if (memdiv_row32(a[k], g[k], lane, hbm, &s, &L)) {
                  if (lane == jj[k]) {
                    my_s = s;
                    my_l = L;
                  }
                } else {
                  slow |= 1u << jj[k];
                }
              }
            }
          } while (selm);
          while (slow) {
            const int j = __ffs(slow) - 1;
            slow &= slow - 1;
            uint32_t s, L;
            const uint64_t a = ld_nc_u64(abase + 32 * __shfl_sync(FULL, arel, j));
            const uint32_t g = __shfl_sync(FULL, G, j);
            memdiv_row64(a, g, lane, &s, &L);
            if (lane == j) {
              my_s = s;
              my_l = L;
            }
          }
          // one vectorised update for the batch: each record's lane adds its own results
          const uint32_t n = __popc(G);
          if (selm_l) {
            atomicAdd(sm + kSmH32 + 32 * (n - 1) + (my_s - 1), 1u);
            atomicAdd(sm + kSmH128 + 32 * (n - 1) + (my_l - 1), 1u);
            if (info & I_PCM)  // this pc's own matrix (sassi_select_memdiv_pcs)
              atomicAdd(s_pcm + 1024 * ((info >> I_PCM_SHIFT) & 3u) + 32 * (n - 1) + (my_s - 1), 1u);
          }
          if (gm) gcount4(selm_l, p.off.mem + 4ull * e.w, make_uint4(1u, n, my_s, my_l));
          else add_counters4(selm_l, PB + 4 * (cidx & 0xFFFFu), make_uint4(1u, n, my_s, my_l), wpriv);
        }
      }
      // ---- Case study III: value profiling (Fig.9): row-per-lane fold of TMA-staged rows ----
      if (H & SASSI_H_VALUE) {
        const bool selv = live && nd > 0 && G != 0;
        if (gm) {
          if (selv) {
            gadd(p.off.val + 2ull * e.w, 1ull);
            gadd(p.off.val + 2ull * e.w + 1, (unsigned long long)__popc(G));
          }
        } else {
          add_counters2(selv, PV + 2 * (cidx >> 16), make_uint2(1u, (uint32_t)__popc(G)), wpriv);
        }
        if (vtot) {
          const uint32_t vsel = selv ? G : 0u;                // lanes written by this lane's record
          // its first value-state slot (global mode: 4 * site, the image's [S][4] words)
          const uint32_t vslot = gm ? 4u * e.w : (info >> I_VD0_SHIFT) & 0xFFFFu;
          // the owner of every value row of the batch (lane ids in the warp's memdiv bitmap words,
          // which are all zero between memdiv rows): each lane records itself for its nd rows
          uint8_t* const owner = reinterpret_cast<uint8_t*>(hbm);
          if (Ly::kMem) {
#pragma unroll
            for (uint32_t d = 0; d < 4; ++d)
              if (d < nd) owner[vpre + d] = (uint8_t)lane;
            __syncwarp();
          }
          for (uint32_t s0 = 0; s0 < vtot; s0 += 32) {
            const uint32_t nr = min(vtot - s0, 32u);
            if (s0) {  // rows beyond the first 32: reuse the buffer once every lane is done with it
              __syncwarp();
              if (lane == 0) bulk_load(vbuf, vsrc + 32 * s0, 128u * nr, vbar);
            }
            mbar_wait(vbar, vphase);
            vphase ^= 1u;
            // owner of row r = s0 + lane: the largest lane j with vpre_j <= r (always one with a
            // value row, since a lane without rows shares vpre with its successor)
            const uint32_t r = s0 + lane;
            uint32_t j = 0;
            if (Ly::kMem) {
              j = owner[r & 127u];
            } else {
#pragma unroll
              for (uint32_t step = 16; step; step >>= 1)
                if (__shfl_sync(FULL, vpre, j + step) <= r) j += step;
            }
            const uint32_t Vj = __shfl_sync(FULL, vsel, j);
            const uint32_t slot = __shfl_sync(FULL, vslot, j) + (r - __shfl_sync(FULL, vpre, j));
            const uint32_t V = lane < nr ? Vj : 0u;
            // lane folds row s0+lane: 8 chunks of 4 values, chunk k ^ (lane & 7) at step k so the
            // 8 lanes of each shared-memory phase hit 8 different bank groups
            const uint4* row = vbuf + 8 * lane;
            uint32_t va = FULL, vo = 0;
            if (__all_sync(FULL, V == FULL || V == 0)) {
#pragma unroll
              for (uint32_t k = 0; k < 8; ++k) {
                const uint4 x = row[k ^ (lane & 7u)];
                va &= x.x & x.y & x.z & x.w;
                vo |= x.x | x.y | x.z | x.w;
              }
            } else {
              // lanes outside V hold garbage: stand in the row's value at a lane of V for them
              // (neutral for both AND and OR)
              const uint32_t ref = V ? reinterpret_cast<const uint32_t*>(row)[__ffs(V) - 1] : 0u;
#pragma unroll
              for (uint32_t k = 0; k < 8; ++k) {
                const uint32_t c = k ^ (lane & 7u);
                const uint4 x = row[c];
                const uint32_t vb = V >> (4 * c);
                const uint32_t x0 = (vb & 1u) ? x.x : ref, x1 = (vb & 2u) ? x.y : ref;
                const uint32_t x2 = (vb & 4u) ? x.z : ref, x3 = (vb & 8u) ? x.w : ref;
                va &= x0 & x1 & x2 & x3;
                vo |= x0 | x1 | x2 | x3;
              }
            }
            if (V != 0 && !gm) {
              uint4* st = s_vstate + slot;
              const uint4 c = *st;
              const uint32_t sc = va == vo ? 1u : 0u;                  // __all(v == leader) (L559)
              if ((c.x & va) != c.x) atomicAnd(&st->x, va);           // constantOnes   (L557)
              if ((c.y & ~vo) != c.y) atomicAnd(&st->y, ~vo);         // constantZeros  (L557)
              if ((c.z & sc) != c.z) atomicAnd(&st->z, sc);           // isScalar       (L561)
            } else if (V != 0) {  // global mode: the image's words (a stale read only adds an AND)
              const uint32_t cx = (uint32_t)__ldcg(table + p.off.ones + slot);
              const uint32_t cy = (uint32_t)__ldcg(table + p.off.zeros + slot);
              const uint32_t cz = (uint32_t)__ldcg(table + p.off.scalar + slot);
              if ((cx & va) != cx) gand(p.off.ones + slot, (unsigned long long)va);
              if ((cy & ~vo) != cy) gand(p.off.zeros + slot, (unsigned long long)(uint32_t)~vo);
              if (cz && va != vo) gand(p.off.scalar + slot, 0ull);
            }
          }
          __syncwarp();
          if (Ly::kMem) {  // the bitmap words back to zero for the next batch's memdiv rows
            hbm[lane] = 0u;
            __syncwarp();
          }
        }
      }
    }
    // a part ending before its chunk's last record has no end of its own to check
    const bool inner_part = it >= n_whole && ((it - n_whole) % kParts + 1) * kPartRec <
                                                 min(p.n - (n_whole + (it - n_whole) / kParts) * SASSI_CHUNK,
                                                     (uint32_t)SASSI_CHUNK);
    if ((H & (SASSI_H_MEMDIV | SASSI_H_VALUE)) && b == nbat && !inner_part && lane == 0 &&
        (arow != aend || vrow != vend))
      err |= kErrRows;  // index disagrees with the rows
  }
  SASSI_STAMP(2, gtime())
  if (H & SASSI_H_INSTCOUNT) {
    if (kVertical) flush_planes();
    if (acc_w != FULL && acc) gadd(p.off.counts + 32ull * acc_w + lane, (unsigned long long)acc);
  }
  // ---- diagnostics: warp-reduce, one smem atomic per warp ----
  uint32_t* const s_diag = sm + kSmDiag;
  c_rec = __reduce_add_sync(FULL, c_rec);
  c_inv = __reduce_add_sync(FULL, c_inv);
  c_unk = __reduce_add_sync(FULL, c_unk);
  c_bad = __reduce_add_sync(FULL, c_bad);
  err = __reduce_or_sync(FULL, err);
  if (lane == 0) {
    atomicAdd(s_diag + 0, c_rec);
    atomicAdd(s_diag + 1, c_inv);
    atomicAdd(s_diag + 2, c_unk);
    atomicAdd(s_diag + 3, c_bad);
    if (err) atomicOr(p.err, err);
  }
  __syncthreads();
  // every warp of the CTA is past its last claim: the launch's last CTA resets the scheduler
  if (kUnitRows && tid == 0) {
    // (every claim of this CTA has returned its value: no fence needed before the count)
    if (atomicAdd(sched + 1, 1u) == gridDim.x - 1) {
      sched[0] = 0;
      sched[1] = 0;
    }
  }

  // ---- flush: sum the warps' private counters, fold into the global u64 image ----
  if (tid < 4 && s_diag[tid]) gadd(tid, (unsigned long long)s_diag[tid]);
  if (kExt && p.dyn_cap)
    for (uint32_t i = tid; i < kDynLocal; i += blockDim.x)
      if (s_dkey[i] != EMPTY_KEY && s_dcnt[i])
        dyn_insert(s_dkey[i], s_dcnt[i], s_dthr[i], p.dyn_keys, p.dyn_vals, p.dyn_cap, p.dyn_lg);
  auto sum_words = [&](uint32_t off) -> uint4 {
    uint4 t = make_uint4(0, 0, 0, 0);
    for (uint32_t w = 0; w < n_regions; ++w) {
      const uint32_t* q = s_priv + w * p.pw + off;
      t.x += q[0];
      t.y += q[1];
      t.z += q[2];
      t.w += q[3];
    }
    return t;
  };
  if ((H & SASSI_H_BRANCH) && !gm) {
    for (uint32_t bi = tid; bi < p.nb; bi += blockDim.x) {
      const uint4 t = sum_words(4 * bi);
      if (t.x == 0) continue;
      const uint64_t g = p.off.br + 5ull * p.flush_b[bi];
      gadd(g + 0, (unsigned long long)t.x);
      gadd(g + 1, (unsigned long long)t.y);
      if (t.z) gadd(g + 2, (unsigned long long)t.z);
      if (t.y - t.z) gadd(g + 3, (unsigned long long)(t.y - t.z));  // not taken = active - taken
      if (t.w) gadd(g + 4, (unsigned long long)t.w);
    }
  }
  if (H & SASSI_H_MEMDIV) {
    for (uint32_t m = tid; !gm && m < p.nm; m += blockDim.x) {
      const uint4 t = sum_words(PB + 4 * m);
      if (t.x == 0) continue;
      const uint64_t g = p.off.mem + 4ull * p.flush_m[m];
      gadd(g + 0, (unsigned long long)t.x);
      gadd(g + 1, (unsigned long long)t.y);
      gadd(g + 2, (unsigned long long)t.z);
      gadd(g + 3, (unsigned long long)t.w);
    }
    for (uint32_t c = tid; c < 2048; c += blockDim.x) {
      const uint32_t v = sm[kSmH32 + c];
      if (v) gadd(c < 1024 ? p.off.h32 + c : p.off.h128 + (c - 1024), (unsigned long long)v);
    }
    for (uint32_t c = tid; c < 1024 * p.npcm; c += blockDim.x)
      if (s_pcm[c]) gadd(p.off.pcmat + c, (unsigned long long)s_pcm[c]);
  }
  if (H & SASSI_H_INSTMIX) {
    unsigned long long* const s_imix = reinterpret_cast<unsigned long long*>(sm + kSmImix);
    if (gm && lane == 0)  // global mode: the warps' Fig.3 totals
      for (uint32_t k = 0; k < 7; ++k)
        if (g_imix[k]) atomicAdd(s_imix + k, g_imix[k]);
    for (uint32_t st = tid; !gm && st < p.S; st += blockDim.x) {
      uint32_t t = 0;
      for (uint32_t w = 0; w < n_regions; ++w) t += s_priv[w * p.pw + p.px + st];
      if (t == 0) continue;
      gadd(p.off.mix + st, (unsigned long long)t);
      const uint32_t cat = p.flush_x[st];
      for (uint32_t k = 0; k < 7; ++k)
        if ((cat >> k) & 1u) atomicAdd(s_imix + k, (unsigned long long)t);
    }
    __syncthreads();
    if (tid < 7 && s_imix[tid]) gadd(p.off.imix + tid, s_imix[tid]);
  }
  if ((H & SASSI_H_VALUE) && !gm) {
    for (uint32_t k = tid; k < p.nv; k += blockDim.x) {
      const uint32_t site = p.flush_v[3 * k], vd0 = p.flush_v[3 * k + 1], nd = p.flush_v[3 * k + 2];
      uint32_t we = 0, te = 0;
      for (uint32_t w = 0; w < n_regions; ++w) {
        we += s_priv[w * p.pw + PV + 2 * k];
        te += s_priv[w * p.pw + PV + 2 * k + 1];
      }
      if (we == 0) continue;
      gadd(p.off.val + 2ull * site, (unsigned long long)we);
      gadd(p.off.val + 2ull * site + 1, (unsigned long long)te);
      for (uint32_t d = 0; d < nd; ++d) {
        const uint4 st = s_vstate[vd0 + d];
        if (st.x != FULL) gand(p.off.ones + 4ull * site + d, (unsigned long long)st.x);
        if (st.y != FULL) gand(p.off.zeros + 4ull * site + d, (unsigned long long)st.y);
        if (st.z != 1u) gand(p.off.scalar + 4ull * site + d, 0ull);
      }
    }
  }
  SASSI_STAMP(3, gtime())
}

__global__ void dyn_reset_kernel(uint32_t* keys, unsigned long long* vals, uint32_t cap) {
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i <= 2 * cap; i += gridDim.x * blockDim.x) {
    if (i < cap) keys[i] = EMPTY_KEY;
    vals[i] = 0;
  }
}

using KernelFn = void (*)(const ConsumeParams);

template <uint32_t H, bool kExt>
KernelFn kernel_for() {
  return consume_kernel<H, kExt>;
}

template <uint32_t... Hs>
KernelFn pick(uint32_t mask, bool dyn, std::integer_sequence<uint32_t, Hs...>) {
  KernelFn fn = nullptr;
  ((mask == Hs + 1 ? (fn = dyn ? kernel_for<Hs + 1, true>() : kernel_for<Hs + 1, false>(), 0) : 0), ...);
  return fn;
}

// one instantiation per non-empty handler set (1..31), plain and extended (dynamic pcs / peers)
#ifndef SASSI_ONLY_H
KernelFn select_kernel(uint32_t mask, bool dyn) {
  if (mask == 0 || mask > SASSI_H_EVERY) return nullptr;
  return pick(mask, dyn, std::make_integer_sequence<uint32_t, SASSI_H_EVERY>{});
}
#else  // development builds (SASS inspection): one handler set only
KernelFn select_kernel(uint32_t mask, bool dyn) {
  if (mask != SASSI_ONLY_H) return nullptr;
  return dyn ? kernel_for<SASSI_ONLY_H, true>() : kernel_for<SASSI_ONLY_H, false>();
}
#endif

}  // namespace

int launch_dyn_reset(sassi_ctx* c, cudaStream_t s) {
  if (!c->dyn_cap) return SASSI_OK;
  dyn_reset_kernel<<<(2 * c->dyn_cap + 256) / 256, 256, 0, s>>>(c->d_dyn_keys, c->d_dyn_vals, c->dyn_cap);
  SASSI_CUDA(cudaGetLastError());
  c->launches += 1;
  return SASSI_OK;
}

int consume_smem_bytes(const sassi_ctx* c, size_t* bytes) {
  const uint32_t H = c->mask;
  size_t words = sm_var_words(H);
  if (!c->gmode) {  // global mode keeps the hash, the value state and the counters in global memory
    words += 4ull * c->cap;
    if (H & SASSI_H_VALUE) words += 4ull * c->nvd;
    if (H & (SASSI_H_BRANCH | SASSI_H_MEMDIV | SASSI_H_VALUE | SASSI_H_INSTMIX))
      words += (c->priv ? kWarpsPerCta : 1) * (size_t)c->pw;
  }
  if (H & SASSI_H_MEMDIV) words += 1024ull * c->npcm;  // per-PC matrices
  if (c->dyn_cap) words += kDynLocalWords;              // the CTA's dynamic-pc cache
  *bytes = 4 * words;
  return 0;
}

int launch_consume(sassi_ctx* c, const ConsumeParams& p, cudaStream_t s) {
  KernelFn fn = select_kernel(c->mask, p.dyn_cap != 0 || p.n_peers != 0 || p.gmode != 0);
  if (!fn) return set_error(SASSI_ESTATE, "no handler attached");
  if ((void*)fn != c->launch_fn || c->smem_bytes != c->launch_smem) {  // configure once per kernel
    {
      // the attribute is per function and per device (CUDA context): only ever raise it, keyed on
      // (device, function) since contexts on one device share kernels
      static std::mutex mu;
      static std::map<std::pair<int, void*>, size_t> attr;
      std::lock_guard<std::mutex> lock(mu);
      size_t& cur = attr[{c->device, (void*)fn}];
      if (c->smem_bytes > cur) {
        SASSI_CUDA(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)c->smem_bytes));
        cur = c->smem_bytes;
      }
    }
    int per_sm = 0;
    SASSI_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, kConsumeThreads, c->smem_bytes));
    if (per_sm < 1) return set_error(SASSI_ENOSPC, "consume kernel does not fit on an SM");
    c->ctas_per_sm = per_sm;
    c->launch_fn = (void*)fn;
    c->launch_smem = c->smem_bytes;
  }
  const int per_sm = c->ctas_per_sm;
  const uint64_t units = ((uint64_t)p.n + SASSI_CHUNK - 1) / SASSI_CHUNK;
  uint64_t grid = (uint64_t)c->num_sms * per_sm;
  const uint64_t need = (units + kWarpsPerCta - 1) / kWarpsPerCta;
  if (grid > need) grid = need ? need : 1;
  ConsumeParams q = p;
  q.sched = c->d_err + 4 + 2 * (c->sched_seq++ % kSchedSlots);
  fn<<<(unsigned)grid, kConsumeThreads, c->smem_bytes, s>>>(q);
  SASSI_CUDA(cudaGetLastError());
  c->launches += 1;
  return SASSI_OK;
}

}  // namespace sassi
