/*
 * sassi.h — C ABI of the B200-native SASSI instrumentation-handler analysis path.
 *
 * What this library computes (PAPER.md = /root/reference/PAPER.md, "Lnnn" = its line):
 *   Stephenson et al., "Flexible Software Profiling of GPU Architectures" (SASSI), ISCA'15.
 *   SASSI calls a user handler at every instrumented SASS instruction (L181-L187, §3.1-3.2).
 *   The paper's four case-study handlers are folded here over warp-wide instruction records:
 *     - SASSI_H_BRANCH    conditional-branch divergence   (§5, Fig.4)
 *     - SASSI_H_MEMDIV    memory address divergence       (§6, Fig.6)
 *                         in 32 B sectors (the paper's "line", L367) and 128 B lines
 *     - SASSI_H_VALUE     value profiling: constant bits + scalar writes (§7, Fig.9)
 *     - SASSI_H_INSTCOUNT per-thread dynamic-instruction counts for error-injection
 *                         site selection (§8.1)
 *   plus the paper's introductory example handler:
 *     - SASSI_H_INSTMIX   instruction mix: thread-level counts of memory / extended memory /
 *                         control-transfer / sync / numeric / texture / all instructions
 *                         (Fig.3)
 *   The handler semantics (which lanes count, init values, counter widths) are spelled out in
 *   DESIGN.md §3 ("Readings"); every table entry is an integer fold, so results are exact.
 *
 * ---------------------------------------------------------------------------------------------
 * RECORD FORMAT "SRF1" (all little-endian, all buffers DEVICE memory unless stated otherwise)
 * ---------------------------------------------------------------------------------------------
 *  The static "where/what" of SASSI (L181-L187) is a site table registered once per context:
 *    sassi_site { pc, flags, mem_width, domain, n_gpr_dst, reg_num[4] }          (16 B)
 *  mirroring the static parts of SASSIBeforeParams.insEncoding / SASSIMemoryParams.properties,
 *  width, domain (Fig.2b/c, L157-L173) and SASSIRegisterParams.GetNumGPRDsts/GetRegNum (L555).
 *
 *  The dynamic part is one 16 B header per dynamic warp-instruction ("record"):
 *    sassi_hdr { pc, warp, active, mask2 }
 *      pc     instruction address (SASSIBeforeParams.GetInsAddr, L159)
 *      warp   global warp id; thread id = 32*warp + lane (L629 "thread ID")
 *      active lanes executing the instruction (__ballot(1), L239 l.13)
 *      mask2  COND_BRANCH sites: lanes whose direction is "taken" (GetDirection, L237 l.8)
 *             all other sites: guard-predicate-true lanes (instrWillExecute, L173, L363 l.4)
 *  plus payload rows, each a full warp wide, in record order:
 *    addr row  uint64_t[32]  one per record at a site with SASSI_F_MEM (any domain):
 *              lane l's effective address (SASSIMemoryParams.GetAddress, L165)
 *    val rows  uint32_t[32]  n_gpr_dst rows per record at a site with n_gpr_dst > 0:
 *              lane l's value written to destination d (GetRegValue, L555)
 *  Rows exist for every record whose pc is registered, whatever its masks (even active == 0).
 *  Records whose pc is NOT registered carry no rows. Lanes outside the relevant mask may hold
 *  any value. Row content outside the masks is never read by the fold.
 *
 *  chunk_base[ceil(n/SASSI_CHUNK)+1]: for chunk c, the index of the first addr row and first
 *  val row belonging to a record with index >= c*SASSI_CHUNK; entry [n_chunks] holds the
 *  totals. It is an index over the row streams so independent workers can start mid-stream;
 *  sassi_index_records() builds it on the device from the headers when the producer did not.
 *
 * ---------------------------------------------------------------------------------------------
 * TABLE IMAGE (what sassi_read_tables returns): one flat uint64_t array, offsets from
 * sassi_table_layout(n_sites, n_warps). S = n_sites in REGISTRATION order, W = n_warps.
 * ---------------------------------------------------------------------------------------------
 *   diag[8]        n_records, n_invalid (active==0), n_unknown_pc, n_bad_warp (instcount record
 *                  with warp >= W), n_sites, n_warps, handler_mask, SASSI_ABI_VERSION
 *   br[S][5]       totalBranches, activeThreads, takenThreads, takenNotThreads,
 *                  divergentBranches                              (BranchStats, Fig.4 l.27-33)
 *   mem[S][4]      warp accesses, active lanes, distinct 32 B sectors, distinct 128 B lines
 *   val[S][2]      warp executions, thread executions ("weight", Fig.9)
 *   ones[S][4]     constantOnes[d]  (low 32 bits used; init 0xFFFFFFFF)   (Fig.9)
 *   zeros[S][4]    constantZeros[d] (low 32 bits used; init 0xFFFFFFFF)   (Fig.9)
 *   scalar[S][4]   isScalar[d]: 1 iff in every warp execution all written lanes wrote one
 *                  value to dst d (AND of allSame; init 1)            (Fig.9)
 *   h32[32][32]    sassi_counters[numActive-1][unique-1], unique = distinct 32 B sectors (Fig.6 l.33)
 *   h128[32][32]   the same matrix with 128 B lines
 *   counts[32*W]   per-thread eligible dynamic-instruction counts (§8.1 (4), L627)
 *   mix[S]         thread executions per site: sum of popc(active) (Fig.3's count, per site)
 *   imix[8]        Fig.3's dynamic_instr_counts[7] = {memory, extended memory (width > 4 B),
 *                  controlxfer, sync, numeric, texture, total executed}, then one zero word
 *   pcsel[4]       sites whose per-PC memdiv matrix is kept: site index + 1 (0 = slot unused);
 *                  configuration (sassi_select_memdiv_pcs), not a counter
 *   pcmat[4][32][32]  per selected pc, the h32 matrix of its own records (L353 "detailed
 *                  accounting of unique references generated per program counter")
 *
 * ---------------------------------------------------------------------------------------------
 * CONVENTIONS
 *   - Every function returns a sassi_status (0 = OK, < 0 = error); no exception crosses the ABI.
 *   - Asynchronous CUDA faults surface as SASSI_ECUDA at the next call that synchronises.
 *   - A context is bound to one device and is NOT thread-safe.
 *   - The context owns its device tables and site hash; the caller owns record buffers and
 *     streams. Record buffers must stay valid until the stream work of the call completes.
 *   - `stream` arguments are cudaStream_t passed as void* (NULL = legacy default stream).
 *   - There is no CPU fallback: without a usable CUDA device every call fails (SASSI_ECUDA).
 */
#ifndef SASSI_H_
#define SASSI_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* Opaque context (one per device; owns the device tables and the site hash). Declared here so
 * the prototypes below all name the same type in C as well as in C++. */
struct sassi_ctx;
typedef struct sassi_ctx sassi_ctx;

#define SASSI_ABI_VERSION 3u
#define SASSI_WARP_SIZE 32u
#define SASSI_CHUNK 256u           /* records per chunk_base entry */
#define SASSI_MAX_SITES 65536u     /* registered sites per context (beyond ~4k: global mode, see attach) */
#define SASSI_MAX_DST 4u           /* GPR destinations per instruction (e.g. 128-bit loads) */
#define SASSI_MAX_PC_MATRICES 4u   /* per-PC memdiv matrices (sassi_select_memdiv_pcs)          */

typedef enum sassi_status {
  SASSI_OK = 0,
  SASSI_EINVAL = -1,     /* bad argument (null pointer, bad flags, duplicate pc, ...)        */
  SASSI_ECUDA = -2,      /* CUDA runtime error (message via sassi_strerror / last error)     */
  SASSI_ENCCL = -3,      /* NCCL error or NCCL library not loadable                          */
  SASSI_ENOSPC = -4,     /* too many sites / handler state does not fit shared memory         */
  SASSI_ESTATE = -5,     /* call not valid in the context's current state                    */
  SASSI_EMISMATCH = -6,  /* site tables differ across ranks in sassi_merge                   */
  SASSI_EFORMAT = -7     /* record stream inconsistent with its row counts / chunk index     */
} sassi_status;

/* Handler kinds for sassi_attach_handler (bit mask). */
enum {
  SASSI_H_BRANCH = 1u,
  SASSI_H_MEMDIV = 2u,
  SASSI_H_VALUE = 4u,
  SASSI_H_INSTCOUNT = 8u,
  SASSI_H_ALL = 15u,       /* the paper's four case-study handlers (§5-§8)                      */
  SASSI_H_INSTMIX = 16u,   /* Fig.3 instruction mix (L193-L199)                                 */
  SASSI_H_EVERY = 31u      /* every handler kind                                                */
};

/* sassi_site.flags — static instruction properties (insEncoding / properties). */
enum {
  SASSI_F_COND_BRANCH = 1u << 0, /* IsCondControlXfer (L159): mask2 = taken lanes              */
  SASSI_F_CTRL = 1u << 1,        /* IsControlXfer                                            */
  SASSI_F_MEM = 1u << 2,         /* IsMem: record carries an addr row                        */
  SASSI_F_MEM_READ = 1u << 3,    /* IsMemRead / IsLoad                                       */
  SASSI_F_MEM_WRITE = 1u << 4,   /* IsMemWrite / IsStore                                     */
  SASSI_F_ATOMIC = 1u << 5,      /* IsAtomic                                                 */
  SASSI_F_SYNC = 1u << 6,        /* IsSync                                                   */
  SASSI_F_NUMERIC = 1u << 7,     /* IsNumeric                                                */
  SASSI_F_TEXTURE = 1u << 8,     /* IsTexture                                                */
  SASSI_F_WRITES_PRED = 1u << 9, /* writes a predicate register (error model, L621)          */
  SASSI_F_WRITES_CC = 1u << 10,  /* writes the condition code (error model, L621)            */
  SASSI_F_ALL = (1u << 11) - 1u
};

/* sassi_site.domain — SASSIMemoryParams.GetDomain (L167); memdiv counts GLOBAL only (L363 l.7). */
enum { SASSI_D_GLOBAL = 0, SASSI_D_SHARED = 1, SASSI_D_LOCAL = 2, SASSI_D_CONST = 3, SASSI_D_TEX = 4 };

typedef struct sassi_site {
  uint32_t pc;         /* instruction address; must be unique; 0xFFFFFFFF is reserved          */
  uint16_t flags;      /* SASSI_F_*; COND_BRANCH excludes MEM and n_gpr_dst > 0                 */
  uint8_t mem_width;   /* bytes per lane access (GetWidth, L167); informational                 */
  uint8_t domain;      /* SASSI_D_* (meaningful with SASSI_F_MEM)                               */
  uint8_t n_gpr_dst;   /* 0..SASSI_MAX_DST GPR destinations (GetNumGPRDsts, L555)               */
  uint8_t reg_num[4];  /* destination register numbers (GetRegNum, L555), for reports          */
  uint8_t reserved[3];
} sassi_site;          /* 16 B */

typedef struct sassi_hdr {
  uint32_t pc, warp, active, mask2;
} sassi_hdr;           /* 16 B */

typedef struct sassi_chunk_base {
  uint64_t addr_row, val_row;
} sassi_chunk_base;    /* 16 B */

typedef struct sassi_records {
  const sassi_hdr* hdr;                /* [n]                                                */
  const uint64_t* addr;                /* [n_addr_rows][32] (may be NULL if n_addr_rows == 0) */
  const uint32_t* val;                 /* [n_val_rows][32]  (may be NULL if n_val_rows == 0)  */
  const sassi_chunk_base* chunk_base;  /* [ceil(n/SASSI_CHUNK)+1]                             */
  uint64_t n_addr_rows, n_val_rows;
} sassi_records;

/* One error-injection site tuple (L629): kernel, dynamic invocation, thread, dynamic instruction
 * index of that thread, seed to choose the destination register, seed to choose the bit. */
typedef struct sassi_inj_site {
  uint32_t kernel, invocation, thread, reg_seed, bit_seed, reserved;
  uint64_t dyn_index;
} sassi_inj_site;      /* 32 B */

typedef struct sassi_layout {
  uint64_t diag, br, mem, val, ones, zeros, scalar, h32, h128, counts, mix, imix, pcsel, pcmat,
      total; /* u64 words */
} sassi_layout;

/* Offsets of the table image (host-only arithmetic; no device needed). */
int sassi_table_layout(uint32_t n_sites, uint32_t n_warps, sassi_layout* out);

/* Create a context on `device` for a program with the given static sites (HOST array, copied)
 * and n_warps trace warps (per-thread counts cover 32*n_warps threads). The site hash (open
 * addressing keyed by pc, L239 l.21-23 "find") is built here and uploaded.
 * Errors: EINVAL (null/invalid site, duplicate pc), ENOSPC (n_sites > SASSI_MAX_SITES), ECUDA. */
int sassi_ctx_create(struct sassi_ctx** out, int device, const sassi_site* sites, uint32_t n_sites,
                     uint32_t n_warps);
void sassi_ctx_destroy(struct sassi_ctx* ctx);

/* Select which handlers run (non-empty subset of SASSI_H_EVERY) — the paper's "what"
 * (L181-L187). Allowed only before the first consume or right after sassi_reset, and not to a
 * different set while peer tables are attached. The fold keeps the pc hash, the value state and
 * the per-site counters in each SM's shared memory when they fit; a larger site table (thousands
 * of sites, up to SASSI_MAX_SITES) runs in "global mode": hash lookups from global memory and
 * per-record u64 atomics into the table image (the paper's own device-global tables),
 * same results, lower throughput (the environment variable SASSI_FORCE_GLOBAL_MODE=1, read here,
 * forces global mode for tests). Errors: EINVAL, ESTATE, ENOSPC (the 32x32 matrices and the
 * per-PC matrices alone exceed shared memory: not reachable with SASSI_MAX_PC_MATRICES). */
int sassi_attach_handler(struct sassi_ctx* ctx, uint32_t kind_mask);

/* Keep a per-PC memory-divergence matrix (pcmat, the Fig.6 32x32 matrix of that pc's own records)
 * for k <= SASSI_MAX_PC_MATRICES registered GLOBAL memory sites given by pc (HOST array; k = 0
 * clears the selection). Like sassi_attach_handler: only before the first consume or right after
 * sassi_reset, not while peer tables are attached; the selection is part of the site-table
 * checksum sassi_merge compares (and of the layout sassi_add_peer_table checks). Takes
 * effect with SASSI_H_MEMDIV attached; costs 4 KB of shared memory per selected pc per CTA.
 * Errors: EINVAL (unknown pc, not a GLOBAL memory site, k too large), ESTATE, ENOSPC. */
int sassi_select_memdiv_pcs(struct sassi_ctx* ctx, const uint32_t* pcs, uint32_t k);

/* Address-row layout of the record streams this context consumes. SASSI_ADDR_ROWS_ALL (default,
 * SRF1 as above): an addr row for every record at a SASSI_F_MEM site, any domain.
 * SASSI_ADDR_ROWS_GLOBAL: the producer writes the rows of GLOBAL memory sites to the addr stream
 * and the others (shared, local, ... memory, which no handler reads: memdiv counts GLOBAL only,
 * L363 l.7) to a stream of their own that is not passed here; chunk_base's addr_row counts the
 * GLOBAL rows only (sassi_index_records follows this setting). sassi_consume_host then copies only
 * those rows over PCIe. Only before the first consume or right after sassi_reset.
 * Errors: EINVAL, ESTATE. */
enum { SASSI_ADDR_ROWS_ALL = 0u, SASSI_ADDR_ROWS_GLOBAL = 1u };
int sassi_set_addr_rows(struct sassi_ctx* ctx, uint32_t which);

/* Top-K per-PC matrices: from the tables of the folds so far, rank the
 * GLOBAL memory sites by distinct 32 B sectors per warp access (mem[s][2] / mem[s][0], compared
 * exactly; ties: more warp accesses first, then the lower site index; sites never accessed are not
 * ranked), then sassi_reset the context and keep the per-PC matrices of the first min(k, ranked)
 * sites (sassi_select_memdiv_pcs) for the next pass over the same records. pcs_out (HOST, k
 * entries) receives their pcs in rank order, *n_out their number. Synchronises `stream`.
 * Errors: EINVAL (k > SASSI_MAX_PC_MATRICES, null pointer), ESTATE (peer tables attached). */
int sassi_select_memdiv_topk(struct sassi_ctx* ctx, uint32_t k, uint32_t* pcs_out, uint32_t* n_out,
                             void* stream);

/* Dynamic sites: Fig.4 l.21-23 (L239) "Find the instruction's counters in a
 * hash table based on its address. Create a new entry if one does not exist." With this enabled,
 * every record whose pc is NOT registered (still counted in diag n_unknown_pc; it carries no rows)
 * also updates an insert-on-miss device hash table keyed by pc: the entry is created on first
 * sight (CAS, linear probing) and counts warp executions (records) and thread executions
 * (popc(active); inactive records add a warp execution and no thread). capacity = the number of
 * distinct unregistered pcs the table must hold (slots: a power of two >= 2 * capacity, >= 32;
 * capacity 0 disables it). Records that find the table full, or carry the reserved pc
 * 0xFFFFFFFF, are counted as dropped; results are exact (order-independent) while no record is
 * dropped. Like sassi_attach_handler: only before the first consume or right after sassi_reset;
 * sassi_reset clears the table; sassi_merge merges it (capacity is part of the checksum ranks
 * compare). Errors: EINVAL (capacity > 2^24), ESTATE, ECUDA. DESIGN.md reading R25. */
int sassi_enable_dynamic_pcs(struct sassi_ctx* ctx, uint32_t capacity);

typedef struct sassi_dyn_pc {
  uint32_t pc, reserved;
  uint64_t warp_execs, thread_execs;
} sassi_dyn_pc;        /* 24 B */

/* Read the dynamic table sorted by pc (canonical: slots depend on insertion order) into HOST
 * host_out[cap_out]; *n_out = the number of entries (only min(n, cap_out) are written; host_out may
 * be NULL when cap_out is 0); *n_dropped (may be NULL) = dropped records. Synchronises `stream`.
 * Errors: EINVAL, ESTATE (not enabled), ECUDA. */
int sassi_read_dynamic_pcs(struct sassi_ctx* ctx, sassi_dyn_pc* host_out, uint32_t cap_out,
                           uint32_t* n_out, uint64_t* n_dropped, void* stream);

/* Fold n records (DEVICE buffers) into the context's tables (and, with peer tables attached,
 * into theirs); asynchronous, stream-ordered. Tables accumulate across calls until sassi_reset.
 * Folds of one context may also run on unordered streams (the table updates are atomic; each
 * launch has its own chunk-scheduler words, up to 64 launches in flight). One kernel launch per
 * 2^29 records (the
 * environment variable SASSI_MAX_LAUNCH_RECORDS, read at sassi_ctx_create, lowers that to a
 * multiple of SASSI_CHUNK for tests). hdr, addr, val and chunk_base must be 16-byte aligned
 * (vector loads, TMA bulk copies and bulk L2 prefetches read them). Errors: EINVAL (incl.
 * misaligned buffers), ESTATE (no handler), ECUDA. */
int sassi_consume(struct sassi_ctx* ctx, const sassi_records* recs, uint64_t n, void* stream);

/* Same fold from HOST buffers (pinned or pageable): the library copies slices to the device
 * (double-buffered on `stream` plus an internal copy stream), consumes them, and returns after
 * the stream work completes. recs->chunk_base is required (host). Only what the attached handlers
 * read crosses PCIe: address rows with SASSI_H_MEMDIV, value rows with SASSI_H_VALUE, the chunk
 * index with either; header-only handler sets copy the headers alone. */
int sassi_consume_host(struct sassi_ctx* ctx, const sassi_records* host_recs, uint64_t n,
                       void* stream);

/* Build chunk_base (DEVICE, ceil(n/SASSI_CHUNK)+1 entries) from device headers using the
 * context's site table (row counts per record follow from the site of its pc). */
int sassi_index_records(struct sassi_ctx* ctx, const sassi_hdr* hdr, uint64_t n,
                        sassi_chunk_base* chunk_base_out, void* stream);

/* Re-initialise all tables, and the dynamic-pc table when enabled (CUPTI kernel-launch callback
 * analogue, L217). Asynchronous. With peer tables attached it resets this context's image only:
 * every rank resets its own, then a barrier, before any rank folds (see sassi_add_peer_table). */
int sassi_reset(struct sassi_ctx* ctx, void* stream);

/* Copy the table image (sassi_table_layout(...).total words) to HOST memory; synchronises
 * `stream` (CUPTI kernel-exit callback analogue, L217). Errors: EINVAL (n_words too small),
 * EFORMAT (a consume since the last sassi_reset found the record stream inconsistent with its rows
 * or chunk index: the tables are then incomplete), EMISMATCH (a sassi_merge found other site
 * tables on another rank and left the tables unmerged). */
int sassi_read_tables(struct sassi_ctx* ctx, uint64_t* host_out, uint64_t n_words, void* stream);

/* Device pointer to the live table image (owned by the context; read-only for the caller). */
int sassi_tables_device(struct sassi_ctx* ctx, const uint64_t** dev_ptr, uint64_t* n_words);

/* Exclusive scan of the per-thread counts and k draws of injection sites (L629), uniform over
 * all eligible dynamic thread-instructions, with replacement, draw j from splitmix64(seed + j).
 * out is a HOST array of k tuples; synchronises `stream` once (scan, draws and the copy back are
 * stream-ordered with no host round trip in between). Errors: ESTATE if the total is 0 (out is
 * then unspecified). */
int sassi_sample_sites(struct sassi_ctx* ctx, uint32_t k, uint64_t seed, sassi_inj_site* host_out,
                       void* stream);

/* The same scan and draws with DEVICE outputs and no host synchronisation (stream-ordered, so
 * back-to-back profiling passes keep the GPU busy): dev_out[k] receives the tuples, *dev_status
 * (device u32) is set to 0, or to 1 when the total is 0 (nothing to sample; dev_out untouched).
 * Buffers are the caller's and must stay valid until the stream work completes.
 * Errors: EINVAL (null pointer), ESTATE (n_warps = 0). */
int sassi_sample_sites_device(struct sassi_ctx* ctx, uint32_t k, uint64_t seed,
                              sassi_inj_site* dev_out, uint32_t* dev_status, void* stream);

/* An injection campaign over several kernel invocations (L629 "the static kernel name, dynamic
 * kernel invocation ID, thread ID, dynamic instruction count"): one profile per invocation, each a
 * context whose per-thread counts (SASSI_H_INSTCOUNT) were folded from that invocation, with the
 * kernel and invocation ids its tuples carry. k draws uniform over all eligible dynamic
 * thread-instructions of all profiles, with replacement (reading R29): draw j takes
 * kk = floor(splitmix64(seed + j) * total / 2^64) over the profiles' totals in the given order, the
 * profile holding kk, then thread and dynamic index within it as sassi_sample_sites (one profile
 * with ids 0, 0 gives exactly sassi_sample_sites' tuples). All contexts on one device; HOST
 * profiles[n] and out[k]; synchronises `stream` once. Errors: EINVAL (null, duplicate context,
 * several devices), ESTATE (a profile without warps, or nothing to sample). */
typedef struct sassi_profile {
  struct sassi_ctx* ctx;
  uint32_t kernel, invocation;
} sassi_profile;
int sassi_sample_sites_multi(const sassi_profile* profiles, uint32_t n, uint32_t k, uint64_t seed,
                             sassi_inj_site* host_out, void* stream);

/* Multi-GPU: merge the tables of all ranks of `nccl_comm` (ncclComm_t) in place with one
 * ncclAllReduce(sum, uint64) over a packed image (AND masks carried as byte-expanded bits); with
 * dynamic pcs enabled, also an ncclAllGather of every rank's dynamic table, which each rank
 * re-inserts into a cleared table (every rank then holds the same entries).
 * A 2-word allreduce first compares the ranks' site-table checksums. The first merge of a context
 * over a communicator (and every merge with dynamic pcs enabled) synchronises `stream` to check it
 * on the host (EMISMATCH before any table traffic); later merges check it on the device with no
 * host round trip: a mismatch then leaves the tables unmerged and the next sassi_read_tables
 * returns EMISMATCH. A configuration change (sassi_select_memdiv_pcs, sassi_enable_dynamic_pcs)
 * must be made identically on every rank.
 * Collective: every rank must call it. Errors: ENCCL, EMISMATCH (site tables differ). */
int sassi_merge(struct sassi_ctx* ctx, void* nccl_comm, void* stream);

/* The same merge for n contexts on ONE device (e.g. warp shards folded into separate contexts, or
 * one context per stream): every context ends with the merged tables. It runs sassi_merge's pack
 * and unpack kernels with the allreduce replaced by a device sum of the n packed images
 * (isScalar / mask bytes compared with n), and merges dynamic-pc tables like sassi_merge.
 * Stream-ordered, no host synchronisation. ctxs: HOST array of n distinct contexts (n <= 255) with
 * identical site tables, warps and pc selections (EMISMATCH otherwise), all on one device (EINVAL). */
int sassi_merge_local(struct sassi_ctx* const* ctxs, uint32_t n, void* stream);

/* ---- Fused fold + merge over peer memory (one node: NVLink / NVSwitch P2P, or one device) ----
 * Instead of folding and then running sassi_merge's collective, every rank can fold straight into
 * every rank's table image: each rank exports its image (a CUDA IPC handle of SASSI_IPC_HANDLE_BYTES
 * bytes, exchanged by the caller, e.g. torch.distributed.all_gather_object) and opens the others'
 * with sassi_add_peer_table. From then on every table update of sassi_consume (the CTA-exit flush
 * and the per-thread count adds) is also applied, as an atomic over NVLink, to each peer's image:
 * sums add and the AND masks AND (PAPER.md's tables are commutative folds), so once every rank's
 * folds have completed every image holds the merged tables — sassi_merge's result without a
 * collective. Protocol: sassi_reset on every rank, a barrier, the folds, a barrier (each after a
 * stream synchronise), then sassi_read_tables anywhere. The dynamic-pc table and the inline
 * handlers of sassi_ik_run are not included (use sassi_merge for those).
 * sassi_add_peer_table: only before the first consume or right after sassi_reset; the peer's image
 * must have this context's layout (EMISMATCH otherwise); at most 7 peers (ENOSPC). While peers are
 * attached the handler set cannot change (sassi_attach_handler: ESTATE).
 * sassi_clear_peer_tables synchronises the device and closes the handles. */
#define SASSI_IPC_HANDLE_BYTES 64
int sassi_ipc_table_handle(struct sassi_ctx* ctx, void* handle_out);
int sassi_add_peer_table(struct sassi_ctx* ctx, const void* handle);
int sassi_clear_peer_tables(struct sassi_ctx* ctx);

/* NCCL bootstrap helpers (NCCL is loaded lazily with dlopen; only sassi_merge needs it). */
int sassi_nccl_get_unique_id(void* out_128_bytes);
int sassi_nccl_comm_create(void** comm_out, int nranks, int rank, const void* unique_id_128_bytes,
                           int device);
int sassi_nccl_comm_destroy(void* comm);

/* Number of kernels this context launched so far (for the bench's launch count). */
int sassi_kernel_launches(struct sassi_ctx* ctx, uint64_t* out);

const char* sassi_strerror(int status);
/* Message of the most recent failing call in this process (thread-local). */
const char* sassi_last_error(void);

#ifdef __cplusplus
}
#endif

#endif /* SASSI_H_ */
