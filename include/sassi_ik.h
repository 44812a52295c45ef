/*
 * sassi_ik.h — instrumented synthetic kernels (north_star subsystem 4).
 *
 * Four CUDA kernels with hand-placed instrumentation sites, each runnable
 *   - uninstrumented (SASSI_IK_NONE) — the baseline t / k of Table 3;
 *   - with inline handlers folding straight into a sassi_ctx's tables: one handler
 *     (SASSI_H_BRANCH / MEMDIV / VALUE / INSTCOUNT / INSTMIX), the four case studies
 *     (SASSI_H_ALL) or every handler (SASSI_H_EVERY);
 *   - with a null handler called through a non-inlined ABI call with stack-allocated parameter
 *     objects (SASSI_IK_NULL_ABI) — the paper's stubbed-handler experiment (L687);
 *   - in trace mode (SASSI_IK_TRACE), appending SRF1 records per warp, so the same execution can
 *     be folded by sassi_consume and compared with the inline tables.
 * Kernels: SASSI_IK_VECADD (c1 shape: grid-stride vector add + divergent i%3 branch guarding a
 * 128 B-stride load), SASSI_IK_BFS (pull-style relaxation over a CSR graph: gathers, data-dependent
 * trip counts), SASSI_IK_SGEMM (fp32 shared-memory tiled GEMM on CUDA cores), SASSI_IK_STENCIL
 * (5-point 2-D stencil with a divergent boundary test).
 * All functions return sassi_status codes (include/sassi.h); all buffers are owned by the object.
 */
#ifndef SASSI_IK_H_
#define SASSI_IK_H_

#include "sassi.h"

#ifdef __cplusplus
extern "C" {
#endif

enum { SASSI_IK_VECADD = 0, SASSI_IK_BFS = 1, SASSI_IK_SGEMM = 2, SASSI_IK_STENCIL = 3 };
enum { SASSI_IK_NONE = 0u, SASSI_IK_TRACE = 64u, SASSI_IK_NULL_ABI = 128u,  /* above SASSI_H_EVERY */
       SASSI_IK_SMEM = 1024u };  /* | a handler mask: opt-in per-CTA shared-memory aggregation */

typedef struct sassi_ik sassi_ik;

/* Build a kernel instance: `size` scales the problem (elements / nodes / matrix dim / grid dim;
 * 0 = the default timing size), inputs are filled on the device from `seed`. */
int sassi_ik_create(sassi_ik** out, int kernel, uint32_t size, uint64_t seed, int device);
void sassi_ik_destroy(sassi_ik* ik);

/* The kernel's static site table (register it with sassi_ctx_create(sites, n_warps)). */
int sassi_ik_sites(sassi_ik* ik, sassi_site* out, uint32_t cap, uint32_t* n_sites, uint32_t* n_warps);

/* Run once. mode = SASSI_IK_NONE | SASSI_IK_NULL_ABI | SASSI_IK_TRACE | one of the handler masks
 * above (1, 2, 4, 8, 16, 15, 31; EINVAL otherwise), optionally | SASSI_IK_SMEM. By default the
 * inline handlers use no shared memory (a handler's use of it can break or slow a kernel that needs
 * it all): each warp's totals go to global memory at kernel exit. SASSI_IK_SMEM opts
 * in to per-CTA tables in shared memory (the warps fold into them at exit, one flush per CTA; up
 * to 14 words per site + 8 KB with memdiv), which is faster for kernels of many short-lived warps;
 * handler bits fold into ctx's tables (ctx must hold exactly this kernel's sites / warps).
 * Asynchronous on `stream` except SASSI_IK_TRACE, which synchronises. */
int sassi_ik_run(sassi_ik* ik, uint32_t mode, struct sassi_ctx* ctx, void* stream);

/* After a TRACE run: totals of the warp-major SRF1 stream the run produced (EFORMAT if a warp
 * overflowed its trace region), and a copy of that stream into caller-owned DEVICE buffers
 * (hdr[n_rec], addr[n_addr_rows][32], val[n_val_rows][32]); build its chunk index with
 * sassi_index_records. */
int sassi_ik_trace_totals(sassi_ik* ik, uint64_t* n_rec, uint64_t* n_addr_rows, uint64_t* n_val_rows);
int sassi_ik_trace_copy(sassi_ik* ik, sassi_hdr* hdr, uint64_t* addr, uint32_t* val, void* stream);

/* ---- Online trace mode ("SASSI traces driving other tools") ----
 * Trace the kernel and fold its records into ctx's tables segment by segment, each segment's
 * fold overlapping the tracing of the next. First a count pass runs the kernel once counting
 * every warp's records and payload rows (exclusive prefixes over the warps give each warp's place
 * in the warp-major SRF1 stream). Then, per segment of `blocks_per_segment` thread blocks (0 = at
 * least 4 segments of about 1 GiB of trace each), the producer (the caller's `stream`) runs the
 * segment's blocks in trace mode writing every record and row straight into its final place in
 * one of two ring slots sized for the largest segment; a consumer stream owned by the instance
 * builds the slot's chunk index (sassi_index_records), runs sassi_consume on it and frees the slot
 * for the segment after next. The pipeline is enqueued without host round trips. Device memory is
 * bounded by two segments, not by the length of the trace. The kernel must be deterministic
 * (the four synthetic kernels are): the trace pass checks its counts against the count pass.
 * The result equals sassi_consume over the whole-kernel TRACE stream (and the inline handlers'
 * tables): every table is a fold that does not depend on record order.
 * flags: SASSI_IK_SERIAL disables the overlap (each segment is folded before the next is traced;
 * for measurement). ctx must hold exactly this kernel's sites / warps with handlers attached.
 * Blocking: returns after the last fold (stream synchronised). Errors: EINVAL, ESTATE, ECUDA,
 * EFORMAT (the trace pass produced other counts than the count pass). `stats` (may be NULL)
 * receives the totals. */
enum { SASSI_IK_SERIAL = 1u };
typedef struct sassi_ik_trace_stats {
  uint64_t n_records, n_addr_rows, n_val_rows;  /* folded, over all segments                  */
  uint64_t max_segment_records;                 /* the largest segment                        */
  uint64_t ring_bytes;                          /* device bytes of the two ring slots + counts */
  uint32_t segments, blocks_per_segment;
} sassi_ik_trace_stats;                         /* 48 B */
int sassi_ik_trace_fold(sassi_ik* ik, struct sassi_ctx* ctx, uint32_t blocks_per_segment,
                        uint32_t flags, sassi_ik_trace_stats* stats, void* stream);

/* Checksum of the kernel's output buffers (to prove instrumentation does not change results). */
int sassi_ik_output_checksum(sassi_ik* ik, uint64_t* out);

/* ---- Error injection (§8.1 step 3, L631-L633) -------------------------------
 * One run per tuple (tuples as sassi_sample_sites draws them from a SASSI_H_INSTCOUNT profile of
 * the same kernel): the thread `thread` counts its eligible, not-predicated-out dynamic
 * instructions (the ones the profile counted, L627) and at number `dyn_index` (0-based) flips bit
 * bit_seed % 32 of the value its destination register receives — the kernel continues with the
 * corrupted value — or, for a store, of the 32-bit word it wrote (reading R23). The run
 * is classified against an error-free reference run (L633):
 *   MASKED       outputs identical
 *   SDC          outputs differ (potential silent data corruption)
 *   DUE          a corrupted data-dependent index left its array (the crash analogue: the
 *                kernel checks the index, records the symptom and skips the access)
 *   HANG         a loop ran past its watchdog (kHangCap trips)
 *   NOT_REACHED  the thread executed fewer eligible instructions (outputs unchanged)
 * Synchronises `stream` after every run; leaves the outputs as an error-free run leaves them. */
enum { SASSI_INJ_MASKED = 0, SASSI_INJ_SDC = 1, SASSI_INJ_DUE = 2, SASSI_INJ_HANG = 3,
       SASSI_INJ_NOT_REACHED = 4 };
enum { SASSI_INJ_TARGET_GPR = 0, SASSI_INJ_TARGET_MEM = 1 };
typedef struct sassi_ik_outcome {
  uint32_t outcome;         /* SASSI_INJ_*                                                      */
  uint32_t site;            /* static site of the injected instruction (0xFFFFFFFF: not reached) */
  uint32_t target;          /* SASSI_INJ_TARGET_*                                               */
  uint32_t bit;             /* flipped bit                                                      */
  uint32_t before, after;   /* the value (GPR) or stored word (MEM) before / after the flip     */
  uint32_t reserved[2];
} sassi_ik_outcome;         /* 32 B */
int sassi_ik_inject(sassi_ik* ik, const sassi_inj_site* sites, uint32_t n, sassi_ik_outcome* out,
                    void* stream);

#ifdef __cplusplus
}
#endif

#endif /* SASSI_IK_H_ */
