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
enum { SASSI_IK_NONE = 0u, SASSI_IK_TRACE = 64u, SASSI_IK_NULL_ABI = 128u };  /* above SASSI_H_EVERY */

typedef struct sassi_ik sassi_ik;

/* Build a kernel instance: `size` scales the problem (elements / nodes / matrix dim / grid dim;
 * 0 = the default timing size), inputs are filled on the device from `seed`. */
int sassi_ik_create(sassi_ik** out, int kernel, uint32_t size, uint64_t seed, int device);
void sassi_ik_destroy(sassi_ik* ik);

/* The kernel's static site table (register it with sassi_ctx_create(sites, n_warps)). */
int sassi_ik_sites(sassi_ik* ik, sassi_site* out, uint32_t cap, uint32_t* n_sites, uint32_t* n_warps);

/* Run once. mode = SASSI_IK_NONE | SASSI_IK_NULL_ABI | SASSI_IK_TRACE | one of the handler masks
 * above (1, 2, 4, 8, 16, 15, 31; EINVAL otherwise);
 * handler bits fold into ctx's tables (ctx must hold exactly this kernel's sites / warps).
 * Asynchronous on `stream` except SASSI_IK_TRACE, which synchronises. */
int sassi_ik_run(sassi_ik* ik, uint32_t mode, struct sassi_ctx* ctx, void* stream);

/* After a TRACE run: totals of the warp-major SRF1 stream the run produced (EFORMAT if a warp
 * overflowed its trace region), and a copy of that stream into caller-owned DEVICE buffers
 * (hdr[n_rec], addr[n_addr_rows][32], val[n_val_rows][32]); build its chunk index with
 * sassi_index_records. */
int sassi_ik_trace_totals(sassi_ik* ik, uint64_t* n_rec, uint64_t* n_addr_rows, uint64_t* n_val_rows);
int sassi_ik_trace_copy(sassi_ik* ik, sassi_hdr* hdr, uint64_t* addr, uint32_t* val, void* stream);

/* Checksum of the kernel's output buffer (to prove instrumentation does not change results). */
int sassi_ik_output_checksum(sassi_ik* ik, uint64_t* out);

#ifdef __cplusplus
}
#endif

#endif /* SASSI_IK_H_ */
