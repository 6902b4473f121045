/*
 * medusa.h -- C ABI of libmedusa.so, the B200 (sm_100a) implementation of the
 * data-parallel hot path of Medusa's CUDA-graph state materialization
 * (Zeng et al., "Medusa: Accelerating Serverless LLM Inference with
 * Materialization", ASPLOS'25; citations P:<line> are lines of the paper text).
 *
 *   medusa_materialize      offline: indirect-index-pointer analysis (§4.1,
 *                           P:204-212) of every 8-byte word of every captured
 *                           kernel node's parameter image against the
 *                           allocation trace -> the indirect index pointer
 *                           table.
 *   medusa_kernel_table_set online: install the kernel addresses resolved by the
 *                           triggering kernels (§5).
 *   medusa_restore          online: replay-based data pointer restoration
 *                           (§4.2) with per-slot validation
 *                           and the kernel-address fill of every node.
 *
 * Conventions (all entry points)
 *   - d_* arguments are DEVICE pointers on the calling thread's current CUDA
 *     device; h_* are host pointers.  All memory is owned by the caller; the
 *     library never frees caller memory.  It owns only a per-device kernel
 *     address table and internal scratch that it allocates itself.
 *   - 64-bit values are little-endian; pointers to u64 arrays must be 8-byte
 *     aligned (16-byte alignment of word arrays enables the vectorised path).
 *   - The return value reports argument, trace and launch errors only.
 *     Data-dependent validation failures of a restore are not call errors:
 *     they are counted in the device-side medusa_report (the call is async).
 *   - Thread-safe: calls may come from several host threads and devices; calls
 *     on different devices never wait for each other.  The materialize entry
 *     points of one device share that device's scratch: the synchronous one
 *     holds the device's lock until its work is done (other threads' materialize
 *     calls on that device wait); an asynchronous one holds it while enqueueing
 *     only and must be ordered (same stream, or events) against every other
 *     materialize on the device.
 *   - Work is enqueued on the caller's `stream`.  Materialize forks part of its
 *     work onto an internal stream and joins it back before returning, so the
 *     call is one stream-ordered unit (and capturable, see below).
 *   - There is no CPU fallback: without a usable sm_100a device every call
 *     that would touch the GPU returns MEDUSA_ERR_CUDA.
 */
#ifndef MEDUSA_H
#define MEDUSA_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#ifndef __DRIVER_TYPES_H__
typedef struct CUstream_st *cudaStream_t; /* identical to CUDA's own typedef */
#endif

typedef enum {
    MEDUSA_OK = 0,
    MEDUSA_ERR_INVALID_ARG = -1, /* bad pointer/size/alignment, or an input that breaks
                                    the contract below (limits, CSR shape, launch order) */
    MEDUSA_ERR_TRACE = -2,       /* allocation trace is not well-formed (see medusa_materialize) */
    MEDUSA_ERR_CAPACITY = -3,    /* slot table too small; *h_n_slots holds the size needed */
    MEDUSA_ERR_NO_TABLE = -4,    /* restore asked for the kernel-address fill before any
                                    medusa_kernel_table_set on this device */
    MEDUSA_ERR_CUDA = -5,        /* CUDA runtime error; see medusa_last_cuda_error() */
    MEDUSA_ERR_RETRY = -6        /* (medusa_materialize_async result only) the library's
                                    scratch was too small for this trace: call
                                    medusa_materialize once, which sizes it exactly */
} medusa_status;

/* One allocation of the trace, 24 bytes.  Its index in the trace array is the
 * allocation ordinal -- the paper's "indirect index pointer" i: "if a pointer is
 * returned by the i-th buffer allocation, its corresponding indirect index
 * pointer is i".  base/size: the returned address and the recorded
 * extent [base, base+size).  t_alloc/t_free: positions of the allocation and of
 * its free in the one total order of allocation, free and cudaLaunchKernel
 * events.  t_free = MEDUSA_T_END: never freed.  The allocation is live
 * at event position t iff t_alloc < t < t_free. */
typedef struct {
    uint64_t base;
    uint64_t size;
    uint32_t t_alloc;
    uint32_t t_free;
} medusa_alloc;

/* The materialized indirect-index-pointer table, in device memory the
 * caller owns.  For an image of n_words words:
 *   d_mask:       u32[ceil(n_words/32)]; bit (g % 32) of d_mask[g / 32] is 1 iff
 *                 word g is a data pointer slot;
 *   d_chunk_base: u32[ceil(n_words/MEDUSA_CHUNK_WORDS) + 1]; entry c = number of
 *                 slots among words [0, c*MEDUSA_CHUNK_WORDS); the last entry is
 *                 the total;
 *   d_slot:       u64[capacity]; the k-th slot in word order as
 *                 (allocation index << MEDUSA_OFF_BITS) | byte offset.        */
typedef struct {
    uint32_t *d_mask;
    uint32_t *d_chunk_base;
    uint64_t *d_slot;
    uint64_t capacity;
} medusa_slots;

/* Restore report (device memory, 64 bytes).  "none" = UINT64_MAX.
 *   n_bad_slot     slots that failed validation (= n_bad_id + n_bad_range + n_stale);
 *                  a failing slot leaves the source word in place
 *   first_bad_word least word index of a failing slot
 *   n_bad_id       slot's allocation index >= n_alloc of the replay
 *   n_bad_range    slot's offset >= the replayed allocation's size
 *   n_stale        source word != old_base[i] + offset (the image no longer holds
 *                  the pointer that was materialized)
 *   n_bad_func     nodes whose kernel-name id is >= the table size or maps to 0
 *                  (unresolved); their func_out is 0
 *   first_bad_node least such node index
 *   n_bad_chunk    chunks whose d_chunk_base range disagrees with their mask
 *                  (see medusa_restore, "table consistency"); their words are
 *                  copied unchanged and their slots counted nowhere else     */
typedef struct {
    uint64_t n_bad_slot, first_bad_word, n_bad_id, n_bad_range, n_stale;
    uint64_t n_bad_func, first_bad_node, n_bad_chunk;
} medusa_report;

#define MEDUSA_CHUNK_WORDS 2048u   /* chunk size of d_chunk_base (fixed; part of the ABI) */
#define MEDUSA_ID_BITS 24u         /* allocation index < 2^24 */
#define MEDUSA_OFF_BITS 40u        /* byte offset < 2^40 */
#define MEDUSA_T_END 0xFFFFFFFFu   /* t_free of an allocation that is never freed */

/* medusa_materialize -- offline analysis stage (§4.1).
 *
 * Inputs (device):
 *   d_words[n_words]          every kernel node's parameter image (the bytes the
 *                             node's param array points to), each zero-
 *                             padded to a multiple of 8 bytes and concatenated in
 *                             node order; word g = the u64 at byte 8*g;
 *   d_node_word_off[n_nodes+1] CSR: node j owns words [off[j], off[j+1]);
 *                             off[0] = 0, non-decreasing, off[n_nodes] = n_words;
 *   d_node_t[n_nodes]         event position of node j's cudaLaunchKernel; nodes
 *                             are listed in launch order (strictly increasing);
 *   d_alloc[n_alloc]          the allocation trace.
 * Output: *slots filled (see medusa_slots), *h_n_slots = number of slots.
 *
 * Semantics: word g of node j with value w is a slot (i, w - base_i) iff
 * allocation i is live at node j's launch and base_i <= w < base_i + size_i
 * ("identical or within the range of the allocated buffer").  On a
 * well-formed trace at most one such i exists; it is exactly the first match of
 * the paper's backward search from the launch among allocations not yet
 * freed ("kernels would always use the allocated buffers before they have been
 * deallocated").  Every other word is a constant.
 *
 * Errors:
 *   MEDUSA_ERR_INVALID_ARG: null pointers where data is needed; n_alloc > 2^24;
 *     n_words >= 2^32; some size > 2^40 or base + size wraps past 2^64; the CSR
 *     is malformed; node times not strictly increasing.
 *   MEDUSA_ERR_TRACE: t_alloc not strictly increasing in the index, some
 *     t_alloc >= t_free, or two allocations live at the same time overlap in
 *     address (zero-size allocations overlap nothing).
 *   MEDUSA_ERR_CAPACITY: slots->capacity < number of slots.  d_mask and
 *     d_chunk_base are complete, d_slot holds the first `capacity` records and
 *     *h_n_slots the number needed.
 * On INVALID_ARG / TRACE the outputs are unspecified and *h_n_slots = 0.
 * Work is ordered on `stream`; the call synchronizes `stream` before returning
 * (it reads the slot count back).  Scratch is allocated by the library.      */
medusa_status medusa_materialize(const uint64_t *d_words, uint64_t n_words,
                                 const uint64_t *d_node_word_off, uint32_t n_nodes,
                                 const uint32_t *d_node_t,
                                 const medusa_alloc *d_alloc, uint32_t n_alloc,
                                 medusa_slots *slots, uint64_t *h_n_slots,
                                 cudaStream_t stream);

/* Result of medusa_materialize_async, written to device memory (16 bytes):
 * status = one of medusa_status (OK, INVALID_ARG, TRACE, CAPACITY, RETRY),
 * n_slots as *h_n_slots of medusa_materialize. */
typedef struct {
    int32_t status;
    uint32_t reserved;
    uint64_t n_slots;
} medusa_mat_result;

/* medusa_materialize_async -- the same analysis as medusa_materialize, fully
 * asynchronous on `stream` (no host synchronization; capturable into a CUDA
 * graph once the library's scratch has been sized by one medusa_materialize
 * call on this device for a trace of the same or larger size).  The data-
 * dependent outcome goes to *d_result (device); host-detectable argument errors
 * are returned synchronously.  If d_result->status is not MEDUSA_OK, the table
 * and anything computed from it are unspecified.  Calls on one device must be
 * ordered (one stream, or events): they share the device's scratch. */
medusa_status medusa_materialize_async(const uint64_t *d_words, uint64_t n_words,
                                       const uint64_t *d_node_word_off, uint32_t n_nodes,
                                       const uint32_t *d_node_t,
                                       const medusa_alloc *d_alloc, uint32_t n_alloc,
                                       medusa_slots *slots, medusa_mat_result *d_result,
                                       cudaStream_t stream);

/* n_slots value for medusa_restore: take the slot count from the table itself
 * (d_chunk_base), e.g. after medusa_materialize_async with no host round trip. */
#define MEDUSA_N_SLOTS_FROM_TABLE UINT64_MAX

/* medusa_kernel_table_set -- install, for the current device, the kernel
 * address of every kernel-name id: d_func_addr[n_func] (device),
 * 0 = unresolved.  In the paper these come from dlsym / cudaGetFuncBySymbol and,
 * for kernels hidden from the symbol tables, from enumerating the modules that
 * the triggering kernels (the model's first layer) loaded.
 * The copy is ordered on `stream`; a later medusa_restore must be ordered after
 * it (same stream, or an event).  Replaces any previous table of this device.
 * The first call on a device (or one with a larger n_func) allocates the table:
 * make it before capturing a CUDA graph that contains this call.             */
medusa_status medusa_kernel_table_set(const uint64_t *d_func_addr, uint32_t n_func,
                                      cudaStream_t stream);

/* medusa_restore -- online restoration (§4.2; §5).
 *
 *   dst = src; then for every slot k (word g, allocation i, offset off) of the
 *   table produced by medusa_materialize:
 *     i >= n_alloc                   -> n_bad_id
 *     off >= d_new_size[i]           -> n_bad_range
 *     src[g] != d_old_base[i] + off  -> n_stale          (u64 wrap-around)
 *     otherwise dst[g] = d_new_base[i] + off              (u64 wrap-around)
 *   d_new_base[i] is the address the i-th allocation returned when the
 *   (de)allocation sequence was replayed.  Non-slot words
 *   are copied unchanged (constants keep their plain values).
 *   Table consistency (DESIGN.md R-TABLE; a table medusa_materialize wrote is
 *   always consistent): chunk c (words [2048c, 2048c + 2048)) is consistent iff
 *   d_chunk_base[c+1] - d_chunk_base[c] (>= 0) equals the number of mask bits of
 *   its words (bits of words >= n_words are ignored).  Then its i-th slot word
 *   (ascending) pairs with record d_chunk_base[c] + i; a record index >= n_slots
 *   means the record is missing: that slot counts as n_bad_id.  An inconsistent
 *   chunk is copied unchanged and counted once in n_bad_chunk.
 *   Kernel-address fill: d_func_out[j] = table[d_func_id[j]] if the id is below
 *   the installed table's size and the entry is non-zero, else 0 (n_bad_func).
 *   d_func_id, d_func_out, n_nodes: all NULL/0 to skip the fill.
 *
 * src/dst: u64[n_words], device; dst == src (in place) is allowed, any other
 * overlap is MEDUSA_ERR_INVALID_ARG.  slots: as produced by medusa_materialize
 * for this image (n_slots = *h_n_slots, or MEDUSA_N_SLOTS_FROM_TABLE).  d_old_base: the trace's base of each
 * allocation (the materialization-time addresses).  d_report (device) is
 * written completely by the call.  Fully asynchronous on `stream`; capturable
 * into a CUDA graph.                                                         */
medusa_status medusa_restore(const uint64_t *d_src_words, uint64_t *d_dst_words, uint64_t n_words,
                             const medusa_slots *slots, uint64_t n_slots,
                             const uint64_t *d_old_base, const uint64_t *d_new_base,
                             const uint64_t *d_new_size, uint32_t n_alloc,
                             const uint32_t *d_func_id, uint64_t *d_func_out, uint32_t n_nodes,
                             medusa_report *d_report, cudaStream_t stream);

/* ---- copy-free buffer contents restoration (§4.3) ------------
 *
 * Besides the pointers, the contents of the buffers the graph nodes point to
 * must be right.  Most need no saving: model-parameter buffers are
 * "allocated before the CUDA graphs capturing" and temporary buffers
 * are allocated during a capture and "deallocated after capturing".
 * Only the permanent ones -- allocated during a capture, never freed, "used
 * across different launches of CUDA graphs" (two 4-byte buffers for
 * 9.0% of the kernels) -- are dumped offline and copied back online.
 *
 * Class of allocation i (d_class[i]):                                         */
#define MEDUSA_BUF_UNUSED 0u /* no slot of the table refers to it (not a graph parameter) */
#define MEDUSA_BUF_PARAM 1u  /* t_alloc inside no capture interval: "allocated before the CUDA
                                graphs capturing" -- contents not saved */
#define MEDUSA_BUF_TEMP 2u   /* allocated during a capture, freed (t_free != MEDUSA_T_END):
                                temporary -- contents discarded */
#define MEDUSA_BUF_PERM 3u   /* allocated during a capture, never freed: permanent
                                -- contents saved and restored */

/* Save / restore report (device memory, 16 bytes): segments not copied and the
 * least such segment index k ("none" = UINT64_MAX). */
typedef struct {
    uint64_t n_bad, first_bad;
} medusa_buf_report;

/* medusa_buffers_plan -- offline: classify every allocation and lay out the blob.
 *
 * Inputs (device): d_alloc[n_alloc] the trace given to medusa_materialize;
 *   d_capture_t[2*n_capture] the event positions (begin, end) of every graph
 *   capture, in the same total order as the trace (cudaStreamBeginCapture /
 *   EndCapture); intervals must satisfy begin < end and end_k <= begin_{k+1}
 *   (graphs are captured one at a time), else MEDUSA_ERR_INVALID_ARG.
 *   Allocation i is made during capture k iff begin_k < t_alloc_i < end_k.
 *   d_slot[n_slots]: the materialized slot records; records whose allocation
 *   index is >= n_alloc are ignored.
 * Outputs (device, caller-owned): d_class u8[n_alloc] (MEDUSA_BUF_*);
 *   d_perm u32[perm_capacity]: the PERM allocation indices, increasing;
 *   d_perm_off u64[perm_capacity + 1]: segment k of the blob is
 *   [d_perm_off[k], d_perm_off[k+1]) and holds the d_alloc[].size bytes of
 *   allocation d_perm[k]; d_perm_off[n_perm] = blob size.
 *   *h_n_perm, *h_blob_bytes (host).  perm_capacity = n_alloc always suffices.
 * Errors: INVALID_ARG (null / misaligned pointers, bad capture intervals),
 *   CAPACITY (n_perm > perm_capacity: d_class complete, *h_n_perm and
 *   *h_blob_bytes hold the sizes needed, the lists are truncated).
 * Synchronizes `stream` (reads the counts back).                             */
medusa_status medusa_buffers_plan(const medusa_alloc *d_alloc, uint32_t n_alloc,
                                  const uint32_t *d_capture_t, uint32_t n_capture,
                                  const uint64_t *d_slot, uint64_t n_slots,
                                  uint8_t *d_class, uint32_t *d_perm, uint64_t *d_perm_off,
                                  uint32_t perm_capacity, uint32_t *h_n_perm, uint64_t *h_blob_bytes,
                                  cudaStream_t stream);

/* medusa_buffers_save -- offline: d_blob[d_perm_off[k] ...] = the bytes of
 * allocation d_perm[k] at address d_base[d_perm[k]] (device memory of this
 * process, normally the trace's bases).  d_perm / d_perm_off / n_perm as
 * produced by medusa_buffers_plan; d_blob: u8[d_perm_off[n_perm]], 16-byte
 * aligned, not overlapping any saved buffer.  Segments with d_perm[k] >=
 * n_alloc are not copied and counted in *d_report.  Fully asynchronous on
 * `stream`; capturable.                                                      */
medusa_status medusa_buffers_save(const uint32_t *d_perm, const uint64_t *d_perm_off, uint32_t n_perm,
                                  const uint64_t *d_base, uint32_t n_alloc, uint8_t *d_blob,
                                  medusa_buf_report *d_report, cudaStream_t stream);

/* medusa_buffers_restore -- online: copy segment k of d_blob to
 * d_new_base[d_perm[k]], the address the replayed allocation returned (P:176,
 * P:186), unless d_perm[k] >= n_alloc (the replay made fewer allocations) or
 * the segment is longer than d_new_size[d_perm[k]]; those segments are not
 * copied and are counted in *d_report (DESIGN.md R-B4).  No other byte is
 * written.  Targets must not overlap the blob or each other.  Fully
 * asynchronous on `stream`; capturable.                                      */
medusa_status medusa_buffers_restore(const uint8_t *d_blob, const uint32_t *d_perm, const uint64_t *d_perm_off,
                                     uint32_t n_perm, const uint64_t *d_new_base, const uint64_t *d_new_size,
                                     uint32_t n_alloc, medusa_buf_report *d_report, cudaStream_t stream);

/* ---- library-owned memory ------------------------------------------------
 * medusa_materialize / _async use per-device scratch the library allocates and
 * grows on demand (x1.5 past the previous size); medusa_kernel_table_set owns a
 * per-device table.  A growth never frees the buffers it replaces: a CUDA graph
 * that captured an earlier call holds their addresses by value, so replaying it
 * stays memory-safe (it keeps reading and writing the old, still-allocated
 * buffers).  They are freed only by medusa_scratch_release or at process exit.
 *
 * medusa_scratch_bytes: live scratch bytes of the current device (retired
 *   buffers excluded).
 * medusa_scratch_release: synchronizes the current device, then frees its
 *   scratch, every retired scratch buffer and every retired kernel table (the
 *   installed table stays).  Every CUDA graph that captured a materialize or a
 *   retired table on this device is invalid afterwards and must not be replayed.
 *   The next materialize reallocates (outside any capture).                   */
uint64_t medusa_scratch_bytes(void);
medusa_status medusa_scratch_release(void);

/* cudaError_t value behind the last MEDUSA_ERR_CUDA returned on this thread. */
int medusa_last_cuda_error(void);

/* Human-readable name of a status code (static storage). */
const char *medusa_status_string(medusa_status status);

/* ---- instrumentation (optional; off by default) --------------------------
 * When enabled on a thread, every kernel libmedusa launches from that thread is
 * bracketed by CUDA events recorded on its launch stream.  medusa_timing_read
 * waits for those events and returns up to `max` (name, milliseconds) pairs of
 * the launches since the last read (then forgets them).                      */
void medusa_timing_enable(int on);
int medusa_timing_read(const char **names, float *ms, int max);

#ifdef __cplusplus
}
#endif

#endif /* MEDUSA_H */
