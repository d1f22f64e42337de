/*
 * ga_bench.h -- C ABI of the workload kernels the tests and bench.py call.
 *
 * A trace is u32 sizes[R][T] in DEVICE memory (round-major; 0 = no malloc),
 * with free depth D (tracegen/__init__.py):
 *   D == 1: at round r each thread frees its round r-1 block, then mallocs
 *           sizes[r][t]; round R is a free-all round;
 *   D == 0: at round r every thread mallocs, then every round-r block is freed.
 * Thread t of the trace is global thread t of the launch; blocks of `block`
 * threads (0 -> 256).  Failed mallocs count as calls (R-17).
 *
 * counts (DEVICE u64[8], accumulated, caller zeroes): [0] malloc calls,
 * [1] NULL returns, [2] frees, [3] tag errors (a block's two 8-byte tags, written
 * after malloc, differed at free time: an overlap while live).
 *
 * Log (correctness mode, optional): 16-byte records at 2*(round*T + t) + op,
 * op 0 = malloc, 1 = free: u64 offset from the heap base (~0 = NULL / none),
 * u32 requested size, u32 t | round << 20 | op << 31 (0 for empty records).
 * Same format as the oracle's log (oracle/ga_oracle.c), written independently.
 *
 * Errors: GA_EINVAL for null pointers / T == 0 / D > 1 / round out of range;
 * GA_ECUDA when a launch fails.  All calls are asynchronous on `stream` except
 * the *_host variant, which synchronises.
 */
#ifndef GA_BENCH_H_
#define GA_BENCH_H_

#include "ga.h"

#ifdef __cplusplus
extern "C" {
#endif

typedef struct { uint64_t off; uint32_t size; uint32_t meta; } ga_log_rec;

enum { GA_TRACE_LOG = 1, GA_TRACE_TAG = 2 };

/* Scope of the allocator calls a trace kernel makes (flags bits 8..11 of
 * ga_trace_phase, `scope` of ga_trace_timed_scope):
 *   0     -- warp path: ga_malloc / ga_free (include/ga_device.cuh);
 *   1     -- block-collective: ga_malloc_block / ga_free_block;
 *   2..8  -- cluster-collective over clusters of that many CTAs:
 *            ga_malloc_cluster / ga_free_cluster (the grid is padded to a
 *            multiple of the cluster; block * cluster <= 2048).
 * Collective kernels keep every thread in every call (threads past T pass
 * n == 0 / NULL).  Invalid scopes return GA_EINVAL. */
#define GA_TRACE_SCOPE(s) ((uint32_t)(s) << 8)

/* Correctness mode: one kernel per phase.  held: DEVICE u64[2*T] (block, size),
 * all ~0 / 0 before round 0.  D == 1: round in [0, R], phase ignored.
 * D == 0: round in [0, R), phase 0 = malloc, 1 = free. */
ga_status ga_trace_phase(ga_heap_t h, ga_stream_t stream, const uint32_t* sizes, uint32_t R,
                         uint32_t T, uint32_t D, uint32_t round, uint32_t phase, uint64_t* held,
                         ga_log_rec* log, uint64_t* counts, uint32_t flags, uint32_t block);

/* Timing mode: ONE kernel runs every round (and the free-all) with no log,
 * no tags and no extra memory traffic: the allocator alone. */
ga_status ga_trace_timed(ga_heap_t h, ga_stream_t stream, const uint32_t* sizes, uint32_t R,
                         uint32_t T, uint32_t D, uint64_t* counts, uint32_t block);

/* ga_trace_timed with the calls at `scope` (see GA_TRACE_SCOPE; 0 is
 * ga_trace_timed itself). */
ga_status ga_trace_timed_scope(ga_heap_t h, ga_stream_t stream, const uint32_t* sizes, uint32_t R,
                               uint32_t T, uint32_t D, uint64_t* counts, uint32_t block, uint32_t scope);

/* End-to-end: HOST sizes (pinned for overlap) copied H2D, the timed kernel,
 * counts copied D2H into host u64[4]; synchronises `stream`.  Scratch device
 * buffers are cached in the heap handle. */
ga_status ga_trace_timed_host(ga_heap_t h, ga_stream_t stream, const uint32_t* host_sizes,
                              uint32_t R, uint32_t T, uint32_t D, uint64_t* host_counts,
                              uint32_t block);

/* Device-API edge cases (readings R-15, R-16): thread t < T calls
 * ga_malloc(sizes[t]) with any u64 size (0 and sizes above the heap return
 * NULL and are not failures), writes the offset from the heap base to offs[t]
 * (~0 = NULL), calls ga_free(NULL) (a no-op), and with flags & 1 frees its
 * block.  sizes, offs: DEVICE u64[T].  T need not be a multiple of 32, so the
 * last warp runs partial. */
ga_status ga_edge_calls(ga_heap_t h, ga_stream_t stream, const uint64_t* sizes, uint32_t T,
                        uint64_t* offs, uint32_t flags, uint32_t block);

/* The same workloads on CUDA's built-in device malloc/free (the baseline of
 * P:L1490-1494).  Set the CUDA heap limit before the first such launch. */
ga_status ga_cuda_set_heap_limit(size_t bytes);
ga_status ga_cuda_trace_phase(ga_stream_t stream, const uint32_t* sizes, uint32_t R, uint32_t T,
                              uint32_t D, uint32_t round, uint32_t phase, uint64_t* held,
                              uint64_t* counts, uint32_t flags, uint32_t block);
ga_status ga_cuda_trace_timed(ga_stream_t stream, const uint32_t* sizes, uint32_t R, uint32_t T,
                              uint32_t D, uint64_t* counts, uint32_t block);

/* Registers per thread and resident blocks per SM of the trace kernels.
 * which: 0 ga timed, 1 ga phase, 2 cuda timed. */
ga_status ga_kernel_info(int which, uint32_t block, int* regs, int* blocks_per_sm, int* local_bytes);

/* L2-atomic peak microbenchmark (the roofline denominator).
 * Each of grid*block threads performs `iters` 64-bit atomics on d_buf:
 *   pattern 0: ATOMG add, distinct words 32 B apart (spread over L2 slices)
 *   pattern 1: REDG add (no return), distinct words 32 B apart
 *   pattern 2: ATOMG add, one hot word (address not provably uniform: no aggregation)
 *   pattern 3: ATOMG add, 1,184 words 32 B apart (semaphore-like)
 *   pattern 4: CAS increment loop, distinct words 32 B apart
 *   pattern 5: CAS increment loop, one word per SM (148 words)
 * n_words: words available in d_buf (>= grid*block*4 for patterns 0/1/4). */
ga_status ga_l2_atomic_bench(ga_stream_t stream, int pattern, uint64_t* d_buf, uint64_t n_words,
                             uint32_t iters, uint32_t grid, uint32_t block, uint64_t* d_sink);

/* Bulk-semaphore microbenchmark (config d2, Sec. 5.1).
 * variant: 0 warp-aggregated bulk semaphore (ga_bsem_wait: the CUDA path's
 *          fetch-add form, one wait per warp group), 1 per-thread bulk semaphore
 *          in the paper's CAS form (one CAS per decision),
 *          2 per-thread counting semaphore (Sec. 3.2, k forced to 1), 3 plain
 *          per-thread atomicAdd(-k)/(+k), 4 per-thread bulk semaphore in the
 *          fetch-add form (ga_bsem_wait per thread).
 * k: units per thread per wait (1..32); 0 = per-lane random 1..32.
 * B: batch size; n_sems: 1 (global) or one per SM; acquire_only: 1 = Fig. 5
 * mode (no release).  sems: DEVICE u64[n_sems*4] (zeroed by the call).
 * out: DEVICE u64[8]: [0] units granted, [1] waits, [2] batches produced,
 * [3] units produced, [4] sum over sems of final C, [5] max |D|. */
typedef struct {
    uint32_t variant, k, B, n_sems, iters, acquire_only, grid, block;
    uint64_t seed;
} ga_bsem_cfg;
ga_status ga_bsem_bench(ga_stream_t stream, const ga_bsem_cfg* cfg, uint64_t* sems, uint64_t* out);

/* Diagnostics: allocate a host-mapped buffer u64[8 + 4*256] (*host_records)
 * readable while a kernel runs or hangs, and attach it to heap h.  The
 * allocator's safety net (nfc_repair) leaves one dump of the arena it repaired
 * in words 1..7 (every build); -DGA_DEBUG=1 builds also record spin loops that
 * ran ~2^18 iterations as (site, sm|warp|lane, a, b) at [8 + 4i], [0] = count.
 * The buffer lives until process exit.  GA_EINVAL on null arguments. */
ga_status ga_debug_attach(ga_heap_t h, uint64_t** host_records);

#ifdef __cplusplus
}
#endif
#endif /* GA_BENCH_H_ */
