/*
 * ga_device.cuh -- device interface of the B200-native throughput-oriented allocator.
 *
 *   __device__ void* ga_malloc(ga_dev_heap h, size_t n);
 *   __device__ void  ga_free  (ga_dev_heap h, void* p);
 *
 * The standard malloc / free interface for device threads (Gelado & Garland,
 * PPoPP'19), callable concurrently by every thread of a
 * full-occupancy grid, from converged or divergent code.
 *
 * ga_malloc: rounds n up to a power of two >= 16 B (R-13, R-14); 16..2048 B
 *   come from one-page bins (UAlloc), 4..64 KiB from "spans" (one
 *   64-page chunk split into 64..4 slots, served like bins; DESIGN.md section 7;
 *   GA_NSPAN=0 restores the paper's routing), larger sizes from TBuddy
 *   (P:L834-1016).  Returns a pointer aligned to its class (bins) or its block
 *   size (TBuddy, relative to the 2 MiB aligned base, R-31), or NULL when n == 0,
 *   n exceeds the heap, or no arena can serve the request after every fallback
 *   (R-26, R-27).  Never traps.
 * ga_free: p == NULL is a no-op (R-16).  p must come from ga_malloc on the same
 *   heap and not be freed twice (undefined behaviour otherwise).
 *
 * The lanes of a warp that call at the same time are grouped by size class
 * with __match_any_sync; one leader per group performs the semaphore and bitmap
 * operations for the whole group (the collective critical sections of
 * P:L1246-1312), so a warp-uniform request costs one semaphore atomic per warp.
 * Calls are correct from divergent code, but only lanes that arrive together
 * share a group: under independent thread scheduling, lanes that left an
 * earlier divergent call late arrive alone.  Reconverge first (__syncwarp())
 * when the whole warp calls: on the mixed trace that is 2.7 instead of 1.2
 * lanes per group and 2.3x the throughput.
 *
 * `h` comes from ga_heap_device() (include/ga.h) and is passed by value to the
 * kernel.  Compile with -gencode arch=compute_100a,code=sm_100a.
 */
#ifndef GA_DEVICE_CUH_
#define GA_DEVICE_CUH_

#include "ga.h"
#include "../paper_conf_ppopp_geladog19_b200/csrc/ga_device_impl.cuh"

__device__ __forceinline__ void* ga_malloc(ga_dev_heap h, size_t n) {
    uint64_t off = ga::ga_malloc_off(h.desc, (uint64_t)n);
    return off == ga::kNull ? nullptr : (void*)(h.base + off);
}

__device__ __forceinline__ void ga_free(ga_dev_heap h, void* p) {
    ga::ga_free_off(h.desc, p ? (uint64_t)((char*)p - h.base) : ga::kNull);
}

/* Block- and cluster-collective calls (the paper's collective synchronization
 * primitives at thread-block scope, Sec. 4.2.2; cluster scope
 * through distributed shared memory is the B200 extension).
 *
 * EVERY thread of the CTA (ga_*_block) or of the thread-block cluster
 * (ga_*_cluster) must make the same sequence of calls, like __syncthreads();
 * threads with nothing to do pass n == 0 / p == NULL.  Each call contains one
 * (free) or two (malloc) barriers of that scope.  Call ga_block_begin /
 * ga_cluster_begin once per kernel, by every thread, before the first call.
 * A block or cluster call serves at most 2048 threads.  Per class, ONE thread
 * performs the semaphore operation for the whole collective's demand, and the
 * released units of a collective free reach the semaphores as one signal per
 * class.  Sizes above 64 KiB (TBuddy) take the warp path inside the call.
 * The static shared state (~170 B per CTA) is only allocated in kernels that
 * use these calls.  Same results and failure rules as ga_malloc/ga_free. */
__device__ __forceinline__ void ga_block_begin(ga_dev_heap h) { ga::coll_begin<false>(h.desc); }
__device__ __forceinline__ void* ga_malloc_block(ga_dev_heap h, size_t n) {
    uint64_t off = ga::malloc_coll_off<false>(h.desc, (uint64_t)n);
    return off == ga::kNull ? nullptr : (void*)(h.base + off);
}
__device__ __forceinline__ void ga_free_block(ga_dev_heap h, void* p) {
    ga::free_coll_off<false>(h.desc, p ? (uint64_t)((char*)p - h.base) : ga::kNull);
}
__device__ __forceinline__ void ga_cluster_begin(ga_dev_heap h) { ga::coll_begin<true>(h.desc); }
__device__ __forceinline__ void* ga_malloc_cluster(ga_dev_heap h, size_t n) {
    uint64_t off = ga::malloc_coll_off<true>(h.desc, (uint64_t)n);
    return off == ga::kNull ? nullptr : (void*)(h.base + off);
}
__device__ __forceinline__ void ga_free_cluster(ga_dev_heap h, void* p) {
    ga::free_coll_off<true>(h.desc, p ? (uint64_t)((char*)p - h.base) : ga::kNull);
}

/* Bulk-semaphore primitives (Alg. 1 / Alg. 2), exported for the
 * semaphore microbenchmark.  A ga_bsem word packs (C, D = E - R) (R-6). */
typedef unsigned long long ga_bsem;
#define GA_ACQUIRED 0
#define GA_GROW (-1)
__device__ __forceinline__ int ga_bsem_wait(ga_bsem* s, unsigned n, unsigned b) {
    return ga::bsem_wait((uint64_t*)s, n, b, ga::NoSpin());
}
__device__ __forceinline__ void ga_bsem_signal(ga_bsem* s, unsigned n, unsigned b) {
    ga::bsem_signal((uint64_t*)s, n, b);
}
__device__ __forceinline__ bool ga_bsem_trywait(ga_bsem* s, unsigned n) {
    return ga::bsem_trywait((uint64_t*)s, n);
}

#endif /* GA_DEVICE_CUH_ */
