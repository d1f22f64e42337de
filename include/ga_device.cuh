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
 *   come from one-page bins (UAlloc), larger sizes from TBuddy
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
