/*
 * ga.h -- host C ABI of the B200-native throughput-oriented device allocator.
 *
 * Method: Gelado & Garland, "Throughput-Oriented GPU Memory Allocation",
 * PPoPP'19 (PAPER.md; cited as P:Lnnn).  Device threads call ga_malloc/ga_free
 * (include/ga_device.cuh), the standard malloc/free interface of P:L356-360 and
 * P:L810-814.  The host reserves the pool once, the role cudaMalloc plays in
 * the paper.  Everything here is extern "C": plain pointers and
 * sizes, no C++ or torch types.  Host calls never throw; they return ga_status.
 *
 * Threading: host calls are not thread-safe per handle.  Streams: every call
 * that takes a stream enqueues on it; kernels that use a heap must be ordered
 * after ga_heap_create / ga_heap_reset on their stream.
 */
#ifndef GA_H_
#define GA_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    GA_OK = 0,
    GA_EINVAL = 1,   /* bad argument (null handle, size below one chunk, misaligned buffer) */
    GA_ENOMEM = 2,   /* cudaMalloc of the pool or metadata failed                           */
    GA_ECUDA = 3,    /* a CUDA runtime call or kernel launch failed                         */
    GA_EBUSY = 4     /* reserved                                                            */
} ga_status;

typedef struct CUstream_st* ga_stream_t;     /* == cudaStream_t; NULL = legacy default stream */
typedef struct ga_heap_s* ga_heap_t;          /* opaque; owned by the library                  */

/* Layout constants of this build (readings R-9..R-13). */
typedef struct {
    uint32_t page;          /* 4096: bin size and TBuddy order-0 block (R-9)  */
    uint32_t chunk_pages;   /* 64: bins per chunk (R-10)                 */
    uint32_t min_class;     /* 16: smallest class (R-13)                               */
    uint32_t bin_max;       /* 2048: largest bin class; >= 4096 goes to TBuddy (R-12)  */
    uint32_t n_classes;     /* 8 bin classes 16..2048                                  */
    uint32_t bitmap_bits;   /* 256: out-of-band bitmap bits per page                   */
    uint32_t n_span_classes;/* 5 span classes 4..64 KiB, one 64-page chunk per span
                               (DESIGN.md "Spans"); 0 in a GA_NSPAN=0 build          */
    uint32_t span_max;      /* 65536: largest span class; larger sizes go to TBuddy    */
} ga_layout_t;

/* Device-resident heap descriptor (lives at the start of the metadata
 * allocation; device code reads it through L1).  Owned by the library. */
typedef struct ga_desc {
    char* base;               /* pool base, 2 MiB aligned (R-31)                        */
    uint64_t pages;           /* usable pages (pool rounded down to whole chunks, R-30) */
    uint64_t nchunks;
    uint32_t L;               /* tree height: 2^L >= pages                              */
    uint32_t n_arenas;        /* one arena per SM                        */
    uint32_t chunk_words;     /* u64 words of a per-arena chunk bitmap                  */
    uint32_t flags;
    uint64_t* bits;           /* [pages][4] slot bitmaps, all ones when not a live bin   */
    uint32_t* kind;           /* [pages] page kind (R-18)                               */
    uint64_t* chunk_used;     /* [nchunks] used pages; all ones when not owned          */
    uint32_t* chunk_owner;    /* [nchunks] arena + 1, 0 = in the tree                   */
    uint64_t* chunk_nonfull;  /* [nchunks][13] per class: bins / the span with a free slot */
    uint64_t* chunk_cand;     /* [nchunks] bins that went empty (reclaim candidates)    */
    uint64_t* sem;            /* [n_arenas][13] class bulk semaphores (8 bin + 5 span classes), 32 B apart */
    uint64_t* psem;           /* [n_arenas] page bulk semaphores, 32 B apart            */
    uint32_t* hint;           /* [n_arenas][13] current bin / span head page per class  */
    uint64_t* ahb;            /* [n_arenas][2+13] chunk summaries (3-level bitsets): chunks
                                 with free pages, with reclaim candidates, with non-full
                                 bins (spans) of class c (c = 0..12)                    */
    uint64_t* avail;          /* TBuddy availability bitmaps, all levels (3-level each)  */
    uint64_t* tsem;           /* [L+1] per-order bulk semaphores, 32 B apart            */
    uint64_t* stats;          /* device counters, see ga_stats_t                        */
    uint32_t ahb_words;       /* u64 words of one chunk summary                          */
    uint32_t pad0;
    uint64_t lvl_off[48];     /* word offset of level n in avail                        */
    uint32_t lvl_words[48];   /* u64 words of level n's availability bits               */
    uint32_t* lvl_hint;       /* [48] last level-n word a claim succeeded in            */
    uint64_t* dbg;            /* host-mapped diagnostic records (ga_debug_attach), or 0  */
    uint64_t* actr;           /* [n_arenas][8] per-arena call counters: [0] mallocs, [1] frees
                                 (warp-aggregated; summed by ga_stats)                  */
} ga_desc;

/* Plain-old-data handle passed BY VALUE to kernels that call ga_malloc /
 * ga_free (16 bytes: cheap to pass, no per-thread copy of the descriptor). */
typedef struct {
    const ga_desc* desc;      /* device pointer to the descriptor                      */
    char* base;               /* pool base (== desc->base)                             */
} ga_dev_heap;

/* Device counters (failures are the paper's fragmentation
 * proxy).  Counted on the device by the allocator itself:
 * n_malloc / n_free per warp call into per-arena words, reserved pages on every
 * TBuddy allocation / free, the peak with an atomicMax on the growth side. */
typedef struct {
    uint64_t heap_bytes;          /* usable pool bytes                                     */
    uint64_t metadata_bytes;      /* separate metadata allocation (R-29)                   */
    uint64_t reserved_bytes;      /* pages held outside the free tree x PAGE (device counter) */
    uint64_t peak_reserved_bytes; /* max of reserved_bytes since create/reset (device atomicMax
                                     on every allocation from the tree)                    */
    uint64_t n_malloc;            /* ga_malloc calls, NULL returns and n == 0 included (R-15, R-17) */
    uint64_t n_free;              /* ga_free calls with p != NULL                          */
    uint64_t n_bin_grow;          /* new bins made (class GROW)                            */
    uint64_t n_chunk_grow;        /* chunks taken from TBuddy                               */
    uint64_t n_bin_reclaim;       /* empty bins returned to their chunk                    */
    uint64_t n_chunk_reclaim;     /* empty chunks returned to TBuddy                       */
    uint64_t n_fallback;          /* group waits degraded to per-lane (R-27)               */
    uint64_t n_fail;              /* mallocs that returned NULL after every fallback (n > 0) */
    uint64_t n_pending_reclaim;   /* candidate bins not yet reclaimed                      */
    uint64_t n_repair_nonfull;    /* safety net: non-full bits re-published (expected 0)   */
    uint64_t n_repair_summary;    /* safety net: chunk summary bits re-published (expected 0) */
    uint64_t n_waiter_reclaim;    /* of n_bin_reclaim: bins reclaimed by threads blocked in an
                                     arena semaphore wait (the delegation of P:L1206-1244)  */
    uint32_t n_arenas;
    uint32_t pad;
} ga_stats_t;

/* Create a heap on `device`.  buf == NULL: the library allocates the pool
 * (cudaMalloc, 2 MiB aligned); else `buf` (device pointer, 2 MiB aligned) is
 * borrowed and must outlive the heap.  `bytes` is rounded down to whole
 * 256 KiB chunks (R-30); fewer than one chunk -> GA_EINVAL.  Metadata is a
 * separate device allocation (R-29).  Initialisation is enqueued on `stream`.
 * flags: 0.  On success *out receives the handle. */
ga_status ga_heap_create(int device, ga_stream_t stream, void* buf, size_t bytes,
                         uint32_t flags, ga_heap_t* out);
/* Synchronises the device, frees metadata and an owned pool. */
ga_status ga_heap_destroy(ga_heap_t h);
/* Return the heap to empty (asynchronous on `stream`); invalidates every pointer. */
ga_status ga_heap_reset(ga_heap_t h, ga_stream_t stream);
/* Counters (stream-ordered D2H copies on `stream`, then a sync of `stream`). */
ga_status ga_stats(ga_heap_t h, ga_stream_t stream, ga_stats_t* out);
/* The POD view to pass to kernels. */
ga_status ga_heap_device(ga_heap_t h, ga_dev_heap* out);
/* Usable bytes of the pool and its base. */
ga_status ga_heap_info(ga_heap_t h, uint64_t* heap_bytes, void** base, uint64_t* metadata_bytes);
ga_status ga_layout(ga_layout_t* out);

/* Test hooks (exported, not on the perf path). */
/* Drain deferred reclamation: every empty bin returns to its chunk,
 * every empty chunk to TBuddy.  Must not overlap kernels using the heap. */
ga_status ga_heap_quiesce(ga_heap_t h, ga_stream_t stream);
/* Canonical snapshot (format below) into host memory; *used = bytes needed.
 * Stream-synchronous.  If cap < *used nothing is written and GA_EINVAL returned. */
ga_status ga_heap_snapshot(ga_heap_t h, ga_stream_t stream, void* host, size_t cap, size_t* used);
/* Pages held outside the free tree, computed from the tree bitmaps (device
 * reduction, stream-synchronous). */
ga_status ga_reserved_pages(ga_heap_t h, ga_stream_t stream, uint64_t* out);

const char* ga_status_str(ga_status s);

/*
 * Canonical snapshot (logical, little endian; the oracle writes the same format
 * independently, oracle/ga_oracle.c ora_snapshot):
 *   u64 magic "GASNAP01"; u64 heap_bytes; u64 pages; u64 page | (L+1) << 32;
 *   u64 min_class | n_classes << 32 | 5 << 40 (class entries above the bins) | chunk_pages << 48;
 *   u8 kind[pages]: 0x00 free page inside an Available tree node (not its head),
 *                   0x40|n head of an Available node of order n, 0x80|n head of an
 *                   allocated user block of order n, 0x01 tail page of such a block,
 *                   0x02 free page of an arena chunk, 0x10|c bin of class c,
 *                   0x20|s first page of a span of span class s (blocks of page << s),
 *                   0x04 any other page of a span;
 *   for each bin or span head page in ascending order: its slots bits (a bin of
 *                   class c: page / (min_class << c); a span of class s:
 *                   chunk_pages >> s), LSB first, padded to bytes;
 *   for each level n = 0..L: 2^(L-n) availability bits, LSB first, padded to bytes;
 *   for each size class 16 B .. 64 KiB (the 8 bin classes, then 5 entries for
 *                   4 .. 64 KiB whatever the build routes to spans): i64 sum over
 *                   arenas of C, i64 max over arenas of |E-R| (zeros for sizes the
 *                   build -- or the oracle, which routes them to TBuddy as the
 *                   paper does -- does not serve from spans);
 *   i64 sum of page-semaphore C, i64 max |E-R|;
 *   for each order n = 0..L: i64 C, i64 E-R;
 *   u64 pending reclamation candidates.
 */

#ifdef __cplusplus
}
#endif
#endif /* GA_H_ */
