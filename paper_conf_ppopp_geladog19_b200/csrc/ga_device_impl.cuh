// ga_device_impl.cuh -- device implementation of the B200-native allocator.
//
// Method: Gelado & Garland, "Throughput-Oriented GPU Memory Allocation", PPoPP'19
// (PAPER.md, cited P:Lnnn).  Written for sm_100a from the paper's description;
// the paper's Volta design is prior art.
//
// Sections:
//   1. constants, PTX helpers
//   2. bulk semaphore (Alg. 1 / Alg. 2) packed as (C, D = E - R) in
//      one 64-bit word (reading R-6): a load-gated fetch-add fast path, the exact
//      CAS form for arena semaphores, an optimistic form for TBuddy orders
//   3. three-level summary bitsets (scattered search starts)
//   4. TBuddy over per-level availability bitmaps; lock-free merge
//      via a CAS on the word holding both siblings (reading R-21)
//   5. UAlloc: per-SM arenas, 64-page chunks, one-page bins with
//      out-of-band 256-bit slot bitmaps, per-(arena, class) chunk summaries
//   6. deferred reclamation delegated to waiting threads
//   7. warp-collective front end: __match_any_sync groups a warp's lanes by size
//      class; one semaphore operation serves the group; the group claims its
//      slots collectively, one atomicOr per bitmap word
//
// Invariants:
//   * bits[p][*] == all ones whenever page p is not a live bin, so a stale
//     claimer's atomicOr can never take a slot in a recycled page;
//   * kind[p] is written only while bits[p] is all ones; claimers re-validate it;
//   * chunk_used[k] == all ones whenever chunk k is not owned by an arena;
//   * at quiescence: class semaphore C == free slots of the arena's class bins,
//     page semaphore C == free pages of the arena's chunks, tree C[n] ==
//     available nodes of order n, every D == 0.
#pragma once
#include <cstdint>
#include <cooperative_groups.h>
#include "ga.h"

namespace ga {
// (functions are static: this header is compiled into every including TU)

// ---------------------------------------------------------------------------
// 1. constants and PTX helpers
// ---------------------------------------------------------------------------
constexpr int kPageShift = 12;                  // 4 KiB pages / bins (R-9)
constexpr uint64_t kPage = 1ull << kPageShift;
constexpr int kChunkShift = 6;                  // 64 pages per chunk (R-10)
constexpr uint32_t kChunkPages = 1u << kChunkShift;
constexpr int kChunkOrder = kChunkShift;        // a chunk is a TBuddy block of order 6
// Size classes with per-arena semaphores.  Bins serve 16 B ..
// 2 KiB out of one 4 KiB page each.  Spans (a B200 departure, DESIGN.md
// "Spans") serve 4 KiB .. 64 KiB out of one 64-page chunk each, with the same
// semaphore / bitmap / collective machinery, so mid sizes stop funnelling
// through TBuddy's global per-order semaphores; TBuddy keeps chunk supply and
// every size above the span range.  GA_NSPAN=0 restores the paper's routing.
#ifndef GA_NSPAN
#define GA_NSPAN 5
#endif
constexpr int kNbin = 8;                        // bin classes 16 .. 2048 B
constexpr int kNspan = GA_NSPAN;                // span classes 4 KiB .. 2^(11+kNspan) B
static_assert(kNspan >= 0 && kNspan <= 5, "span classes: 4 KiB .. 64 KiB");
constexpr int kNcls = kNbin + kNspan;           // classes 0 .. kNcls-1
// Span arenas are shared by GA_SPAN_SHARE consecutive SMs: fewer, larger pools
// smooth the per-pool high-water marks that set reserved memory (DESIGN.md
// "Spans").  GA_SPAN_EAGER=1: a free that empties a span returns it to the
// tree at once when the class keeps a span's worth of free slots elsewhere.
#ifndef GA_SPAN_SHARE
#define GA_SPAN_SHARE 2
#endif
#ifndef GA_SPAN_EAGER
#define GA_SPAN_EAGER 0
#endif
constexpr int kMinShift = 4;                    // 16 B minimum class (R-13)
constexpr int kBinWords = 4;                    // 256-bit slot bitmap per page
constexpr uint64_t kNull = ~0ull;
constexpr uint32_t kKindBin = 0x40000000u;      // | arena << 8 | class
constexpr uint32_t kKindTree = 0x80000000u;     // | order
constexpr int kSemStride = 4;                   // u64 words between semaphores (32 B)
constexpr int kMaxLevels = 48;
// tuning switches; defaults are the measured best
#ifndef GA_LVL_HINT
#define GA_LVL_HINT 0            // 1: claim from the last successful level word first
#endif
#ifndef GA_TREE_SPIN_CAP
#define GA_TREE_SPIN_CAP 256     // max __nanosleep backoff (ns) of a blocked TBuddy wait
#endif
#ifndef GA_SPAN_CLEAR_CHECK
#define GA_SPAN_CLEAR_CHECK 1    // 1: a failed span claim clears the summary bit only when it is stale
#endif
#ifndef GA_EAGER_AT
#define GA_EAGER_AT 9            // empty spans go back to TBuddy at once above GA_EAGER_AT/10 of the heap reserved (10: never)
#endif
#ifndef GA_DEFER_RECHECK
#define GA_DEFER_RECHECK 0       // 1: the lockstep claim validates its slots' page kinds once after the loop, not per iteration
#endif
#ifndef GA_LAZY_CLEAR
#define GA_LAZY_CLEAR 0          // 1: a claim that fills a page leaves its non-full bit; the next claimer to find it full clears it
#endif
#ifndef GA_INL_CLAIM
#define GA_INL_CLAIM 1           // 1: inline the hint lookup and page claim into the collective claim
#endif
#ifndef GA_CLAIM_LOCALMASK
#define GA_CLAIM_LOCALMASK 0     // 1: a group retries the other non-full pages of its chunk before searching again
#endif
#ifndef GA_PREFETCH
#define GA_PREFETCH 1            // 1: the malloc leader loads its block's hinted chunk beside the semaphore fetch-add
#endif
#ifndef GA_COUNT_ITERS
#define GA_COUNT_ITERS 0         // diagnostic: count collective-claim calls / iterations in the repair stats
#endif
#ifndef GA_HINT_LDCA
#define GA_HINT_LDCA 0           // 1: read the per-(arena, class) hint through L1
#endif
#if GA_INL_CLAIM
#define GA_CLAIM_FN __forceinline__
#else
#define GA_CLAIM_FN __noinline__
#endif
constexpr uint32_t kReclaimKeep = 64;           // free slots a delegated reclaim leaves per class

enum { kStatBinGrow = 0, kStatChunkGrow, kStatBinReclaim, kStatChunkReclaim, kStatFallback,
       kStatFail, kStatRepairNonfull, kStatRepairSummary, kNumStats };
// device words of the reserved-page counter and its peak (own 32 B sectors of
// the stats block), and the per-arena call counters (ga_stats_t)
constexpr int kStatReserved = 8, kStatPeakReserved = 12, kStatWords = 16;
constexpr int kStatWaiterReclaim = 9;           // bins reclaimed by threads blocked in a wait
constexpr int kStatDrainLock = 10, kStatDrainGen = 11;   // reclaim_all: one drain at a time, and its generation
constexpr int kActrStride = 8;                  // u64 words per arena: [0] mallocs, [1] frees

static __device__ __forceinline__ uint32_t lane_id() { uint32_t r; asm volatile("mov.u32 %0, %%laneid;" : "=r"(r)); return r; }
static __device__ __forceinline__ uint32_t lanemask_lt() { uint32_t r; asm volatile("mov.u32 %0, %%lanemask_lt;" : "=r"(r)); return r; }
static __device__ __forceinline__ uint32_t smid() { uint32_t r; asm volatile("mov.u32 %0, %%smid;" : "=r"(r)); return r; }
// Warp masks for the *_sync intrinsics (R-42).  Lanes that call the
// allocator from divergent code enter in separate groups, each with its own
// __activemask(), and the hardware can merge the groups again at a later
// convergence barrier (BSYNC).  ptxas treats a vote result (__activemask,
// __ballot_sync) as warp-uniform: it reads such a mask through one uniform
// register (R2UR) and skips the synchronisation when "every lane of the mask is
// active" -- with merged groups holding different masks, some lanes then skip
// a _sync the others wait in (a hang found by cuda-gdb: a group's leader left
// alone at a shuffle its lanes had passed).  A __match_any_sync result is not
// assumed uniform: ptxas checks it (REDUX.OR + R2UR P) and takes the per-lane
// collective path (WARPSYNC.COLLECTIVE) when co-active lanes differ.  So every
// mask the allocator passes to a _sync intrinsic is a match result or an AND
// of match results, taken right after __activemask() (no barrier between), and
// __syncwarp(mask) is not used at all.
static __device__ __forceinline__ unsigned active_lanes() { return __match_any_sync(__activemask(), 0u); }
// the lanes of mask m whose predicate equals this lane's (a ballot, as a match)
static __device__ __forceinline__ unsigned lanes_where(unsigned m, bool pred) { return __match_any_sync(m, (unsigned)pred); }
// Every lane of `grp` has performed its prior writes at gpu scope (fence) and
// reached this point (ballot) before any lane of grp continues: a leader's
// release signal that follows publishes every lane's writes.
static __device__ __forceinline__ void warp_release(unsigned grp) {
    asm volatile("fence.acq_rel.gpu;" ::: "memory");
    (void)__ballot_sync(grp, 1);
}

static __device__ __forceinline__ uint64_t ld_rlx(const uint64_t* p) {
    uint64_t v; asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory"); return v;
}
static __device__ __forceinline__ uint32_t ld_rlx32(const uint32_t* p) {
    uint32_t v; asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory"); return v;
}
static __device__ __forceinline__ void st_rlx32(uint32_t* p, uint32_t v) {
    asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" :: "l"(p), "r"(v) : "memory");
}
// one 256-bit load of a page's slot bitmap (LDG.E.ENL2.256 on sm_100a)
static __device__ __forceinline__ void ld_bitmap(const uint64_t* p, uint64_t w[4]) {
    asm volatile("ld.relaxed.gpu.global.v4.u64 {%0,%1,%2,%3}, [%4];"
                 : "=l"(w[0]), "=l"(w[1]), "=l"(w[2]), "=l"(w[3]) : "l"(p) : "memory");
}
static __device__ __forceinline__ uint64_t a_or(uint64_t* p, uint64_t v) { return atomicOr((unsigned long long*)p, (unsigned long long)v); }
static __device__ __forceinline__ uint64_t a_and(uint64_t* p, uint64_t v) { return atomicAnd((unsigned long long*)p, (unsigned long long)v); }
static __device__ __forceinline__ uint64_t a_cas(uint64_t* p, uint64_t c, uint64_t v) { return atomicCAS((unsigned long long*)p, (unsigned long long)c, (unsigned long long)v); }
static __device__ __forceinline__ uint64_t a_add(uint64_t* p, uint64_t v) { return atomicAdd((unsigned long long*)p, (unsigned long long)v); }
static __device__ __forceinline__ uint64_t a_exch(uint64_t* p, uint64_t v) { return atomicExch((unsigned long long*)p, (unsigned long long)v); }
static __device__ __forceinline__ void red_add_release(uint64_t* p, uint64_t v) {
    asm volatile("red.release.gpu.global.add.u64 [%0], %1;" :: "l"(p), "l"(v) : "memory");
}
// fence(): release/acquire ordering of our own accesses (publication paths);
// fence_sc(): store -> load ordering for the clear-then-recheck (Dekker) patterns
static __device__ __forceinline__ void fence() { asm volatile("fence.acq_rel.gpu;" ::: "memory"); }
static __device__ __forceinline__ void fence_sc() { __threadfence(); }
// The re-check read of a clear-then-recheck (Dekker) pattern.  GA_RECHECK_RMW=1
// reads the word with an atomicOr(0): RMWs on one address are totally ordered at
// L2, and the read is issued only after the clearing RMW returned, so no SC fence
// is needed; 0 uses fence.sc + a relaxed load.
#ifndef GA_RECHECK_RMW
#define GA_RECHECK_RMW 0
#endif
static __device__ __forceinline__ uint64_t recheck_read(uint64_t* p) {
#if GA_RECHECK_RMW
    return atomicOr((unsigned long long*)p, 0ull);
#else
    fence_sc();
    return ld_rlx(p);
#endif
}
static __device__ __forceinline__ void stat_add(const ga_desc* h, int i, uint64_t v) { a_add(&h->stats[i], v); }
// pages leaving (d > 0) or returning to (d < 0) the free tree; the peak is an
// atomicMax on the growth side only (SURVEY 8(a) a10, 8(d) "peak_reserved_X")
static __device__ __noinline__ void reserve_add(const ga_desc* h, int64_t d) {
    if (d <= 0) {
        asm volatile("red.relaxed.gpu.global.add.u64 [%0], %1;" :: "l"(&h->stats[kStatReserved]), "l"((uint64_t)d) : "memory");
        return;
    }
    const uint64_t v = a_add(&h->stats[kStatReserved], (uint64_t)d) + (uint64_t)d;
    if (v > ld_rlx(&h->stats[kStatPeakReserved])) atomicMax((unsigned long long*)&h->stats[kStatPeakReserved], (unsigned long long)v);
}

// GA_DEBUG builds: a spin loop that runs ~2^20 times records (site, ids, a, b)
// into host-mapped memory, readable while a kernel hangs (tools/hang_probe.py)
#ifndef GA_DEBUG
#define GA_DEBUG 0
#endif
// host-mapped records of GA_DEBUG builds' spin loops (ga_debug_attach sets
// ga_bench.cu's copy; those loops have no heap descriptor at hand).  The
// safety-net dump in nfc_repair reads the descriptor's dbg field instead, so it
// works from every translation unit.
static __device__ uint64_t* g_ga_dbg;
#if GA_DEBUG
#define SPIN_NOTE(cnt, site, a, b) spin_note((cnt), (site), (uint64_t)(a), (uint64_t)(b))
#define GA_DBG_CNT uint32_t dbg_cnt = 0
static __device__ __noinline__ void spin_note(uint32_t& cnt, int site, uint64_t a, uint64_t b) {
    if ((++cnt & ((1u << 18) - 1)) != 0 || !g_ga_dbg) return;
    uint64_t* dbg = g_ga_dbg;
    unsigned long long i = atomicAdd((unsigned long long*)&dbg[0], 1ull);
    if (i >= 255) return;
    uint32_t w; asm volatile("mov.u32 %0, %%warpid;" : "=r"(w));
    uint32_t sm; asm volatile("mov.u32 %0, %%smid;" : "=r"(sm));
    uint32_t ln; asm volatile("mov.u32 %0, %%laneid;" : "=r"(ln));
    volatile uint64_t* r = (volatile uint64_t*)&dbg[8 + i * 4];
    r[0] = (uint64_t)site; r[1] = ((uint64_t)sm << 32) | (w << 8) | ln; r[2] = a; r[3] = b;
    __threadfence_system();
}
#else
#define SPIN_NOTE(cnt, site, a, b) ((void)0)
#define GA_DBG_CNT ((void)0)
#endif

static __device__ __forceinline__ uint32_t hash32(uint32_t x) {
    x ^= x >> 16; x *= 0x7feb352dU; x ^= x >> 15; x *= 0x846ca68bU; x ^= x >> 16; return x;
}
// a per-warp scatter seed (ScatterAlloc-style hashing of the search start)
static __device__ __forceinline__ uint32_t scatter_seed() {
    uint32_t w; asm volatile("mov.u32 %0, %%warpid;" : "=r"(w));
    return hash32((smid() << 8) ^ w ^ (uint32_t)clock());
}
// rotate right
static __device__ __forceinline__ uint64_t rotr(uint64_t x, uint32_t r) { r &= 63; return r ? (x >> r) | (x << (64 - r)) : x; }
// index of the first set bit of x at or after position r (cyclic); x != 0
static __device__ __forceinline__ uint32_t first_from(uint64_t x, uint32_t r) { return (uint32_t)((__ffsll((long long)rotr(x, r)) - 1 + r) & 63); }
// mask of the lowest k set bits of x
static __device__ __forceinline__ uint32_t nth_set(uint64_t x, uint32_t n);
static __device__ __forceinline__ uint64_t lowest_bits(uint64_t x, int k) {
    if (k <= 0) return 0;
    if (__popcll(x) <= k) return x;
    const uint32_t pos = nth_set(x, (uint32_t)k - 1);       // the k-th set bit: keep bits <= pos
    return x & (pos == 63 ? ~0ull : ((2ull << pos) - 1));
}
// position of the n-th (0-based) set bit of x
// (branch-free popc binary search; __fns is emulated with a loop on sm_100a)
static __device__ __forceinline__ uint32_t nth_set(uint64_t x, uint32_t n) {
    uint32_t pos = 0, c;
    c = __popc((uint32_t)x);          if (n >= c) { n -= c; x >>= 32; pos += 32; }
    uint32_t v = (uint32_t)x;
    c = __popc(v & 0xFFFFu);          if (n >= c) { n -= c; v >>= 16; pos += 16; }
    c = __popc(v & 0xFFu);            if (n >= c) { n -= c; v >>= 8; pos += 8; }
    c = __popc(v & 0xFu);             if (n >= c) { n -= c; v >>= 4; pos += 4; }
    c = __popc(v & 0x3u);             if (n >= c) { n -= c; v >>= 2; pos += 2; }
    c = v & 1u;                       if (n >= c) { pos += 1; }
    return pos;
}

// OR of v over my group g, for groups that partition the uniform mask m, with
// every collective on m.  A collective whose mask differs between the lanes
// executing it (e.g. __reduce_or_sync(g)) compiles to a divergent path
// (BRA.DIV ... ENDCOLLECTIVE) that runs the groups one after another: on the
// mixed trace the free path ran with 1 active lane per instruction.  Here the
// trip count is the largest group's size, uniform over m.
static __device__ __forceinline__ uint64_t group_or(unsigned m, unsigned g, uint64_t v) {
    if (__all_sync(m, g == m))                                // one group (warp-uniform calls)
        return ((uint64_t)__reduce_or_sync(m, (uint32_t)(v >> 32)) << 32) | __reduce_or_sync(m, (uint32_t)v);
    const uint32_t n = __reduce_max_sync(m, (uint32_t)__popc(g));
    const uint32_t mine = __popc(g);
    uint64_t acc = 0;
    for (uint32_t j = 0; j < n; j++) {
        const int src = j < mine ? (int)nth_set((uint64_t)g, j) : (int)lane_id();
        const uint64_t x = __shfl_sync(m, v, src);
        if (j < mine) acc |= x;
    }
    return acc;
}
static __device__ __forceinline__ bool is_span(int c) { return c >= kNbin; }
static __device__ __forceinline__ uint32_t slots_of(int c) { return c < kNbin ? 256u >> c : kChunkPages >> (c - kNbin); }
// first page of the bin / span holding page p (its slot bitmap and kind live there)
// log2 of the lanes one page (span) serves in a collective claim: min(slots, 64)
static __device__ __forceinline__ uint32_t per_page_shift(int c) {
    const int s = c < kNbin ? 8 - c : 14 - c;                   // log2 slots_of(c)
    return s < 6 ? (uint32_t)s : 6u;
}
static __device__ __forceinline__ uint64_t bin_head(uint64_t p, int c) { return is_span(c) ? p & ~(uint64_t)(kChunkPages - 1) : p; }
static __device__ __forceinline__ int words_of(int c) { return c == 0 ? 4 : c == 1 ? 2 : 1; }
static __device__ __forceinline__ uint64_t valid_mask(int c, int w) {
    int s = (int)slots_of(c) - 64 * w;
    return s >= 64 ? ~0ull : s <= 0 ? 0ull : ((1ull << s) - 1);
}
static __device__ __forceinline__ uint32_t arena_of(const ga_desc* h) { return smid() % h->n_arenas; }
// SMs sharing one arena for class c (reading R-41).  An arena holds at least
// one 64-page chunk per class it serves, so per-SM arenas reserve 148 chunks
// (37 MiB) for a class whatever its live set: at full occupancy a 16 B class
// holds 4.6 MiB live and the reserve dominated fragmentation (7.8x the
// oracle's on d3).  The tiny classes share arenas so an arena's live set of
// the class at full occupancy (2,048 threads per SM) is a little UNDER a whole
// number of chunks: 7 SMs x 2,048 x 16 B = 56 pages, x 32 B = 112, x 64 B =
// 224 (7/8 of 1, 2, 4 chunks).  Exactly one chunk's worth (8 SMs at 16 B, 4 at
// 32 B) spilled into a second chunk whenever a few extra bins were grown
// (d3 fragmentation 1.46x the oracle's at 16 / 32 B).  Spans share
// GA_SPAN_SHARE SMs.
#ifndef GA_SMALL_SHARE
#define GA_SMALL_SHARE 1
#endif
static __device__ __forceinline__ uint32_t class_share(int c) {
    if (c >= kNbin) return GA_SPAN_SHARE;
#if GA_SMALL_SHARE
    return c <= 2 ? 7 : c == 3 ? 2 : 1;                           // 16 / 32 / 64 B: 7, 128 B: 2
#else
    return 1;
#endif
}
static __device__ __forceinline__ uint64_t* sem_ptr(const ga_desc* h, uint32_t A, int c) { return h->sem + ((uint64_t)A * kNcls + c) * kSemStride; }
static __device__ __forceinline__ uint64_t* psem_ptr(const ga_desc* h, uint32_t A) { return h->psem + (uint64_t)A * kSemStride; }
static __device__ __forceinline__ uint64_t* tsem_ptr(const ga_desc* h, int n) { return h->tsem + (uint64_t)n * kSemStride; }
static __device__ __forceinline__ uint64_t* page_bits(const ga_desc* h, uint64_t p) { return h->bits + p * kBinWords; }

// ---------------------------------------------------------------------------
// 2. bulk semaphore: word = (C:int32 << 32) | (D + 2^31), D = E - R (R-6)
// ---------------------------------------------------------------------------
enum { kAcquired = 0, kGrow = -1, kBlocked = 1 };
static __device__ __forceinline__ int32_t sem_C(uint64_t w) { return (int32_t)(uint32_t)(w >> 32); }
static __device__ __forceinline__ int32_t sem_D(uint64_t w) { return (int32_t)((uint32_t)w - 0x80000000u); }

// Alg. 2 (R-3): C += N, E -= B.  Release: everything the caller
// published (bins, bitmap bits) is visible before the units are.
static __device__ __forceinline__ void bsem_signal(uint64_t* s, uint32_t N, uint32_t B) {
    red_add_release(s, ((uint64_t)N << 32) - (uint64_t)B);
}
// signal after atomics whose returned values were already consumed (so they
// have performed at L2): no release fence needed
static __device__ __forceinline__ void bsem_signal_after_rmw(uint64_t* s, uint32_t N) {
    asm volatile("red.relaxed.gpu.global.add.u64 [%0], %1;" :: "l"(s), "l"((uint64_t)N << 32) : "memory");
}

// Conservative in-flight encoding (R-35; model-checked by
// oracle/bsem.py explore_gpu, tests/test_oracle_bsem.py).  A fetch-add that
// speculates moves units from C into D instead of removing them: (C -= N,
// D += N) keeps C + D.  While it is in flight the word therefore only shows
// LESS value (C) and MORE cover (C + D) than the state with every decided
// operation applied, so no other thread can take units that are not there or
// decide GROW when that state would not.  Each speculation is settled by one
// more add: a repayment of D, or the reverse move.
static __device__ __forceinline__ uint64_t dCD(int32_t dc, int32_t dd) {
    return ((uint64_t)(int64_t)dc << 32) + (uint64_t)(int64_t)dd;
}
static __device__ __forceinline__ void red_rlx(uint64_t* s, uint64_t v) {
    asm volatile("red.relaxed.gpu.global.add.u64 [%0], %1;" :: "l"(s), "l"(v) : "memory");
}

// try-wait (R-7): C -= N iff C >= N (+ keep units stay behind).
// direct: no pre-load (callers that expect success, e.g. a merge whose buddy
// bit was just seen set).
static __device__ __forceinline__ bool bsem_trywait_direct(uint64_t* s, uint32_t N, uint32_t keep = 0) {
    uint64_t old = a_add(s, dCD(-(int32_t)N, (int32_t)N));
    if (sem_C(old) >= (int32_t)(N + keep)) { red_rlx(s, dCD(0, -(int32_t)N)); return true; }
    red_rlx(s, dCD((int32_t)N, -(int32_t)N));
    return false;
}
static __device__ __forceinline__ bool bsem_trywait(uint64_t* s, uint32_t N, uint32_t keep = 0) {
    if (sem_C(ld_rlx(s)) < (int32_t)(N + keep)) return false;
    return bsem_trywait_direct(s, N, keep);
}

// Alg. 1 as the CUDA path runs it: fetch-adds only, no CAS retry
// loop on hot words.  The first fetch-add (C -= N, D += B) is conservative for
// every outcome (see dCD); its pre-image decides in Alg. 1's order, and one
// more add settles it:
//   pre C + D < N   -> GROW:     (C += N, D -= N)       net E += B - N
//   pre C >= N      -> ACQUIRED: (D -= B)               net C -= N
//   otherwise       -> reserve:  (C += N, D -= N + B)   net R += N; spin while
//                      C < N and C + D >= 0 (R-2), running `spin()` -- the
//                      delegated work of Sec. 4.2.1 -- between polls; then
//                      R -= N and decide again.
// Returns kAcquired (0) or kGrow (-1): the caller must produce B units, keep N
// and signal(B - N, B - N), or signal(0, B - N) on failure.
// Model-checked as form "fa" (oracle/bsem.py explore_gpu): exact for unit
// demands, no deadlock, no over-grant (tests/test_oracle_bsem.py).
static __device__ __forceinline__ int bsem_decide(uint64_t* s, uint64_t old, uint32_t N, uint32_t B, uint64_t* w) {
    const int32_t C = sem_C(old), D = sem_D(old);
    if ((int64_t)C + D < (int64_t)N) { red_rlx(s, dCD((int32_t)N, -(int32_t)N)); return kGrow; }
    if (C >= (int32_t)N) { red_rlx(s, dCD(0, -(int32_t)B)); return kAcquired; }
    const uint64_t res = dCD((int32_t)N, -(int32_t)(N + B));
    *w = a_add(s, res) + res;
    return kBlocked;
}
template <uint32_t kCap, class Spin>
static __device__ __noinline__ int bsem_wait_slow(uint64_t* s, uint32_t N, uint32_t B, Spin spin, uint64_t w) {
    GA_DBG_CNT;
    for (;;) {
        uint32_t ns = 32;
        while (sem_C(w) < (int32_t)N && (int64_t)sem_C(w) + sem_D(w) >= 0) {                    // R-2
            spin();
            SPIN_NOTE(dbg_cnt, 1, (uint64_t)(uintptr_t)s, w);
            __nanosleep(ns);
            if (ns < kCap) ns <<= 1;
            w = ld_rlx(s);
        }
        red_rlx(s, (uint64_t)N);                                                             // R -= N
        const int r = bsem_decide(s, a_add(s, dCD(-(int32_t)N, (int32_t)B)), N, B, &w);
        if (r != kBlocked) return r;
    }
}
// kCap: the __nanosleep backoff cap of a blocked waiter (R-5; arena semaphores
// 2 us, TBuddy orders GA_TREE_SPIN_CAP)
template <uint32_t kCap = 2048, class Spin>
static __device__ __forceinline__ int bsem_wait(uint64_t* s, uint32_t N, uint32_t B, Spin spin) {
    uint64_t w = 0;
    const int r = bsem_decide(s, a_add(s, dCD(-(int32_t)N, (int32_t)B)), N, B, &w);
    return r != kBlocked ? r : bsem_wait_slow<kCap>(s, N, B, spin, w);
}
template <class Spin>
static __device__ __forceinline__ int bsem_wait_fast(uint64_t* s, uint32_t N, uint32_t B, Spin spin) {
    return bsem_wait<GA_TREE_SPIN_CAP>(s, N, B, spin);
}

// Alg. 1 as one CAS per decision on the packed word (the paper's form,
// P:L766-772) -- only the d2 microbenchmark's per-thread CAS variant uses it.
static __device__ __noinline__ int bsem_wait_cas(uint64_t* s, uint32_t N, uint32_t B) {
    uint64_t w = ld_rlx(s);
    for (;;) {
        int32_t C = sem_C(w), D = sem_D(w);
        uint64_t nw;
        int res;
        if ((int64_t)C + D < (int64_t)N) { nw = w + (uint64_t)(B - N); res = kGrow; }          // E += B - N
        else if (C >= (int32_t)N) { nw = w - ((uint64_t)N << 32); res = kAcquired; }        // C -= N
        else { nw = w - (uint64_t)N; res = kBlocked; }                                       // R += N
        uint64_t old = a_cas(s, w, nw);
        if (old != w) { w = old; continue; }
        if (res != kBlocked) return res;
        uint32_t ns = 64;
        do { __nanosleep(ns); if (ns < 2048) ns <<= 1; w = ld_rlx(s); }
        while (sem_C(w) < (int32_t)N && (int64_t)sem_C(w) + sem_D(w) >= 0);                   // R-2
        w = a_add(s, (uint64_t)N) + (uint64_t)N;                                             // R -= N
    }
}
struct NoSpin { __device__ void operator()() const {} };

// ---------------------------------------------------------------------------
// 3. hierarchical bitsets: level 0 holds the data bits, level k+1 has one bit per
// non-zero word of level k.  Summary bits may be transiently stale in either
// ---------------------------------------------------------------------------
// 3. three-level summary bitsets ("HB3").  Layout [w0 | w1 | w2]: w0 holds the
// bits, bit j of w1 says "w0 word j may be non-zero", bit j of w2 the same for
// w1.  Summary bits may be stale in either direction for a moment: finders
// skip zero words (false positive), and callers that hold semaphore units retry
// on a false negative (a setter is about to publish).  Used for the TBuddy
// availability levels and for the per-arena chunk summaries.
// ---------------------------------------------------------------------------
struct HB3 { uint64_t* w0; uint32_t n0; };
static __host__ __device__ __forceinline__ uint32_t hb3_n1(uint32_t n0) { return (n0 + 63) / 64; }
static __host__ __device__ __forceinline__ uint32_t hb3_n2(uint32_t n0) { return (hb3_n1(n0) + 63) / 64; }
static __host__ __device__ __forceinline__ uint32_t hb3_words(uint32_t n0) { return n0 + hb3_n1(n0) + hb3_n2(n0); }
static __device__ __forceinline__ uint64_t* hb3_w1(HB3 b) { return b.w0 + b.n0; }
static __device__ __forceinline__ uint64_t* hb3_w2(HB3 b) { return b.w0 + b.n0 + hb3_n1(b.n0); }

// w0 word j went from zero to non-zero: publish it in the summaries
static __device__ __forceinline__ void hb3_up_set(HB3 b, uint32_t j) {
    if (a_or(&hb3_w1(b)[j >> 6], 1ull << (j & 63)) == 0) a_or(&hb3_w2(b)[j >> 12], 1ull << ((j >> 6) & 63));
}
// set bit i of w0
static __device__ __forceinline__ void hb3_set(HB3 b, uint64_t i) {
    if (a_or(&b.w0[i >> 6], 1ull << (i & 63)) == 0) hb3_up_set(b, (uint32_t)(i >> 6));
}
// w0 word j was seen zero: clear its summary bit, then re-check (clear-then-recheck)
static __device__ __noinline__ void hb3_up_clear(HB3 b, uint32_t j) {
    uint64_t* w1 = hb3_w1(b);
    uint64_t bit = 1ull << (j & 63);
    uint64_t old = a_and(&w1[j >> 6], ~bit);
    if (recheck_read(&b.w0[j]) != 0) { if (a_or(&w1[j >> 6], bit) == 0) a_or(&hb3_w2(b)[j >> 12], 1ull << ((j >> 6) & 63)); return; }
    if ((old & ~bit) != 0) return;
    uint32_t j1 = j >> 6;
    uint64_t* w2 = hb3_w2(b);
    uint64_t bit2 = 1ull << (j1 & 63);
    a_and(&w2[j1 >> 6], ~bit2);
    if (recheck_read(&w1[j1]) != 0) a_or(&w2[j1 >> 6], bit2);
}
// Bit i of w0 summarises an outside data word (*data).  Clear the bit when the
// data says "empty", re-checking the data after the clear.
static __device__ __noinline__ void hb3_clear_summarised(HB3 b, uint64_t i, const uint64_t* data, uint64_t empty_value) {
    uint64_t bit = 1ull << (i & 63);
    uint64_t old = a_and(&b.w0[i >> 6], ~bit);
    if (recheck_read((uint64_t*)data) != empty_value) { if (a_or(&b.w0[i >> 6], bit) == 0) hb3_up_set(b, (uint32_t)(i >> 6)); return; }
    if (old == bit) hb3_up_clear(b, (uint32_t)(i >> 6));
}
// a w0 word that looks non-zero, searched from a scattered start; -1 if none
static __device__ __noinline__ int64_t hb3_find(HB3 b, uint32_t seed) {
    const uint32_t n1 = hb3_n1(b.n0), n2 = hb3_n2(b.n0);
    const uint64_t* w1 = hb3_w1(b);
    const uint64_t* w2 = hb3_w2(b);
    for (uint32_t t = 0; t < n2; t++) {
        uint32_t j2 = (seed + t) % n2;
        uint64_t x2 = ld_rlx(&w2[j2]);
        while (x2) {
            uint32_t b2 = first_from(x2, seed);
            x2 &= ~(1ull << b2);
            uint32_t j1 = j2 * 64 + b2;
            if (j1 >= n1) continue;
            uint64_t x1 = ld_rlx(&w1[j1]);
            while (x1) {
                uint32_t b1 = first_from(x1, seed >> 6);
                x1 &= ~(1ull << b1);
                uint32_t j0 = j1 * 64 + b1;
                if (j0 < b.n0 && ld_rlx(&b.w0[j0]) != 0) return (int64_t)j0;
            }
        }
    }
    return -1;
}
static __device__ __forceinline__ bool hb3_any(HB3 b) {
    const uint64_t* w2 = hb3_w2(b);
    for (uint32_t j = 0, n2 = hb3_n2(b.n0); j < n2; j++) if (ld_rlx(&w2[j])) return true;
    return false;
}

// per-arena chunk summaries: which chunks of arena A have free pages (FPC),
// reclaim candidates (CND), non-full bins of class c (NFC + c)
enum { kAhbFpc = 0, kAhbCnd = 1, kAhbNfc = 2, kAhbPerArena = 2 + kNcls };
static __device__ __forceinline__ HB3 arena_hb(const ga_desc* h, uint32_t A, int which) {
    HB3 b; b.n0 = h->chunk_words; b.w0 = h->ahb + ((uint64_t)A * kAhbPerArena + which) * h->ahb_words; return b;
}
static __device__ __forceinline__ HB3 level_hb(const ga_desc* h, int n) {
    HB3 b; b.n0 = h->lvl_words[n]; b.w0 = h->avail + h->lvl_off[n]; return b;
}

// ---------------------------------------------------------------------------
// 4. TBuddy over per-level availability bitmaps: bit i of level n
// set <=> node (n, i) is Available.  Partial/Busy are implied by
// the bits below a node, so no parent state needs locking.
// ---------------------------------------------------------------------------
static __device__ __forceinline__ bool node_inside(const ga_desc* h, int n, uint64_t i) { return ((i + 1) << n) <= h->pages; }

// make node i of level n available (a split's right child) and count it
static __device__ __forceinline__ void tree_publish(const ga_desc* h, int n, uint64_t i, uint32_t expected) {
    hb3_set(level_hb(h, n), i);
    bsem_signal(tsem_ptr(h, n), 1, expected);            // C += 1, retire the expected unit
}

// claim up to `need` available nodes of level n from one bitmap word (the
// caller holds `need` units of tsem[n]); returns the claimed mask, word in *wj
static __device__ __noinline__ uint64_t tree_claim_word(const ga_desc* h, int n, int need, uint32_t seed, uint64_t* wj) {
    GA_DBG_CNT;
    HB3 b = level_hb(h, n);
    uint32_t ns = 32;
#if GA_LVL_HINT
    int64_t j = ld_rlx32(&h->lvl_hint[n]);                   // the last word a claim succeeded in
    if (j >= b.n0 || ld_rlx(&b.w0[j]) == 0) j = -1;
#else
    int64_t j = -1;
#endif
    for (;;) {
        if (j < 0) j = hb3_find(b, seed);
        if (j >= 0) {
            uint64_t x = ld_rlx(&b.w0[j]);
            while (x) {
                uint64_t m = lowest_bits(x, need);
                uint64_t old = a_and(&b.w0[j], ~m);
                uint64_t got = old & m;
                if (old != 0 && (old & ~m) == 0) hb3_up_clear(b, (uint32_t)j);
                if (got) {
#if GA_LVL_HINT
                    if ((old & ~m) && ld_rlx32(&h->lvl_hint[n]) != (uint32_t)j) st_rlx32(&h->lvl_hint[n], (uint32_t)j);
#endif
                    *wj = (uint64_t)j;
                    return got;
                }
                x = old & ~m;
            }
        }
        j = -1;
        SPIN_NOTE(dbg_cnt, 4, ((uint64_t)n << 32) | (uint32_t)need, seed);
        __nanosleep(ns); if (ns < 1024) ns <<= 1;
        seed = hash32(seed + 1);
    }
}

// Single-thread allocation of one order-o block: climb while wait
// says GROW, claim at the first level that grants, split down publishing the
// right halves.  Returns the node at level o, or -1 (every E retracted).
static __device__ __noinline__ int64_t tree_alloc_one(const ga_desc* h, int o) {
    int m = o;
    for (;;) {
        if (m > (int)h->L) {
            for (int k = o; k < m; k++) bsem_signal(tsem_ptr(h, k), 0, 1);   // failure signal
            return -1;
        }
        if (bsem_wait_fast(tsem_ptr(h, m), 1, 2, NoSpin()) == kAcquired) break;   // batch two
        m++;
    }
    uint64_t wj;
    uint64_t got = tree_claim_word(h, m, 1, scatter_seed(), &wj);
    uint64_t x = wj * 64 + (uint64_t)(__ffsll((long long)got) - 1);
    for (int k = m - 1; k >= o; k--) { x = 2 * x; tree_publish(h, k, x + 1, 1); }
    reserve_add(h, (int64_t)1 << o);
    return (int64_t)x;
}

// Free node x of level n: merge with the buddy when try-wait and
// the buddy's available->busy transition both succeed, cascading upwards
// (R-19); otherwise mark x available with ONE CAS on the word holding both
// siblings (R-21), so two siblings never both end up available.
static __device__ __noinline__ void tree_free(const ga_desc* h, int n, uint64_t x) {
    GA_DBG_CNT;
    uint32_t ns = 32;
    reserve_add(h, -((int64_t)1 << n));
    for (;;) {
        HB3 b = level_hb(h, n);
        uint64_t* wp = &b.w0[x >> 6];
        uint64_t xb = 1ull << (x & 63), yb = 1ull << ((x ^ 1) & 63);
        bool root = (n >= (int)h->L) || !node_inside(h, n, x ^ 1);
        uint64_t w = ld_rlx(wp);
        if (!root && (w & yb)) {
            if (bsem_trywait(tsem_ptr(h, n), 1)) {
                uint64_t old = a_and(wp, ~yb);
                if (old & yb) {                               // merged: free the parent at n + 1
                    if (old == yb) hb3_up_clear(b, (uint32_t)(x >> 6));
                    x >>= 1; n++; ns = 32;
                    continue;
                }
                bsem_signal(tsem_ptr(h, n), 1, 0);            // buddy claimed meanwhile: give back
            } else {
                SPIN_NOTE(dbg_cnt, 5, ((uint64_t)n << 56) | x, w);
                __nanosleep(ns); if (ns < 1024) ns <<= 1;     // the buddy's unit is held by a claimer
            }
            continue;
        }
        uint64_t old = a_cas(wp, w, w | xb);
        if (old != w) continue;                               // the pair changed: re-evaluate
        if (w == 0) hb3_up_set(b, (uint32_t)(x >> 6));
        bsem_signal(tsem_ptr(h, n), 1, 0);
        return;
    }
}

// Supply visible to a failed climber (after it retracted its own E):
//   units  -- some order k >= o holds an available node now (C >= 1);
//   growth -- some order k >= o expects units nobody reserved yet (D > 0).
// At true exhaustion both are false.  Growth also counts other failing
// climbers' transient E, so only the first retries may wait on it.
static __device__ __noinline__ bool tree_has_supply(const ga_desc* h, int o, bool count_growth) {
    for (int k0 = o; k0 <= (int)h->L; k0 += 8) {                 // 8 independent loads per round trip
        uint64_t w[8];
#pragma unroll
        for (int i = 0; i < 8; i++) w[i] = k0 + i <= (int)h->L ? ld_rlx(tsem_ptr(h, k0 + i)) : dCD(0, 0);
#pragma unroll
        for (int i = 0; i < 8; i++)
            if (sem_C(w[i]) >= 1 || (count_growth && sem_D(w[i]) > 0)) return true;
    }
    return false;
}

// ---------------------------------------------------------------------------
// 5. UAlloc: chunks of 64 pages owned by one arena, one-page bins
// ---------------------------------------------------------------------------
static __device__ __forceinline__ uint32_t kind_bin(uint32_t A, int c) { return kKindBin | (A << 8) | (uint32_t)c; }
// Clear bit ch of one of arena A's chunk summaries when chunk ch is no longer
// A's or its data word reads `empty_value`; re-check both after the clear
// (clear-then-recheck).  A chunk that left A for another arena (spans recycle
// chunks often) must not stay visible in A's summary, or A's searches would
// keep returning it.
static __device__ __noinline__ void hb3_clear_owned(const ga_desc* h, HB3 b, uint64_t ch, uint32_t A,
                                                    const uint64_t* data, uint64_t empty_value) {
    uint64_t bit = 1ull << (ch & 63);
    uint64_t old = a_and(&b.w0[ch >> 6], ~bit);
    fence_sc();
    if (ld_rlx32(&h->chunk_owner[ch]) == A + 1 && ld_rlx(data) != empty_value) {
        if (a_or(&b.w0[ch >> 6], bit) == 0) hb3_up_set(b, (uint32_t)(ch >> 6));
        return;
    }
    if (old == bit) hb3_up_clear(b, (uint32_t)(ch >> 6));
}
static __device__ __forceinline__ uint64_t* nonfull_word(const ga_desc* h, uint64_t ch, int c) { return &h->chunk_nonfull[ch * kNcls + c]; }
static __device__ __forceinline__ bool page_full(const uint64_t w[4], int c) {
#pragma unroll
    for (int i = 0; i < 4; i++) if (i < words_of(c)) if ((w[i] | ~valid_mask(c, i)) != ~0ull) return false;
    return true;
}

static __device__ int reclaim_arena(const ga_desc* h, uint32_t A, int budget, uint32_t keep);
// delegated work run by threads blocked in an arena semaphore wait (Sec. 4.2.1);
// what they reclaim is counted (ga_stats n_waiter_reclaim)
struct ArenaSpin {
    const ga_desc* h; uint32_t A;
    __device__ void operator()() const {
        if (const int n = reclaim_arena(h, A, 4, kReclaimKeep)) stat_add(h, kStatWaiterReclaim, (uint64_t)n);
    }
};

// Data bit `bit` of *data (a per-chunk word: non-full pages, reclaim
// candidates) goes up, and chunk ch must then be visible in summary b.  The
// data word can hold a stale bit from the chunk's previous life (a free's
// delayed publication that landed after the page was reclaimed, while a stale
// summary bit was being cleaned up under another owner), so "the word was
// already non-zero" does not prove the summary has ch: the summary bit is
// checked after the data RMW has performed (a clearer re-checks the data after
// its own clear, so one of the two always sees the other).
static __device__ __noinline__ void summarised_set(HB3 b, uint64_t ch, uint64_t* data, uint64_t bit) {
    const uint64_t cb = 1ull << (ch & 63);
    if ((ld_rlx(data) & bit) == bit && (ld_rlx(&b.w0[ch >> 6]) & cb)) return;
    if (a_or(data, bit) == 0 || !(ld_rlx(&b.w0[ch >> 6]) & cb)) hb3_set(b, ch);
}
static __device__ __forceinline__ void mark_candidate(const ga_desc* h, uint64_t p, uint32_t A) {
    summarised_set(arena_hb(h, A, kAhbCnd), p >> kChunkShift, &h->chunk_cand[p >> kChunkShift],
                   1ull << (p & (kChunkPages - 1)));
}
// page p (class c, arena A) has a free slot again
static __device__ __forceinline__ void nonfull_set(const ga_desc* h, uint64_t p, int c, uint32_t A) {
    summarised_set(arena_hb(h, A, kAhbNfc + c), p >> kChunkShift, nonfull_word(h, p >> kChunkShift, c),
                   1ull << (p & (kChunkPages - 1)));
}
// drop p from the non-full set if it is really full (clear-then-recheck)
static __device__ __noinline__ void nonfull_clear_if_full(const ga_desc* h, uint64_t p, int c, uint32_t A) {
    uint64_t ch = p >> kChunkShift;
    uint64_t* nf = nonfull_word(h, ch, c);
    uint64_t bit = 1ull << (p & (kChunkPages - 1));
    uint64_t old = a_and(nf, ~bit);
    uint64_t w[4];
#if GA_RECHECK_RMW
    for (int i = 0; i < 4; i++) w[i] = i < words_of(c) ? recheck_read(&page_bits(h, p)[i]) : ~0ull;
#else
    fence_sc();
    ld_bitmap(page_bits(h, p), w);
#endif
    // Re-set the bit if p is a non-full class-c bin of ANY arena: a stale caller
    // (its chunk went back to the tree and on to another arena, which made p a
    // class-c bin again) must not leave the new owner's bin invisible.
    const uint32_t k = ld_rlx32(&h->kind[p]);
    if ((k & 0xC0000000u) == kKindBin && (int)(k & 0xFF) == c && !page_full(w, c)) {
        summarised_set(arena_hb(h, (k >> 8) & 0xFFFFu, kAhbNfc + c), ch, nf, bit);
        return;
    }
    if (old == bit) hb3_clear_owned(h, arena_hb(h, A, kAhbNfc + c), ch, A, nf, 0);
}

// Take a new chunk from TBuddy for arena A, keep its first k pages, open the rest.
static __device__ __noinline__ int64_t tree_alloc_one_retry(const ga_desc* h, int o, bool chunk_supply);
static __device__ __noinline__ int64_t chunk_acquire(const ga_desc* h, uint32_t A, uint32_t k) {
    int64_t ch = tree_alloc_one_retry(h, kChunkOrder, true);
    if (ch < 0) return -1;
    st_rlx32(&h->chunk_owner[ch], A + 1);
    fence();
    uint64_t keep = k >= 64 ? ~0ull : ((1ull << k) - 1);
    a_and(&h->chunk_used[ch], keep);                          // open pages k..63 (all ones while unowned)
    if (k < 64) hb3_set(arena_hb(h, A, kAhbFpc), (uint64_t)ch);
    stat_add(h, kStatChunkGrow, 1);
    return ch;
}

// Claim up to `need` free pages from ONE chunk of arena A (caller holds `need`
// units of psem[A]): one atomicOr per attempt.  Returns the page mask, chunk in *ch_out.
static __device__ __noinline__ uint64_t page_claim(const ga_desc* h, uint32_t A, int need, uint64_t* ch_out) {
    GA_DBG_CNT;
    HB3 fb = arena_hb(h, A, kAhbFpc);
    uint32_t seed = scatter_seed();
    uint32_t ns = 32;
    for (;;) {
        int64_t j = hb3_find(fb, seed);
        if (j >= 0) {
            uint64_t cm = ld_rlx(&fb.w0[j]);
            while (cm) {
                uint32_t bit = first_from(cm, seed);
                cm &= ~(1ull << bit);
                uint64_t ch = (uint64_t)j * 64 + bit;
                if (ld_rlx32(&h->chunk_owner[ch]) != A + 1) {        // left the arena: stale bit
                    hb3_clear_owned(h, fb, ch, A, &h->chunk_used[ch], ~0ull);
                    continue;
                }
                uint64_t u = ld_rlx(&h->chunk_used[ch]);
                while (~u) {
                    uint64_t m = lowest_bits(~u, need);
                    uint64_t old = a_or(&h->chunk_used[ch], m);
                    uint64_t got = m & ~old;
                    u = old | m;
                    if (!got) continue;
                    if (const uint32_t o = ld_rlx32(&h->chunk_owner[ch]); o != A + 1) {
                        // recycled chunk (now o's): undo, then re-publish the chunk
                        // in its owner's free-page summary -- a claimer of o may
                        // have seen our bits, found the chunk full and cleared it.
                        // Our bits kept the chunk from being released meanwhile,
                        // so o is its owner.
                        a_and(&h->chunk_used[ch], ~got);
                        if (o != 0) hb3_set(arena_hb(h, o - 1, kAhbFpc), (uint64_t)ch);
                        break;
                    }
                    if (u == ~0ull) hb3_clear_summarised(fb, ch, &h->chunk_used[ch], ~0ull);
                    *ch_out = ch;
                    return got;
                }
                if (u == ~0ull) hb3_clear_summarised(fb, ch, &h->chunk_used[ch], ~0ull);
            }
        }
        SPIN_NOTE(dbg_cnt, 6, A, need);
        __nanosleep(ns); if (ns < 1024) ns <<= 1;
        seed = hash32(seed + 5);
    }
}

static __device__ void chunk_release(const ga_desc* h, uint64_t ch);
// Return page p to its chunk (C += 1 on the owner's page semaphore); an empty
// chunk goes back to TBuddy (R-23).
static __device__ __noinline__ void page_release(const ga_desc* h, uint64_t p) {
    uint64_t ch = p >> kChunkShift;
    uint32_t A = ld_rlx32(&h->chunk_owner[ch]) - 1;
    uint64_t bit = 1ull << (p & (kChunkPages - 1));
    uint64_t old = a_and(&h->chunk_used[ch], ~bit);
    if (old == ~0ull) hb3_set(arena_hb(h, A, kAhbFpc), ch);
    bsem_signal(psem_ptr(h, A), 1, 0);
    if ((old & ~bit) == 0) chunk_release(h, ch);
}

// An empty chunk back to TBuddy: try-wait its 64 page units, then take every
// page with one CAS (0 -> all ones).  Failure leaves the chunk with its arena.
static __device__ __noinline__ void chunk_release(const ga_desc* h, uint64_t ch) {
    uint32_t A = ld_rlx32(&h->chunk_owner[ch]) - 1;
    if (A >= h->n_arenas) return;
    if (!bsem_trywait(psem_ptr(h, A), kChunkPages)) return;
    if (a_cas(&h->chunk_used[ch], 0ull, ~0ull) != 0ull) { bsem_signal(psem_ptr(h, A), kChunkPages, 0); return; }
    // ABA (as in bin_reclaim): the chunk may have left A and come back empty
    // under another arena between the owner read and the CAS.  It cannot move
    // while its used word is all ones, so the owner read here decides.
    if (const uint32_t o2 = ld_rlx32(&h->chunk_owner[ch]); o2 != A + 1) {
        a_and(&h->chunk_used[ch], 0ull);
        bsem_signal(psem_ptr(h, A), kChunkPages, 0);
        if (o2 != 0) hb3_set(arena_hb(h, o2 - 1, kAhbFpc), ch);
        return;
    }
    hb3_clear_summarised(arena_hb(h, A, kAhbFpc), ch, &h->chunk_used[ch], ~0ull);
    if (a_exch(&h->chunk_cand[ch], 0)) hb3_clear_summarised(arena_hb(h, A, kAhbCnd), ch, &h->chunk_cand[ch], 0);
    st_rlx32(&h->chunk_owner[ch], 0);
    fence();
    stat_add(h, kStatChunkReclaim, 1);
    tree_free(h, kChunkOrder, ch);
}

// Make page p a bin of class c for arena A; the caller keeps slots [0, take),
// the others are opened (the bitmap is all ones while p is not a bin).
static __device__ __forceinline__ void st_kinds_span(const ga_desc* h, uint64_t head, uint32_t k) {
    uint32_t* kp = &h->kind[head];                          // 64 u32 = 16 x 16-byte stores
    for (int i = 0; i < (int)kChunkPages; i += 4)
        asm volatile("st.relaxed.gpu.global.v4.u32 [%0], {%1,%1,%1,%1};" :: "l"(kp + i), "r"(k) : "memory");
}
static __device__ __forceinline__ void bin_init(const ga_desc* h, uint64_t p, uint32_t A, int c, uint32_t take) {
    if (is_span(c)) st_kinds_span(h, p, kind_bin(A, c));    // free() looks up any page of the span
    else st_rlx32(&h->kind[p], kind_bin(A, c));
    fence();
    uint64_t* bw = page_bits(h, p);
    for (int w = 0; w < words_of(c); w++) {
        int lo = (int)take - 64 * w;
        uint64_t keep = lo >= 64 ? ~0ull : lo <= 0 ? 0ull : ((1ull << lo) - 1);
        uint64_t open = valid_mask(c, w) & ~keep;
        if (open) a_and(&bw[w], ~open);
    }
    if (take < slots_of(c)) nonfull_set(h, p, c, A);
}

// Give back slots `got` of word i of page p, taken by a stale claimer after p
// became a bin of another incarnation (kind k2), and re-publish p for it.
static __device__ __noinline__ void undo_claim(const ga_desc* h, uint64_t p, int i, uint64_t got, uint32_t k2) {
    a_and(&page_bits(h, p)[i], ~got);
    if ((k2 & 0xC0000000u) == kKindBin) {
        nonfull_set(h, p, (int)(k2 & 0xFF), (k2 >> 8) & 0xFFFFu);
        mark_candidate(h, p, (k2 >> 8) & 0xFFFFu);
    }
}

// Claim up to `need` slots of page p (an (A, c) bin) from one bitmap word with
// one atomicOr.  Returns the claimed mask (word in *wi); 0 if none.  The page
// kind and the bitmap are loaded together (independent round trips), and the
// word scan starts at `rot` so concurrent warps on one page spread over its
// words (scattered search).  Loops stay rolled: this is the hottest
// code of the allocator and instruction-fetch stalls dominate.
static __device__ GA_CLAIM_FN uint64_t bin_claim_page(const ga_desc* h, uint64_t p, uint32_t A, int c, int need, int* wi,
                                                       uint32_t rot, bool recheck = true) {
    uint64_t* bw = page_bits(h, p);
    uint64_t w[4];
    const uint32_t k0 = ld_rlx32(&h->kind[p]);
    ld_bitmap(bw, w);
    if (k0 != kind_bin(A, c)) {
        // A stale non-full bit: a free's delayed nonfull_set can land after the
        // page was reclaimed (or re-classed).  Drop it (the helper re-sets it if
        // p is in fact a non-full class-c bin), or every claimer that lands on
        // p would retry it forever.
        nonfull_clear_if_full(h, p, c, A);
        return 0;
    }
    const int nw = words_of(c);
#pragma unroll 1
    for (int t = 0; t < nw; t++) {
        const int i = (int)((t + rot) & (uint32_t)(nw - 1));
        const uint64_t vm = valid_mask(c, i);
        uint64_t wi_v = i == 0 ? w[0] : i == 1 ? w[1] : i == 2 ? w[2] : w[3];
        uint64_t fr = ~wi_v & vm;
        while (fr) {
            uint64_t m = lowest_bits(fr, need);
            uint64_t old = a_or(&bw[i], m);
            uint64_t got = m & ~old;
            if (got) {
                if (const uint32_t k2 = recheck ? ld_rlx32(&h->kind[p]) : kind_bin(A, c); k2 != kind_bin(A, c)) {
                    // recycled page: undo, then re-publish it for its real
                    // owner (as bin_reclaim's ABA path does): a claimer of
                    // (A', c') may have seen our bits and dropped the page
                    undo_claim(h, p, i, got, k2);
                    return 0;
                }
                if (!GA_LAZY_CLEAR && ((old | m) | ~vm) == ~0ull) {   // this word is full now
                    ld_bitmap(bw, w);
                    if (page_full(w, c)) nonfull_clear_if_full(h, p, c, A);
                }
                *wi = i;
                return got;
            }
            fr = ~(old | m) & vm;
        }
    }
    nonfull_clear_if_full(h, p, c, A);
    return 0;
}

#if GA_DEBUG
// Debug builds: a claimer stuck in bin_find_chunk audits arena A's class-c
// bins once (single auditor) into the debug header words 1..7.
static __device__ __noinline__ void nfc_audit(const ga_desc* h, uint32_t A, int c) {
    uint64_t* dbg = h->dbg;
    if (!dbg || atomicCAS((unsigned long long*)&dbg[1], 0ull, 1ull) != 0ull) return;
    HB3 nb = arena_hb(h, A, kAhbNfc + c);
    uint64_t nbins = 0, nfree = 0, lost_nf = 0, lost_sum = 0, lost_up = 0;
    for (uint64_t ch = 0; ch < h->nchunks; ch++) {
        if (ld_rlx32(&h->chunk_owner[ch]) != A + 1) continue;
        uint64_t nf = ld_rlx(nonfull_word(h, ch, c));
        for (uint32_t j = 0; j < kChunkPages; j++) {
            uint64_t p = ch * kChunkPages + j;
            if (ld_rlx32(&h->kind[p]) != kind_bin(A, c) || bin_head(p, c) != p) continue;
            nbins++;
            uint64_t w[4];
            ld_bitmap(page_bits(h, p), w);
            uint64_t fr = 0;
            for (int i = 0; i < words_of(c); i++) fr += __popcll(~w[i] & valid_mask(c, i));
            nfree += fr;
            if (fr && !((nf >> j) & 1)) lost_nf++;
        }
        if (nf) {
            if (!((ld_rlx(&nb.w0[ch >> 6]) >> (ch & 63)) & 1)) lost_sum++;
            else if (!((ld_rlx(&hb3_w1(nb)[ch >> 12]) >> ((ch >> 6) & 63)) & 1) ||
                     !((ld_rlx(&hb3_w2(nb)[ch >> 18]) >> ((ch >> 12) & 63)) & 1)) lost_up++;
        }
    }
    uint64_t sw = ld_rlx(sem_ptr(h, A, c));
    volatile uint64_t* r = (volatile uint64_t*)dbg;
    r[2] = ((uint64_t)A << 8) | (uint64_t)c | ((uint64_t)(uint32_t)sem_C(sw) << 32);
    r[3] = nbins; r[4] = nfree; r[5] = lost_nf; r[6] = lost_sum;
    r[7] = lost_up | ((uint64_t)(uint32_t)sem_D(sw) << 32);
    __threadfence_system();
    r[1] = 2;
}
#endif

// Safety net for a claimer that holds units but finds no non-full (A, c) bin
// for a long time (hundreds of microseconds: growers publish before they
// signal, so a legitimate wait is short).  Walk arena A's chunks and re-publish
// what the per-chunk words and summaries should show: (A, c) bins with a free
// slot and no non-full bit, and non-full words whose chunk is missing from the
// summary.  Each repair is counted (ga_stats n_repair_*), so a run that needed
// one is visible; the measured runs of profiles/ report zero.
static __device__ __noinline__ void nfc_repair(const ga_desc* h, uint32_t A, int c) {
    HB3 nb = arena_hb(h, A, kAhbNfc + c);
    const uint32_t step = is_span(c) ? kChunkPages : 1;
    for (uint64_t ch = 0; ch < h->nchunks; ch++) {
        if (ld_rlx32(&h->chunk_owner[ch]) != A + 1) continue;
        uint64_t* nf = nonfull_word(h, ch, c);
        for (uint32_t j = 0; j < kChunkPages; j += step) {
            const uint64_t p = ch * kChunkPages + j;
            if (ld_rlx32(&h->kind[p]) != kind_bin(A, c)) continue;
            uint64_t w[4];
            ld_bitmap(page_bits(h, p), w);
            if (!page_full(w, c) && !((ld_rlx(nf) >> j) & 1)) {
                summarised_set(nb, ch, nf, 1ull << j);
                stat_add(h, kStatRepairNonfull, 1);
            }
        }
        if (ld_rlx(nf) && !((ld_rlx(&nb.w0[ch >> 6]) >> (ch & 63)) & 1)) {
            hb3_set(nb, ch);
            stat_add(h, kStatRepairSummary, 1);
        }
    }
    if (h->dbg && atomicCAS((unsigned long long*)&h->dbg[1], 0ull, 1ull) == 0ull) {
        // one diagnostic dump (header words 2..7): where are arena A's class-c
        // units?  Spans / bins of kind (A, c) anywhere, their free slots, how
        // many sit in chunks not owned by A, how many lack their non-full bit.
        uint64_t nb_all = 0, free_all = 0, foreign = 0, nf_missing = 0, free_foreign = 0;
        for (uint64_t p = 0; p < h->pages; p += step) {
            if (ld_rlx32(&h->kind[p]) != kind_bin(A, c)) continue;
            uint64_t w[4];
            ld_bitmap(page_bits(h, p), w);
            uint64_t fr = 0;
            for (int i = 0; i < 4; i++) if (i < words_of(c)) fr += __popcll(~w[i] & valid_mask(c, i));
            nb_all++; free_all += fr;
            const uint64_t ch = p >> kChunkShift;
            if (ld_rlx32(&h->chunk_owner[ch]) != A + 1) { foreign++; free_foreign += fr; }
            if (fr && !((ld_rlx(nonfull_word(h, ch, c)) >> (p & (kChunkPages - 1))) & 1)) nf_missing++;
        }
        // chunks owned by A + 1 and what their head page says
        uint64_t owned = 0, owned_k0 = 0, owned_other = 0;
        for (uint64_t ch = 0; ch < h->nchunks; ch++) {
            if (ld_rlx32(&h->chunk_owner[ch]) != A + 1) continue;
            owned++;
            const uint32_t k = ld_rlx32(&h->kind[ch * kChunkPages]);
            if (k == 0) owned_k0++;
            else if (k != kind_bin(A, c)) owned_other++;
        }
        const uint64_t sw = ld_rlx(sem_ptr(h, A, c));
        volatile uint64_t* r = (volatile uint64_t*)h->dbg;
        r[2] = ((uint64_t)A << 8) | (uint64_t)c | ((uint64_t)(uint32_t)sem_C(sw) << 32);
        r[3] = nb_all; r[4] = free_all; r[5] = foreign | (free_foreign << 32); r[6] = nf_missing;
        r[7] = ((uint64_t)(uint32_t)sem_D(sw) << 32);
        r[8 + 4 * 255 + 0] = owned; r[8 + 4 * 255 + 1] = owned_k0; r[8 + 4 * 255 + 2] = owned_other;
        r[8 + 4 * 255 + 3] = ld_rlx(&h->stats[kStatChunkGrow]) | (ld_rlx(&h->stats[kStatChunkReclaim]) << 32);
        __threadfence_system();
        r[1] = 2;
    }
    for (uint32_t j = 0; j < nb.n0; j++)                      // upper summary levels
        if (ld_rlx(&nb.w0[j]) && !((ld_rlx(&hb3_w1(nb)[j >> 6]) >> (j & 63)) & 1)) {
            hb3_up_set(nb, j);
            stat_add(h, kStatRepairSummary, 1);
        }
}

// Per block: the chunk (as a page index) a claim of class c last used -- the
// block's warps share one arena, so this is a copy of the (A, c) hint that
// costs a shared-memory load instead of an L2 round trip.  Only a hint: its
// owner and non-full word are validated before use.
static __shared__ uint32_t s_chunk_hint[kNcls];

// A chunk of arena A with non-full class-c bins, and its non-full page mask:
// the hint's chunk first, then the (A, c) summary.  Spins until one shows up
// (the caller holds units, so a free slot exists or is being published).
static __device__ __noinline__ uint64_t bin_find_chunk_search(const ga_desc* h, uint32_t A, int c, uint64_t* mask_out);
static __device__ GA_CLAIM_FN uint64_t bin_find_chunk(const ga_desc* h, uint32_t A, int c, uint64_t* mask_out) {
#if GA_HINT_LDCA
    // the hint is only a hint: an L1-cached (possibly stale) read saves an L2
    // round trip; the chunk's owner and non-full word below are read fresh
    uint32_t hp = __ldca(&h->hint[A * kNcls + c]);
#else
    uint32_t hp = ld_rlx32(&h->hint[A * kNcls + c]);
#endif
    if (hp < h->pages) {                                      // the hint's chunk, if still A's
        const uint32_t own = ld_rlx32(&h->chunk_owner[hp >> kChunkShift]);
        uint64_t m = ld_rlx(nonfull_word(h, hp >> kChunkShift, c));
        if (own == A + 1 && m) { s_chunk_hint[c] = hp; *mask_out = m; return hp >> kChunkShift; }
    }
    return bin_find_chunk_search(h, A, c, mask_out);
}
// the (A, c) summary search behind the hint (out of line: rare, and it spins)
static __device__ __noinline__ uint64_t bin_find_chunk_search(const ga_desc* h, uint32_t A, int c, uint64_t* mask_out) {
    GA_DBG_CNT;
    HB3 nb = arena_hb(h, A, kAhbNfc + c);
    uint32_t seed = scatter_seed();
    uint32_t ns = 32, spins = 0;
    for (;;) {
        int64_t j = hb3_find(nb, seed);
        if (j >= 0) {
            uint64_t cm = ld_rlx(&nb.w0[j]);
            while (cm) {
                uint32_t bit = first_from(cm, seed);
                cm &= ~(1ull << bit);
                uint64_t ch = (uint64_t)j * 64 + bit;
                const uint32_t own = ld_rlx32(&h->chunk_owner[ch]);
                uint64_t m = ld_rlx(nonfull_word(h, ch, c));
                if (own == A + 1 && m) {
                    st_rlx32(&h->hint[A * kNcls + c], (uint32_t)(ch * kChunkPages + (__ffsll((long long)m) - 1)));
                    s_chunk_hint[c] = (uint32_t)(ch * kChunkPages);
                    *mask_out = m;
                    return ch;
                }
                hb3_clear_owned(h, nb, ch, A, nonfull_word(h, ch, c), 0);    // stale summary bit
            }
        }
#if GA_DEBUG
        if (((dbg_cnt + 1) & ((1u << 18) - 1)) == 0) nfc_audit(h, A, c);
#endif
        SPIN_NOTE(dbg_cnt, 7, ((uint64_t)A << 8) | c, ns);
        __nanosleep(ns); if (ns < 1024) ns <<= 1;
        seed = hash32(seed + 7);
        if ((++spins & 255) == 0) nfc_repair(h, A, c);
    }
}

#ifndef GA_SPAN_ROT
#define GA_SPAN_ROT 0            // 1: span claims start at a per-warp rotation within the summary word
#endif
#ifndef GA_SPREAD
#define GA_SPREAD 1              // 1: lockstep retries pick their chunk from the hint's summary word by warp rotation
#endif
// A retry's chunk: every warp of an SM starts at the same hinted chunk, and a
// class with few slots per page (2 KiB: 2) fills it long before the warps are
// served (6-7 warp iterations per call on d3 1-2 KiB).  A retry instead takes
// the summary word holding the hinted chunk (up to 64 of arena A's chunks with
// non-full class-c pages) and picks one by the warp's rotation, so the warps
// of an arena spread over its chunks.  Falls back to bin_find_chunk.
static __device__ __forceinline__ uint64_t bin_spread_chunk(const ga_desc* h, uint32_t A, int c, uint32_t sel,
                                                            uint64_t* mask_out) {
    const uint32_t hp = s_chunk_hint[c];
    if (hp < h->pages) {
        const uint64_t w = ld_rlx(&arena_hb(h, A, kAhbNfc + c).w0[hp >> (2 * kChunkShift)]);
        if (w) {
            const uint64_t ch = ((uint64_t)(hp >> (2 * kChunkShift)) << kChunkShift) + nth_set(w, sel % (uint32_t)__popcll(w));
            const uint32_t own = ld_rlx32(&h->chunk_owner[ch]);
            const uint64_t m = ld_rlx(nonfull_word(h, ch, c));
            if (own == A + 1 && m) { *mask_out = m; return ch; }
        }
    }
    return bin_find_chunk(h, A, c, mask_out);
}

// Spans: one candidate per CHUNK, so a chunk's non-full mask names one span
// and a group needing more slots than one span holds would take one span per
// iteration (36 warp iterations per call on d3 64 KiB).  Instead the leader
// takes a whole level-0 word of the (A, c) non-full summary: up to 64 spans
// with free slots, over which the group's lanes spread by rank.  Returns the
// summary word index j; *mask_out = its chunk bits (non-zero).  Stale bits
// are validated by the claim (page kind) and cleaned by the claimer.
static __device__ __forceinline__ uint64_t span_find_word(const ga_desc* h, uint32_t A, int c, uint64_t* mask_out) {
    HB3 nb = arena_hb(h, A, kAhbNfc + c);
    const uint32_t hp = ld_rlx32(&h->hint[A * kNcls + c]);
    if (hp < h->pages) {
        const uint64_t j = (uint64_t)hp >> (2 * kChunkShift);
        const uint64_t m = ld_rlx(&nb.w0[j]);
        if (m) { *mask_out = m; return j; }
    }
    uint64_t m1;
    const uint64_t ch = bin_find_chunk_search(h, A, c, &m1);             // spins until a span shows up
    const uint64_t j = ch >> kChunkShift;
    *mask_out = ld_rlx(&nb.w0[j]) | (1ull << (ch & 63));
    return j;
}

// ---------------------------------------------------------------------------
// 6. deferred reclamation: a free that empties a bin only marks
// it; threads blocked in a semaphore wait, growers about to take a new chunk,
// failing mallocs and ga_heap_quiesce do the reclaiming.
// ---------------------------------------------------------------------------
// An empty span's chunk back to TBuddy (its slots were taken by the reclaimer;
// chunk_used stays all ones, as for any chunk outside an arena).
static __device__ __noinline__ void span_release(const ga_desc* h, uint64_t ch, uint32_t A) {
    st_kinds_span(h, ch * kChunkPages, 0);
    if (a_exch(&h->chunk_cand[ch], 0)) hb3_clear_summarised(arena_hb(h, A, kAhbCnd), ch, &h->chunk_cand[ch], 0);
    st_rlx32(&h->chunk_owner[ch], 0);
    fence();
    stat_add(h, kStatChunkReclaim, 1);
    tree_free(h, kChunkOrder, ch);
}

// Reclaim page p if it is an empty bin: try-wait all its slots (R-22), then take
// every slot word with a CAS (all free -> all ones).  `keep`: leave at least
// that many free slots of the class behind -- delegated reclamation must not
// take the bins the waiting threads are about to use (0 for quiesce).
static __device__ __noinline__ bool bin_reclaim(const ga_desc* h, uint64_t p, uint32_t keep) {
    uint32_t k = ld_rlx32(&h->kind[p]);
    if ((k & 0xC0000000u) != kKindBin) return false;
    uint32_t A = (k >> 8) & 0xFFFFu;
    int c = (int)(k & 0xFF);
    if (is_span(c) && (p & (kChunkPages - 1))) return false;   // spans: the head page only
    uint64_t* bw = page_bits(h, p);
    uint64_t w[4];
    ld_bitmap(bw, w);
#pragma unroll
    for (int i = 0; i < 4; i++) if (i < words_of(c) && (w[i] & valid_mask(c, i))) return false;
    uint32_t slots = slots_of(c);
    if (is_span(c) && keep > slots) keep = slots;             // delegated: keep one span's worth
    if (!bsem_trywait(sem_ptr(h, A, c), slots, keep)) return false;
    int i = 0;
    for (; i < words_of(c); i++) {
        uint64_t v = valid_mask(c, i);
        if (a_cas(&bw[i], ~v, ~0ull) != ~v) break;
    }
    if (i < words_of(c)) {                                    // a slot was claimed meanwhile: undo
        for (int q = 0; q < i; q++) a_and(&bw[q], ~valid_mask(c, q));
        bsem_signal(sem_ptr(h, A, c), slots, 0);
        return false;
    }
    // ABA: between the kind read and the CAS, p may have been reclaimed by
    // someone else and re-made an empty bin of another arena (chunks move
    // between arenas); the units just taken are then the wrong semaphore's.
    // With every slot word now all ones the incarnation cannot change under
    // us, so the kind read here decides: on a mismatch restore the words, give
    // the units back and re-publish the page for its real owner.
    if (const uint32_t k2 = ld_rlx32(&h->kind[p]); k2 != k) {
        for (int q = 0; q < words_of(c); q++) a_and(&bw[q], ~valid_mask(c, q));
        bsem_signal(sem_ptr(h, A, c), slots, 0);
        if ((k2 & 0xC0000000u) == kKindBin) {
            nonfull_set(h, p, (int)(k2 & 0xFF), (k2 >> 8) & 0xFFFFu);
            mark_candidate(h, p, (k2 >> 8) & 0xFFFFu);
        }
        return false;
    }
    uint64_t ch = p >> kChunkShift;
    uint64_t* nf = nonfull_word(h, ch, c);
    uint64_t bit = 1ull << (p & (kChunkPages - 1));
    if (a_and(nf, ~bit) == bit) hb3_clear_owned(h, arena_hb(h, A, kAhbNfc + c), ch, A, nf, 0);
    stat_add(h, kStatBinReclaim, 1);
    if (is_span(c)) { span_release(h, ch, A); return true; }
    st_rlx32(&h->kind[p], 0);
    fence();
    page_release(h, p);
    return true;
}


// Reclaim up to `budget` candidate bins of arena A (budget < 0: all), leaving
// at least `keep` free slots per class (0: reclaim every empty bin).  Returns
// the number of bins reclaimed.
static __device__ __noinline__ int reclaim_arena(const ga_desc* h, uint32_t A, int budget, uint32_t keep) {
    HB3 cb = arena_hb(h, A, kAhbCnd);
    if (!hb3_any(cb)) return 0;
    uint32_t seed = scatter_seed();
    int done = 0;
    while (budget != 0) {
        int64_t j = hb3_find(cb, seed);
        if (j < 0) return done;
        uint64_t cm = ld_rlx(&cb.w0[j]);
        if (!cm) { hb3_up_clear(cb, (uint32_t)j); continue; }
        uint64_t ch = (uint64_t)j * 64 + (uint64_t)(__ffsll((long long)cm) - 1);
        uint64_t pm = a_exch(&h->chunk_cand[ch], 0);
        hb3_clear_summarised(cb, ch, &h->chunk_cand[ch], 0);
        uint64_t pm_left = 0;
        while (pm) {
            uint32_t pb = (uint32_t)(__ffsll((long long)pm) - 1);
            pm &= pm - 1;
            if (budget == 0) { mark_candidate(h, ch * kChunkPages + pb, A); continue; }
            if (bin_reclaim(h, ch * kChunkPages + pb, keep)) done++;
            else {
                // still empty but the class needs it for now: keep it a candidate
                uint64_t w[4];
                ld_bitmap(page_bits(h, ch * kChunkPages + pb), w);
                if (ld_rlx32(&h->kind[ch * kChunkPages + pb]) & kKindBin) {
                    int c = (int)(ld_rlx32(&h->kind[ch * kChunkPages + pb]) & 0xFF);
                    bool empty = true;
#pragma unroll
                    for (int i = 0; i < 4; i++) if (i < words_of(c) && (w[i] & valid_mask(c, i))) empty = false;
                    if (empty) { pm_left |= 1ull << pb; }
                }
            }
            if (budget > 0) budget--;
        }
        if (pm_left) {                                      // re-mark what could not go yet
            summarised_set(cb, ch, &h->chunk_cand[ch], pm_left);
            return done;                                    // and stop: the rest is in use too
        }
    }
    return done;
}
// Reclaim every candidate of arenas A0, A0 + step, ...: the arenas' top summary
// words are loaded 16 at a time (independent loads, one round trip per batch)
// and only arenas with candidates are visited.
static __device__ __noinline__ void reclaim_arenas(const ga_desc* h, uint32_t A0, uint32_t step) {
    for (uint32_t base = A0; base < h->n_arenas; base += 16 * step) {
        uint64_t top[16];
#pragma unroll
        for (int i = 0; i < 16; i++) {
            const uint32_t A = base + i * step;
            top[i] = A < h->n_arenas ? ld_rlx(hb3_w2(arena_hb(h, A, kAhbCnd))) : 0;
        }
#pragma unroll 1
        for (int i = 0; i < 16; i++)
            if (top[i]) reclaim_arena(h, base + i * step, -1, 0);
    }
}
// Drain every arena's reclaim candidates (failing mallocs, exhausted chunk
// supply).  One drain runs at a time; a caller that finds one running waits
// until a drain that STARTED after its arrival has completed (two completed
// drains past its arrival generation: drains are serialised, so the second
// began after it arrived and saw every candidate it could have seen), then
// returns without a scan of its own.  At exhaustion tens of thousands of
// failing lanes each swept all 148 arenas (a 13 s step at block scope, d3
// 64 KiB); now they share sweeps.  Same guarantee for every caller: all
// candidates present at its arrival have been reclaimed or found in use.
static __device__ __noinline__ void reclaim_all(const ga_desc* h) {
    uint64_t* lock = &h->stats[kStatDrainLock];
    uint64_t* gen = &h->stats[kStatDrainGen];
    const uint64_t g0 = ld_rlx(gen);
    uint32_t ns = 256;
    for (;;) {
        if (ld_rlx(lock) == 0 && a_cas(lock, 0ull, 1ull) == 0ull) {
            fence();
            reclaim_arenas(h, 0, 1);
            fence();
            a_add(gen, 1);
            a_exch(lock, 0ull);
            return;
        }
        if (ld_rlx(gen) >= g0 + 2) { fence(); return; }
        __nanosleep(ns); if (ns < 4096) ns <<= 1;
    }
}

// Per-lane TBuddy allocation with the no-false-starvation retry: the optimistic
// order semaphores can send a lane up the tree while another lane's split is
// still in flight.  Retry while the tree shows supply; drain reclamation once.
// chunk_supply: the caller is a bin / span grower whose failure the arena
// fallback (group_fallback) re-checks against growth in flight, so it fails
// at once when no order >= o holds an Available node (other climbers' expected
// units at exhaustion are failing climbers, and waiting on them convoys).
static __device__ __noinline__ int64_t tree_alloc_one_retry(const ga_desc* h, int o, bool chunk_supply) {
    GA_DBG_CNT;
    bool drained = false;
    uint32_t ns = 64;
    // Nothing Available at any order >= o.  While a split is in flight (some
    // order expects units, D > 0) that is the cold-start convoy behind the
    // first climbers, not exhaustion: wait for it (bounded) instead of
    // draining every arena's reclaim candidates and failing the chunk supply
    // -- that drained bins the arenas needed again at once, and the regrowth
    // churned the tree (d4 steps of 12-17 ms instead of 6; 87 k bin reclaims).
    // Only when no split is in flight (or after ~30 us) drain once, and climb
    // only if that freed something.
    for (int w = 0; chunk_supply && !tree_has_supply(h, o, false); w++) {
        if (w >= 12 || !tree_has_supply(h, o, true)) {
            reclaim_all(h);
            if (!tree_has_supply(h, o, false)) return -1;
            drained = true;
            break;
        }
        __nanosleep(ns); if (ns < 4096) ns <<= 1;
    }
    ns = 64;
    for (int attempt = 0; attempt < 32; attempt++) {
        int64_t x = tree_alloc_one(h, o);
        if (x >= 0) return x;
        if (!tree_has_supply(h, o, attempt < 2)) {
            if (drained) return -1;
            reclaim_all(h);                                     // empty bins / chunks back to the tree
            drained = true;
            continue;
        }
        SPIN_NOTE(dbg_cnt, 8, o, attempt);
        __nanosleep(ns); if (ns < 4096) ns <<= 1;
    }
    return -1;
}

// ---------------------------------------------------------------------------
// 7. front end: warp-collective entry
// ---------------------------------------------------------------------------
// size -> key: 0..7 bin class, 8 + order for TBuddy, -1 for NULL
static __device__ __forceinline__ int size_key(const ga_desc* h, uint64_t n) {
    if (n == 0 || n > (h->pages << kPageShift)) return -1;             // R-15
    if (n <= 16) return 0;
    int lg = 64 - __clzll((long long)(n - 1));                         // ceil(log2 n), R-14
    if (lg <= 11 + kNspan) return lg - kMinShift;                      // <= 2048 B: bins (R-12); spans
    int o = lg - kPageShift;
    if (o > (int)h->L) return -1;
    return kNcls + o;
}

// Per-lane slow path (R-26, R-27): N = 1 waits; after local growth fails, drain
// reclamation, then take pages and slots from other arenas before NULL.  Every
// page source is tried before every other arena's bins (page sources only
// shrink in malloc-only phases), so a malloc fails only if no arena can serve.
static __device__ __noinline__ uint64_t bin_claim_one(const ga_desc* h, uint32_t A, int c) {
    uint64_t csz = 16ull << c;
    for (;;) {
        uint64_t m;
        uint64_t ch = bin_find_chunk(h, A, c, &m);
        uint64_t p = ch * kChunkPages + (uint64_t)(__ffsll((long long)m) - 1);
        int wi;
        uint64_t got = bin_claim_page(h, p, A, c, 1, &wi, 0);
        if (got) return (p << kPageShift) + (uint64_t)(wi * 64 + __ffsll((long long)got) - 1) * csz;
    }
}
// a fresh span for arena A straight from TBuddy (one chunk); -1 if the tree is exhausted
static __device__ __noinline__ int64_t span_acquire(const ga_desc* h, uint32_t A) {
    int64_t ch = tree_alloc_one_retry(h, kChunkOrder, true);
    if (ch < 0) return -1;
    st_rlx32(&h->chunk_owner[ch], A + 1);
    stat_add(h, kStatChunkGrow, 1);
    return ch;
}
static __device__ __noinline__ uint64_t span_malloc_lane(const ga_desc* h, uint32_t A0, int c) {
    uint32_t slots = slots_of(c);
    for (int attempt = 0; attempt < 2; attempt++) {
        if (bsem_wait(sem_ptr(h, A0, c), 1, slots, ArenaSpin{h, A0}) == kAcquired) return bin_claim_one(h, A0, c);
        reclaim_arena(h, A0, -1, kReclaimKeep);
        int64_t ch = span_acquire(h, A0);
        if (ch >= 0) {
            uint64_t p = (uint64_t)ch * kChunkPages;
            bin_init(h, p, A0, c, 1);
            stat_add(h, kStatBinGrow, 1);
            st_rlx32(&h->hint[A0 * kNcls + c], (uint32_t)p);
            bsem_signal(sem_ptr(h, A0, c), slots - 1, slots - 1);
            return p << kPageShift;
        }
        bsem_signal(sem_ptr(h, A0, c), 0, slots - 1);
        if (attempt == 0) reclaim_all(h);
    }
    for (uint32_t t = 1; t <= h->n_arenas; t++) {
        uint32_t B = (A0 + t) % h->n_arenas;
        uint64_t cw = ld_rlx(sem_ptr(h, B, c));
        if (sem_C(cw) < 1 && (int64_t)sem_C(cw) + sem_D(cw) < 1) continue;
        if (bsem_wait(sem_ptr(h, B, c), 1, 1, NoSpin()) == kAcquired) return bin_claim_one(h, B, c);
    }
    stat_add(h, kStatFail, 1);
    return kNull;
}
static __device__ __noinline__ uint64_t bin_malloc_lane(const ga_desc* h, uint32_t A0, int c) {
    if (is_span(c)) return span_malloc_lane(h, A0, c);
    uint32_t slots = slots_of(c);
    for (int attempt = 0; attempt < 2; attempt++) {
        if (bsem_wait(sem_ptr(h, A0, c), 1, slots, ArenaSpin{h, A0}) == kAcquired) return bin_claim_one(h, A0, c);
        uint64_t p = kNull;
        if (bsem_wait(psem_ptr(h, A0), 1, kChunkPages, ArenaSpin{h, A0}) == kAcquired) {
            uint64_t ch;
            uint64_t pm = page_claim(h, A0, 1, &ch);
            p = ch * kChunkPages + (uint64_t)(__ffsll((long long)pm) - 1);
        } else {
            reclaim_arena(h, A0, -1, kReclaimKeep);
            int64_t ch = chunk_acquire(h, A0, 1);
            if (ch >= 0) { bsem_signal(psem_ptr(h, A0), kChunkPages - 1, kChunkPages - 1); p = (uint64_t)ch * kChunkPages; }
            else bsem_signal(psem_ptr(h, A0), 0, kChunkPages - 1);
        }
        if (p != kNull) {
            bin_init(h, p, A0, c, 1);
            stat_add(h, kStatBinGrow, 1);
            st_rlx32(&h->hint[A0 * kNcls + c], (uint32_t)p);
            bsem_signal(sem_ptr(h, A0, c), slots - 1, slots - 1);
            return p << kPageShift;
        }
        bsem_signal(sem_ptr(h, A0, c), 0, slots - 1);
        if (attempt == 0) reclaim_all(h);
    }
    for (uint32_t t = 1; t <= h->n_arenas; t++) {
        uint32_t B = (A0 + t) % h->n_arenas;
        uint64_t pw = ld_rlx(psem_ptr(h, B));
        if (sem_C(pw) < 1 && (int64_t)sem_C(pw) + sem_D(pw) < 1) continue;    // nothing there or expected
        if (bsem_wait(psem_ptr(h, B), 1, 1, NoSpin()) == kAcquired) {
            uint64_t ch;
            uint64_t pm = page_claim(h, B, 1, &ch);
            uint64_t p = ch * kChunkPages + (uint64_t)(__ffsll((long long)pm) - 1);
            bin_init(h, p, B, c, 1);
            stat_add(h, kStatBinGrow, 1);
            bsem_signal(sem_ptr(h, B, c), slots - 1, 0);
            return p << kPageShift;
        }
    }
    for (uint32_t t = 1; t <= h->n_arenas; t++) {
        uint32_t B = (A0 + t) % h->n_arenas;
        uint64_t cw = ld_rlx(sem_ptr(h, B, c));
        if (sem_C(cw) < 1 && (int64_t)sem_C(cw) + sem_D(cw) < 1) continue;
        if (bsem_wait(sem_ptr(h, B, c), 1, 1, NoSpin()) == kAcquired) return bin_claim_one(h, B, c);
    }
    stat_add(h, kStatFail, 1);
    return kNull;
}

// ---- bins: collective claim of one slot per lane (units already acquired) ----
// Lanes spread over the chunk's non-full pages by their rank (each thread walks
// the number of elements its index dictates), lanes that picked
// the same page regroup and that page gets ONE atomicOr for all of them.
static __device__ __noinline__ uint64_t bin_claim_collective(const ga_desc* h, unsigned grp, uint32_t A, int c,
                                                             uint64_t pre_ch = 0, uint64_t pre_m = 0) {
    const uint32_t lane = lane_id();
    const uint64_t csz = 16ull << c;
    // per-warp rotation of the page and word starts: the warps of an SM share
    // the arena, so without it they all pile onto the first non-full page
    uint32_t wid; asm volatile("mov.u32 %0, %%warpid;" : "=r"(wid));
    const uint32_t rot = hash32(wid ^ (smid() << 6));
    uint64_t my = kNull;
    uint32_t it = 0;                                        // retries move on to the next page
    unsigned unsat = grp;                                   // lanes still without a slot (this lane included)
    uint64_t ch = 0, m = 0;                                 // the chunk under claim and its non-full pages
    GA_DBG_CNT;
#if GA_COUNT_ITERS
    if ((int)lane_id() == __ffs(grp) - 1) stat_add(h, kStatRepairNonfull, 1);      // calls (diagnostic build)
#endif
    for (;;) {
        SPIN_NOTE(dbg_cnt, 10, ((uint64_t)A << 8) | c, unsat);
        const int L = __ffs(unsat) - 1;
#if GA_COUNT_ITERS
        if ((int)lane_id() == L) stat_add(h, kStatRepairSummary, 1);               // iterations
#endif
#if GA_CLAIM_LOCALMASK
        if (m == 0) {                                       // uniform over the group
#else
        {
            ch = 0; m = 0;
#endif
            if ((int)lane == L) {
                if (pre_m) { ch = pre_ch; m = pre_m; pre_m = 0; }                   // loaded beside the semaphore
                else if (is_span(c)) ch = span_find_word(h, A, c, &m);              // spans: a summary word
                else ch = bin_find_chunk(h, A, c, &m);
            }
            ch = __shfl_sync(unsat, ch, L);
            m = __shfl_sync(unsat, m, L);
        }
        const uint32_t q = __popc(unsat & lanemask_lt());
        const uint32_t np = __popcll(m);
        uint64_t page = (ch << kChunkShift) + nth_set(m, ((q >> per_page_shift(c)) + rot + it++) % np);
        if (is_span(c)) page <<= kChunkShift;                  // spans: summary word -> span head page
        const unsigned pg = __match_any_sync(unsat, page);
        const int pl = __ffs(pg) - 1;
        uint64_t got = 0;
        int wi = 0;
        if ((int)lane == pl) {
            got = bin_claim_page(h, page, A, c, __popc(pg), &wi, rot >> 8);
            if (!got && is_span(c))                            // a full or stale span: drop its summary bit
                hb3_clear_owned(h, arena_hb(h, A, kAhbNfc + c), page >> kChunkShift, A,
                                nonfull_word(h, page >> kChunkShift, c), 0);
        }
        got = __shfl_sync(pg, got, pl);
        wi = __shfl_sync(pg, wi, pl);
        const uint32_t pr = __popc(pg & lanemask_lt());
        if (pr < (uint32_t)__popcll(got)) my = (page << kPageShift) + (uint64_t)(wi * 64 + nth_set(got, pr)) * csz;
#if GA_CLAIM_LOCALMASK
        {   // pages that came up short leave the group's local copy of the chunk's
            // non-full mask: retries go to the other pages before a new search
            const uint64_t drop = my == kNull ? 1ull << (page & (kChunkPages - 1)) : 0ull;
            m &= ~(((uint64_t)__reduce_or_sync(unsat, (uint32_t)(drop >> 32)) << 32) |
                   __reduce_or_sync(unsat, (uint32_t)drop));
        }
#endif
        unsat = lanes_where(unsat, my == kNull);
        if (my != kNull) break;                             // a satisfied lane leaves the group
    }
    return my;
}

// ---- bins: collective growth (class semaphore said GROW for the group) ------
// The leader accounts ceil(N/slots) pages on the arena page semaphore and
// tracks them one chunk at a time (one atomicOr claims several pages: the
// collective chunk-list split of P:L1282-1292); every lane computes its page
// and slot, the first lane of each page initialises that bin, then the leader
// publishes the spare slots with one signal.  Returns kNull for every lane if
// the group could not grow (the caller degrades to per-lane waits).
static __device__ __noinline__ uint64_t bin_grow_collective(const ga_desc* h, unsigned grp, uint32_t A, int c) {
    const uint32_t lane = lane_id();
    const int leader = __ffs(grp) - 1;
    const uint32_t N = __popc(grp), rank = __popc(grp & lanemask_lt());
    const uint32_t slots = slots_of(c);
    const uint32_t Bp = slots * ((N + slots - 1) / slots);                 // R-8
    const uint32_t k = Bp / slots;
    const uint64_t csz = 16ull << c;
    uint64_t my = kNull;
    int mode = 0;                                                            // 0 claim pages, 1 fresh chunk, -1 fail
    uint64_t ch = 0, pm = 0;
    if ((int)lane == leader) {
        if (bsem_wait(psem_ptr(h, A), k, kChunkPages, ArenaSpin{h, A}) == kGrow) {
            reclaim_arena(h, A, -1, kReclaimKeep);                           // delegated work first
            int64_t nc = chunk_acquire(h, A, k);
            if (nc < 0) {
                bsem_signal(psem_ptr(h, A), 0, kChunkPages - k);
                bsem_signal(sem_ptr(h, A, c), 0, Bp - N);
                mode = -1;
            } else {
                bsem_signal(psem_ptr(h, A), kChunkPages - k, kChunkPages - k);
                mode = 1; ch = (uint64_t)nc; pm = k >= 64 ? ~0ull : ((1ull << k) - 1);
            }
        }
    }
    mode = __shfl_sync(grp, mode, leader);
    if (mode < 0) return kNull;
    uint32_t served = 0, pages_left = k;
    uint64_t last_page = 0;
    while (pages_left) {
        if (mode == 0 && (int)lane == leader) pm = page_claim(h, A, (int)pages_left, &ch);
        ch = __shfl_sync(grp, ch, leader);
        pm = __shfl_sync(grp, pm, leader);
        const uint32_t np = __popcll(pm);
        const uint32_t cap = np * slots;
        if (rank >= served && rank < served + cap) {
            const uint32_t r = rank - served;
            const uint64_t p = ch * kChunkPages + nth_set(pm, r / slots);
            my = (p << kPageShift) + (uint64_t)(r % slots) * csz;
            if (r % slots == 0) {
                const uint32_t left = N - served - (r / slots) * slots;
                bin_init(h, p, A, c, left < slots ? left : slots);
            }
        }
        last_page = ch * kChunkPages + nth_set(pm, np - 1);
        served += cap < N - served ? cap : N - served;
        pages_left -= np;
        mode = 0;
    }
    warp_release(grp);
    if ((int)lane == leader) {
        stat_add(h, kStatBinGrow, k);
        st_rlx32(&h->hint[A * kNcls + c], (uint32_t)last_page);
        bsem_signal(sem_ptr(h, A, c), Bp - N, Bp - N);                      // release: bins are initialised
    }
    return my;
}

// ---- spans: collective growth (class semaphore said GROW for the group) ------
// ceil(N/slots) fresh chunks straight from TBuddy, one at a time: the leader
// takes a chunk, lanes [served, served + take) get its slots and the first of
// them initialises the span.  If the tree runs dry the lanes served so far
// keep their slots, the others get kNull (the caller degrades them to per-lane
// waits) and the unproduced units are retracted (signal(0, B'-N)).
static __device__ __noinline__ uint64_t tree_malloc_group(const ga_desc* h, unsigned grp, int o);
static __device__ __noinline__ uint64_t span_grow_collective(const ga_desc* h, unsigned grp, uint32_t A, int c) {
    const uint32_t lane = lane_id();
    const int leader = __ffs(grp) - 1;
    const uint32_t N = __popc(grp), rank = __popc(grp & lanemask_lt());
    const uint32_t slots = slots_of(c);
    const uint32_t Bp = slots * ((N + slots - 1) / slots);                 // R-8
    const uint64_t csz = 16ull << c;
    uint64_t my = kNull;
    const uint32_t k = Bp / slots;
    if ((int)lane == leader) reclaim_arena(h, A, -1, kReclaimKeep);           // delegated work first
    if (k > 1) {
        // All k chunks in ONE collective TBuddy claim (tree_malloc_group: one
        // semaphore wait per level and up to 64 nodes per bitmap atomic, the
        // collective critical section of) instead of k climbs.
        // All-or-nothing: if the tree cannot serve k at once nothing was taken
        // and the chunk-at-a-time loop below runs.
        const unsigned sub = lanes_where(grp, rank < k);
        int64_t mych = -1;
        if (rank < k) {
            const uint64_t off = tree_malloc_group(h, sub, kChunkOrder);
            if (off != kNull) {
                mych = (int64_t)(off >> (kPageShift + kChunkShift));
                st_rlx32(&h->chunk_owner[mych], A + 1);
                stat_add(h, kStatChunkGrow, 1);
            }
        }
        if (__all_sync(grp, rank >= k || mych >= 0)) {
            const uint32_t j = rank / slots, r = rank % slots;
            const int64_t chj = __shfl_sync(grp, mych, (int)nth_set(grp, j));    // span j: the j-th lane's chunk
            const uint64_t p = (uint64_t)chj * kChunkPages;
            my = (p << kPageShift) + (uint64_t)r * csz;
            if (r == 0) bin_init(h, p, A, c, N - j * slots < slots ? N - j * slots : slots);
            warp_release(grp);
            if ((int)lane == leader) {
                stat_add(h, kStatBinGrow, k);
                st_rlx32(&h->hint[A * kNcls + c], (uint32_t)p);
                bsem_signal(sem_ptr(h, A, c), Bp - N, Bp - N);                  // release: spans initialised
            }
            return my;
        }
    }
    uint32_t served = 0;
    int64_t ch = 0;
    while (served < N) {
        if ((int)lane == leader) ch = span_acquire(h, A);
        ch = __shfl_sync(grp, ch, leader);
        if (ch < 0) break;
        const uint32_t take = N - served < slots ? N - served : slots;
        const uint64_t p = (uint64_t)ch * kChunkPages;
        if (rank >= served && rank < served + take) {
            const uint32_t r = rank - served;
            my = (p << kPageShift) + (uint64_t)r * csz;
            if (r == 0) bin_init(h, p, A, c, take);
        }
        served += take;
    }
    warp_release(grp);
    if ((int)lane == leader) {
        stat_add(h, kStatBinGrow, (served + slots - 1) / slots);
        if (ch >= 0) {
            st_rlx32(&h->hint[A * kNcls + c], (uint32_t)((uint64_t)ch * kChunkPages));
            bsem_signal(sem_ptr(h, A, c), Bp - N, Bp - N);                  // release: spans initialised
        } else {
            bsem_signal(sem_ptr(h, A, c), 0, Bp - N);                       // failure
        }
    }
    return my;
}

// ---- TBuddy, group path -------------------------------------------------------
// One bulk wait of N units per order for the group (batch 2, B' = 2*ceil(N/2));
// on GROW the group climbs with N_{k+1} = ceil(N_k / 2), claims N_m nodes at the
// granting level m and splits them down: each claimed node serves 2^(m-o)
// lanes, the unused right parts of the last node are published.  Returns kNull
// for every lane if the tree could not serve the whole group.
static __device__ __noinline__ uint64_t tree_malloc_group(const ga_desc* h, unsigned grp, int o) {
    const uint32_t lane = lane_id();
    const int leader = __ffs(grp) - 1;
    const uint32_t N = __popc(grp), rank = __popc(grp & lanemask_lt());
    int m = o;
    uint32_t Nm = N;
    if ((int)lane == leader) {
        uint32_t ns = 128;
        for (int attempt = 0;; attempt++) {
            m = o; Nm = N;
            for (;;) {
                if (m > (int)h->L) {                         // nothing to grow from: retract every E
                    uint32_t nk = N;
                    for (int k = o; k < m; k++) { bsem_signal(tsem_ptr(h, k), 0, 2 * ((nk + 1) >> 1) - nk); nk = (nk + 1) >> 1; }
                    m = -1;
                    break;
                }
                if (bsem_wait_fast(tsem_ptr(h, m), Nm, 2 * ((Nm + 1) >> 1), NoSpin()) == kAcquired) break;
                Nm = (Nm + 1) >> 1;
                m++;
            }
            // No false resource starvation: while splits are in flight
            // (cold start) or units are visible at some order >= o, re-climb
            if (m >= 0 || attempt >= 8 || !tree_has_supply(h, o, attempt < 2)) break;
            __nanosleep(ns); if (ns < 8192) ns <<= 1;
        }
    }
    m = __shfl_sync(grp, m, leader);
    if (m < 0) return kNull;
    if ((int)lane == leader) reserve_add(h, (int64_t)N << o);
    Nm = __shfl_sync(grp, Nm, leader);
    const int s = m - o;
    uint64_t my = kNull;
    uint32_t served = 0;
    uint32_t seed = scatter_seed();
    while (served < N) {
        uint64_t wj = 0, got = 0;
        if ((int)lane == leader) got = tree_claim_word(h, m, (int)(Nm - (served >> s)), seed, &wj);
        wj = __shfl_sync(grp, wj, leader);
        got = __shfl_sync(grp, got, leader);
        {
            const uint32_t nn = __popcll(got), rem = N - served;
            if ((nn << s) >= rem && s > 0) {
                // the last node is split: its unused right parts [pos, 2^s) decompose into
                // one aligned block per set bit j of the running position (E at each level
                // o + j); the group's lanes publish them in parallel, lane q doing level o + q
                const uint64_t xlast = wj * 64 + (63 - __clzll((long long)got));
                const uint64_t keep = rem - ((nn - 1) << s);
                for (uint32_t j = rank; j < (uint32_t)s; j += N) {
                    // running position before level j = keep rounded up to a multiple of 2^j
                    const uint64_t pj = (keep + (1ull << j) - 1) & ~((1ull << j) - 1);
                    if ((pj >> j) & 1) tree_publish(h, o + (int)j, ((xlast << s) + pj) >> j, 1);
                }
            }
        }
        const uint32_t cap = (uint32_t)__popcll(got) << s;
        if (rank >= served && rank < served + cap) {
            const uint32_t r = rank - served;
            const uint64_t x = wj * 64 + nth_set(got, r >> s);
            const uint64_t pg = ((x << s) + (r & ((1u << s) - 1))) << o;
            st_rlx32(&h->kind[pg], kKindTree | (uint32_t)o);
            my = pg << kPageShift;
        }
        served += cap < N - served ? cap : N - served;
    }
    // Every right part is published before any lane returns its block: a lane
    // that frees its block at once must find the split's other halves already
    // Available, or its merge (tree_free's CAS on the sibling word, R-21) would
    // mark it Available beside a buddy published a moment later -- two
    // Available siblings (found by tests/test_gpu_edge.py on the GA_NSPAN=0 build).
    warp_release(grp);
    return my;
}

// ---- malloc of a bin / span class in one arena, and the group fallback --------
static __device__ __forceinline__ uint64_t* arena_ctr(const ga_desc* h, int i) { return h->actr + arena_of(h) * kActrStride + i; }
// malloc of class c (bin or span) for the lanes of grp in arena A: Alg. 1 wait,
// then the collective claim or growth.  Lanes it could not serve get kNull.
// pre_ch / pre_m: a chunk and its non-full mask the leader loaded beside the
// fetch-add (pre_m == 0: none).
static __device__ __forceinline__ uint64_t malloc_in_arena(const ga_desc* h, unsigned grp, uint32_t A, int c,
                                                           bool prefetch) {
    const uint32_t lane = lane_id();
    const int leader = __ffs(grp) - 1;
    const uint32_t N = __popc(grp);
    const uint32_t slots = slots_of(c);
    const uint32_t Bp = slots * ((N + slots - 1) / slots);                         // R-8
    int r = kAcquired;
    uint64_t w = 0, pre_ch = 0, pre_m = 0;
    if ((int)lane == leader) {
        uint64_t* sp = sem_ptr(h, A, c);
        const uint32_t hp = GA_PREFETCH && prefetch ? s_chunk_hint[c] : 0xFFFFFFFFu;
        const uint64_t old = a_add(sp, dCD(-(int32_t)N, (int32_t)Bp));           // Alg. 1, first fetch-add
        uint32_t own = 0;
        if (hp < h->pages) {                                                     // in flight with the fetch-add
            pre_ch = hp >> kChunkShift;
            own = ld_rlx32(&h->chunk_owner[pre_ch]);
            pre_m = ld_rlx(nonfull_word(h, pre_ch, c));
            if (is_span(c)) own = 0;                              // spans claim over summary words
        }
        r = bsem_decide(sp, old, N, Bp, &w);
        if (r == kBlocked) r = bsem_wait_slow<2048>(sp, N, Bp, ArenaSpin{h, A}, w);
        if (own != A + 1) pre_m = 0;
    }
    r = __shfl_sync(grp, r, leader);
    return r == kAcquired ? bin_claim_collective(h, grp, A, c, pre_ch, pre_m)
         : is_span(c) ? span_grow_collective(h, grp, A, c) : bin_grow_collective(h, grp, A, c);
}

#ifndef GA_LOCKSTEP
#define GA_LOCKSTEP 1            // 1: the bin/span fast path runs every class group of a warp in one instruction stream
#endif
// The bin / span fast path with every class group of the warp in ONE
// instruction stream.  malloc_in_arena runs a group at a time: on a mixed
// trace a warp holds ~12 class groups, and under independent thread
// scheduling they issued their own copies of the claim loop one after the
// other (4.1 active lanes per instruction, ~4,700 warp instructions per
// warp-call).  Here the control flow is uniform over `bl` (every bin/span
// lane of the call): leaders issue their Alg. 1 fetch-adds as one
// instruction, per-group values travel by shuffles from each lane's own group
// leader, and the claim loop runs while ANY lane of the warp still needs a
// slot -- so the groups' L2 round trips overlap instead of adding up.  The
// per-group work is exactly malloc_in_arena's (one wait of N units per group,
// collective claim by rank over the chunk's non-full pages, one atomicOr per
// page word); only the schedule differs.  Groups whose wait
// blocks or says GROW take the per-group path afterwards.
#ifndef GA_FIND_NOINL
#define GA_FIND_NOINL 0          // 1: the lockstep loop's chunk search out of line (smaller loop code)
#endif
#if GA_FIND_NOINL
#define GA_FIND_FN __noinline__
#else
#define GA_FIND_FN __forceinline__
#endif
// The chunk (bins) or summary word (spans) a lockstep iteration claims from,
// when nothing was loaded beside the semaphore.
static __device__ GA_FIND_FN uint64_t lockstep_find(const ga_desc* h, uint32_t A, int c, uint32_t it, uint32_t rot,
                                                     uint64_t* m) {
    if (is_span(c)) return span_find_word(h, A, c, m);
    if (GA_SPREAD && it > 0) return bin_spread_chunk(h, A, c, rot + it, m);
    return bin_find_chunk(h, A, c, m);
}
// A group whose wait did not grant at once: a blocked wait (reservation taken
// by bsem_decide, re-polled from a fresh load), then the claim or growth.
// Out of line: rare, and its state would otherwise stay live (and spill)
// across the lockstep loop.
static __device__ __noinline__ uint64_t malloc_group_slow(const ga_desc* h, unsigned grp, uint32_t A, int c, int r) {
    const uint32_t N = __popc(grp), slots = slots_of(c);
    const uint32_t Bp = slots * ((N + slots - 1) / slots);                         // R-8
    const int leader = __ffs(grp) - 1;
    if ((int)lane_id() == leader && r == kBlocked) {
        uint64_t* sp = sem_ptr(h, A, c);
        r = bsem_wait_slow<2048>(sp, N, Bp, ArenaSpin{h, A}, ld_rlx(sp));
    }
    r = __shfl_sync(grp, r, leader);
    return r == kAcquired ? bin_claim_collective(h, grp, A, c)
         : is_span(c) ? span_grow_collective(h, grp, A, c) : bin_grow_collective(h, grp, A, c);
}
// held: the group's units were already acquired for it (the block / cluster
// collective's one wait per class, section 8): no fetch-add here.
static __device__ __forceinline__ uint64_t malloc_lockstep(const ga_desc* h, unsigned bl, unsigned grp, int c,
                                                           uint32_t A, bool held = false) {
    const uint32_t lane = lane_id();
    const int leader = __ffs(grp) - 1;
    int r = kAcquired;
    uint64_t pre_m = 0;
    uint32_t hp = 0;
    if ((int)lane == leader) {
        const uint32_t N = __popc(grp), slots = slots_of(c);
        const uint32_t Bp = slots * ((N + slots - 1) / slots);                     // R-8
        uint64_t* sp = sem_ptr(h, A, c);
        uint64_t w;
        hp = GA_PREFETCH ? s_chunk_hint[c] : 0xFFFFFFFFu;
        const uint64_t old = held ? 0 : a_add(sp, dCD(-(int32_t)N, (int32_t)Bp)); // Alg. 1, first fetch-add
        uint32_t own = 0;
        if (hp < h->pages) {                                                     // in flight with the fetch-add
            if (is_span(c)) {                                                    // spans: the hint's summary word
                own = A + 1;
                pre_m = ld_rlx(&arena_hb(h, A, kAhbNfc + c).w0[hp >> (2 * kChunkShift)]);
            } else {
                own = ld_rlx32(&h->chunk_owner[hp >> kChunkShift]);
                pre_m = ld_rlx(nonfull_word(h, hp >> kChunkShift, c));
            }
        }
        if (!held) r = bsem_decide(sp, old, N, Bp, &w);
        if (own != A + 1) pre_m = 0;
    }
    r = __shfl_sync(bl, r, leader);
    uint32_t wid; asm volatile("mov.u32 %0, %%warpid;" : "=r"(wid));
    const uint32_t rot = hash32(wid ^ (smid() << 6));
    uint64_t my = kNull;
    bool need = r == kAcquired;
    bool checked = false;                                      // GA_DEFER_RECHECK: my slot's incarnation validated
#if GA_COUNT_ITERS
    if ((int)lane == __ffs(bl) - 1) stat_add(h, kStatRepairNonfull, 1);                // lockstep calls (diagnostic)
#endif
    for (uint32_t it = 0;; it++) {
        const unsigned un = __ballot_sync(bl, need);
        if (un == 0) break;
#if GA_COUNT_ITERS
        if ((int)lane == __ffs(bl) - 1) stat_add(h, kStatRepairSummary, 1);           // warp iterations
#endif
        const unsigned g = grp & un;                           // my group's lanes still without a slot
        const int L = need ? __ffs(g) - 1 : (int)lane;
        uint64_t ch = 0, m = 0;
        if (need && (int)lane == L) {
            if (pre_m) { ch = hp >> (is_span(c) ? 2 * kChunkShift : kChunkShift); m = pre_m; pre_m = 0; }   // loaded beside the semaphore
            else ch = lockstep_find(h, A, c, it, rot, &m);
        }
        ch = __shfl_sync(bl, ch, L);
        m = __shfl_sync(bl, m, L);
        uint64_t key = kNull;
        uint64_t page = 0;
        if (need) {
            const uint32_t q = __popc(g & lanemask_lt());
            // bins: page of chunk ch; spans: head page of chunk 64 * ch + bit (span_find_word)
            // spans start at the word's lowest span for every warp (GA_SPAN_ROT=0):
            // spreading warps over the word's spans left more spans partly
            // filled (d4 fragmentation 1.13x -> 1.24x the oracle's)
            const uint32_t r0 = (is_span(c) && !GA_SPAN_ROT) ? 0u : rot;
            page = (ch << kChunkShift) + nth_set(m, ((q >> per_page_shift(c)) + r0 + it) % (uint32_t)__popcll(m));
            if (is_span(c)) page <<= kChunkShift;
            key = (page << 4) | (uint64_t)c;                   // a stale bit can name one page in two classes
        }
        const unsigned pg = __match_any_sync(bl, key);
        const int pl = __ffs(pg) - 1;
        uint64_t got = 0;
        int wi = 0;
        if (need && (int)lane == pl) {
            got = bin_claim_page(h, page, A, c, __popc(pg), &wi, rot >> 8, !GA_DEFER_RECHECK);
            if (!got && is_span(c)) {                          // a full or stale span: drop its summary bit
                // A full span was already dropped by the claim (nonfull_clear_if_full);
                // only a STALE summary bit (the chunk's non-full word already
                // empty, or the chunk no longer A's) needs the clear-then-recheck.
                const uint64_t ch = page >> kChunkShift;
                HB3 nb = arena_hb(h, A, kAhbNfc + c);
                if (!GA_SPAN_CLEAR_CHECK ||
                    ((ld_rlx(&nb.w0[ch >> 6]) >> (ch & 63)) & 1 &&
                     (ld_rlx(nonfull_word(h, ch, c)) == 0 || ld_rlx32(&h->chunk_owner[ch]) != A + 1)))
                    hb3_clear_owned(h, nb, ch, A, nonfull_word(h, ch, c), 0);
            }
        }
        got = __shfl_sync(bl, got, pl);
        wi = __shfl_sync(bl, wi, pl);
        if (need) {
            const uint32_t pr = __popc(pg & lanemask_lt());
            if (pr < (uint32_t)__popcll(got)) {
                my = (page << kPageShift) + ((uint64_t)(wi * 64 + nth_set(got, pr)) << (c + kMinShift));
                need = false;
            }
        }
#if GA_DEFER_RECHECK
        if (__ballot_sync(bl, need) == 0) {
            // Every lane holds a slot: validate them all at once (one parallel
            // round trip instead of one per iteration).  A slot taken in a page
            // recycled between the claimer's kind read and its atomicOr (ABA)
            // belongs to another incarnation; while we hold the bit that
            // incarnation cannot be reclaimed, so the kind read now decides
            // (as the immediate recheck did): give the slot back, re-publish
            // the page for its owner, and claim again.
            bool bad = false;
            if (my != kNull && !checked) {
                const uint64_t pg0 = bin_head(my >> kPageShift, c);
                const uint32_t k2 = ld_rlx32(&h->kind[pg0]);
                if (k2 != kind_bin(A, c)) {
                    const uint32_t slot = (uint32_t)((my - (pg0 << kPageShift)) >> (c + kMinShift));
                    a_and(&page_bits(h, pg0)[slot >> 6], ~(1ull << (slot & 63)));
                    if ((k2 & 0xC0000000u) == kKindBin) {
                        nonfull_set(h, pg0, (int)(k2 & 0xFF), (k2 >> 8) & 0xFFFFu);
                        mark_candidate(h, pg0, (k2 >> 8) & 0xFFFFu);
                    }
                    my = kNull;
                    need = true;
                    bad = true;
                }
            }
            checked = !bad && my != kNull;
            if (!__any_sync(bl, bad)) break;
        }
#endif
    }
    if (r != kAcquired) my = malloc_group_slow(h, grp, A, c, r);    // per group: blocked wait, growth
    return my;
}

// The group-level fallback (R-26: a malloc fails only if no arena
// can serve it).  The group's own arena could not grow (the tree is empty).
// Delegated reclamation is drained once, then the group's lanes scan every
// arena's class and page semaphores in parallel (one load each per lane) and
// take the richest arena, where the group runs the normal sequence; repeat for
// the lanes still unserved.  When no arena shows units, pages or a growth in
// flight and the tree has no chunk, the group fails at once -- no per-lane
// scans.  A group that keeps missing for other reasons ends in the exact
// per-lane path (bin_malloc_lane).
static __device__ __noinline__ uint64_t group_fallback(const ga_desc* h, unsigned grp, uint32_t A0, int c) {
    const uint32_t lane = lane_id();
    reclaim_arenas(h, __popc(grp & lanemask_lt()), __popc(grp));                 // P:L1206-1244, lanes in parallel
    (void)__shfl_sync(grp, 0, __ffs(grp) - 1);
    const bool span = is_span(c);
    const uint32_t nA = (h->n_arenas + class_share(c) - 1) / class_share(c);     // arenas of class c
    uint64_t my = kNull;
    unsigned rest = grp;
    bool seen_nothing = false;
    for (int tries = 0; tries < 32; tries++) {
        const uint32_t n = __popc(rest), q = __popc(rest & lanemask_lt());
        const int L = __ffs(rest) - 1;
        uint32_t best = 0;                                                       // units << 8 | arena
        for (uint32_t B = q; B < nA; B += n) {
            const uint64_t sw = ld_rlx(sem_ptr(h, B, c));
            int64_t units = sem_C(sw) > 0 ? sem_C(sw) : 0;
            if (!span) {
                const uint64_t pw = ld_rlx(psem_ptr(h, B));
                units += (int64_t)(sem_C(pw) > 0 ? sem_C(pw) : 0) * slots_of(c);
            }
            const uint32_t pk = ((uint32_t)(units < 0xFFFFFF ? units : 0xFFFFFF) << 8) | B;
            best = pk > best ? pk : best;
        }
        best = __reduce_max_sync(rest, best);
        uint32_t target;
        if (best >> 8) {
            target = best & 0xFF;                                                // an arena with units or pages
        } else {
            // No arena shows units or pages.  The tree may still supply a chunk
            // (grow at home), or a split may be publishing one (count_growth).
            int t = 0;
            if ((int)lane == L) t = tree_has_supply(h, kChunkOrder, false) ? 2 : tree_has_supply(h, kChunkOrder, true) ? 1 : 0;
            t = __shfl_sync(rest, t, L);
            if (t == 2) target = A0;
            else if (t == 1 || !seen_nothing) {
                // a split in flight, or a grower that already holds its pages and
                // is about to publish: look again once it had time to finish
                seen_nothing = t == 0;
                __nanosleep(8192);
                continue;
            } else {
                if ((int)lane == L) stat_add(h, kStatFail, __popc(rest));
                return kNull;                                                    // nothing anywhere: fail
            }
        }
        seen_nothing = false;
        my = malloc_in_arena(h, rest, target, c, false);
        rest = lanes_where(rest, my == kNull);
        if (my != kNull) return my;
    }
    // still unserved after many rounds: the exact per-lane path (R-26, R-27)
    return bin_malloc_lane(h, A0, c);
}

// ---- the entry points ---------------------------------------------------------
// malloc.  Lanes are grouped by size class (__match_any_sync); one leader per
// group runs Alg. 1's fetch-add for the group's N units and, in the same round
// trip, loads the block's hinted chunk for the class (owner and non-full mask,
// from a shared-memory hint), which the collective claim starts from.  Lanes
// the arena cannot serve take the group fallback (R-26, R-27).
static __device__ __noinline__ uint64_t ga_malloc_off(const ga_desc* h, uint64_t n) {
    const unsigned act = active_lanes();
    const uint32_t lane = lane_id();
    if ((int)lane == __ffs(act) - 1) red_rlx(arena_ctr(h, 0), __popc(act));       // n_malloc, per warp
    const int key = size_key(h, n);
    const unsigned grp = __match_any_sync(act, key);
#if GA_LOCKSTEP
    const unsigned bl = __match_any_sync(act, (unsigned)(key >= 0 && key < kNcls));   // valid in bin/span lanes
#endif
    if (key < 0) return kNull;
    uint64_t my;
    if (key < kNcls) {
        const uint32_t A = arena_of(h) / class_share(key);
#if GA_LOCKSTEP
        my = malloc_lockstep(h, bl, grp, key, A);
        // my group's unserved lanes, as a match on the uniform mask bl (see
        // group_or and active_lanes: no ballot result as a _sync mask)
        const unsigned rest = __match_any_sync(bl, ((unsigned)key << 1) | (unsigned)(my == kNull));
#else
        my = malloc_in_arena(h, grp, A, key, true);
        const unsigned rest = lanes_where(grp, my == kNull);
#endif
        if (my == kNull) {
            if ((int)lane == __ffs(rest) - 1) stat_add(h, kStatFallback, 1);
            my = group_fallback(h, rest, A, key);
        }
        return my;
    }
    const int o = key - kNcls;
    my = tree_malloc_group(h, grp, o);
    if (my == kNull) {
        int64_t x = tree_alloc_one_retry(h, o, false);
        if (x >= 0) {
            uint64_t pgt = (uint64_t)x << o;
            st_rlx32(&h->kind[pgt], kKindTree | (uint32_t)o);
            my = pgt << kPageShift;
        } else stat_add(h, kStatFail, 1);
    }
    return my;
}

// free: TBuddy blocks merge inside the warp first (lanes freeing sibling blocks
// pair up with __match_any_sync and continue with the parent -- a collective
// free), then each surviving block runs the merge-on-free protocol; bin slots
// are grouped per bitmap word (one atomicAnd) and per (arena, class) (one signal).
struct CollState;
static __device__ __forceinline__ void coll_signal(const ga_desc* h, CollState* R, uint32_t A, int c, uint32_t n);
template <bool kColl>
static __device__ __forceinline__ void free_body(const ga_desc* h, uint64_t off, CollState* R) {
    const unsigned act = active_lanes();
    uint32_t k = 0;
    uint64_t p = 0;
    if (off != kNull) { p = off >> kPageShift; k = ld_rlx32(&h->kind[p]); }
    const bool is_bin = (off != kNull) && ((k & 0xC0000000u) == kKindBin);
    const bool is_tree = (off != kNull) && !is_bin;
    const unsigned same = __match_any_sync(act, is_bin ? 1u : is_tree ? 2u : 0u);
    const unsigned bins = is_bin ? same : 0u, trees = is_tree ? same : 0u;      // valid in their own lanes
    if ((int)lane_id() == __ffs(same) - 1 && (is_bin || is_tree)) red_rlx(arena_ctr(h, 1), __popc(same));   // n_free
    if (is_tree) {
        int n = (int)(k & 0xFF);                               // order from the page kind (R-18)
        uint64_t x = p >> n;
        st_rlx32(&h->kind[p], 0);
        fence();
        unsigned part = trees;
        bool alive = true;
        for (;;) {
            const uint64_t key = ((uint64_t)n << 58) | (x >> 1);
            const unsigned mm = __match_any_sync(part, key);
            const bool paired = __popc(mm) == 2;
            if (!__any_sync(part, paired)) break;
            if (paired) {
                if ((int)lane_id() == __ffs(mm) - 1) { x >>= 1; n++; }   // both halves are ours: merged
                else alive = false;
            }
            part = lanes_where(part, alive);
            if (!alive) break;
        }
        if (alive) tree_free(h, n, x);
        return;
    }
    if (!is_bin) return;
    const uint32_t A = (k >> 8) & 0xFFFFu;
    const int c = (int)(k & 0xFF);
    p = bin_head(p, c);                                        // spans: bitmap at the chunk's first page
    const uint32_t slot = (uint32_t)((off - (p << kPageShift)) >> (c + kMinShift));
    const int w = (int)(slot >> 6);
    const unsigned g1 = __match_any_sync(bins, (p << 2) | (uint64_t)w);
    const uint64_t bit = 1ull << (slot & 63);
    const uint64_t mask = group_or(bins, g1, bit);
    bool eager = false;
    if ((int)lane_id() == __ffs(g1) - 1) {
        uint64_t* bw = page_bits(h, p);
        const uint64_t old = a_and(&bw[w], ~mask);
        const uint64_t v = valid_mask(c, w);
        if ((old | ~v) == ~0ull) nonfull_set(h, p, c, A);     // the word was full: bin back in the list
        if (((old & ~mask) & v) == 0) {                        // this word is empty: is the bin?
            uint64_t ww[4];
            ld_bitmap(bw, ww);
            bool empty = true;
#pragma unroll
            for (int i = 0; i < 4; i++) if (i < words_of(c) && (ww[i] & valid_mask(c, i))) empty = false;
            if (empty) {
                // reclaim after the signal below: always (GA_SPAN_EAGER), or
                // once the heap is nearly all reserved (deferred reclamation
                // keeps empty spans -- whole chunks -- with their arena until a
                // grower or waiter drains them: the d4 fragmentation excess,
                // and failed calls at the exhaust level)
                if (is_span(c) && (GA_SPAN_EAGER || ld_rlx(&h->stats[kStatReserved]) * 10 > h->pages * GA_EAGER_AT))
                    eager = true;
                else mark_candidate(h, p, A);
            }
        }
    }
    // the match is also the execution barrier: every leader's atomicAnd above
    // has returned (performed at L2) before any lane of `bins` passes it, so
    // the units signalled below never precede their slots (no __syncwarp: see
    // active_lanes)
    const unsigned g2 = __match_any_sync(bins, (A << 4) | (uint32_t)c);     // class < 16
    if ((int)lane_id() == __ffs(g2) - 1) {
        if (kColl) coll_signal(h, R, A, c, __popc(g2));       // block / cluster: one signal per class later
        else bsem_signal_after_rmw(sem_ptr(h, A, c), __popc(g2));
    }
    if (eager) {
        fence();                                               // our slots' units are published
        if (!bin_reclaim(h, p, slots_of(c))) mark_candidate(h, p, A);
    }
}
static __device__ __noinline__ void ga_free_off(const ga_desc* h, uint64_t off) { free_body<false>(h, off, nullptr); }


// ---------------------------------------------------------------------------
// 8. block- and cluster-collective entry points.  The paper's
// collective synchronization primitives work at thread-block scope (Sec.
// 4.2.2): the threads of a block enter one critical section
// together, one elected thread performs the synchronization operation for all
// ("collective acquire": elected acquire + barrier; "collective release":
// barrier + elected release).  Here EVERY thread of the CTA (block scope) or
// of the thread-block cluster (cluster scope, CTAs joined through distributed
// shared memory) calls ga_malloc_block / ga_malloc_cluster together, like
// __syncthreads():
//   1. each warp's class groups add their demand to per-class counters in the
//      collective's shared memory (the root CTA's, through DSMEM for a
//      cluster);
//   2. one barrier; then ONE thread per class runs Alg. 1 for the whole
//      collective's demand of that class -- one semaphore fetch-add for up to
//      kCollMax threads instead of one per warp group (collective acquire);
//   3. a second barrier; every warp claims its slots through the lockstep
//      claim with the units already held (one atomicOr per bitmap word).
// A wait that says GROW is retracted (signal(0, B'-N)) and the
// groups of that class run their own waits and growth (the warp path).
// ga_free_block / ga_free_cluster free through the warp path and add the
// released units of the collective's own arena to per-class counters; after
// one barrier the root CTA issues ONE signal per class (collective release).
// TBuddy sizes (above 64 KiB) take the warp path.  The counters are
// double-buffered by a parity word, so a malloc needs two barriers and a free
// one: a class's decider zeroes its counter of the previous call, which every
// thread finished with before this call's first barrier.  ga_coll_begin
// zeroes the state once per kernel.
// ---------------------------------------------------------------------------
constexpr uint32_t kCollMax = 2048;              // threads of one block- or cluster-collective call
struct CollState {
    uint32_t cnt[2][kNcls];       // demand per class, double-buffered by `parity`
    uint32_t held[kNcls];         // 1: the class's demand was acquired for the collective this call
    uint32_t sig[kNcls];          // free: units owed to the collective arena's class semaphores
    uint32_t parity;
    uint32_t arena;               // arena_of() of the root CTA's SM
};
static __device__ __forceinline__ CollState* coll_local() {
    __shared__ CollState s;                      // one per CTA, only in kernels that use the collective calls
    return &s;
}
template <bool kCluster>
struct Coll {
    static __device__ __forceinline__ CollState* root() {
        if constexpr (kCluster) return cooperative_groups::this_cluster().map_shared_rank(coll_local(), 0u);
        else return coll_local();
    }
    static __device__ __forceinline__ void sync() {
        if constexpr (kCluster) cooperative_groups::this_cluster().sync();
        else __syncthreads();
    }
    static __device__ __forceinline__ uint32_t rank() {
        if constexpr (kCluster) return cooperative_groups::this_cluster().block_rank();
        else return 0;
    }
    static __device__ __forceinline__ uint32_t ncta() {
        if constexpr (kCluster) return cooperative_groups::this_cluster().num_blocks();
        else return 1;
    }
};
static __device__ __forceinline__ uint32_t cta_tid() { return threadIdx.x + blockDim.x * (threadIdx.y + blockDim.y * threadIdx.z); }
static __device__ __forceinline__ uint32_t cta_threads() { return blockDim.x * blockDim.y * blockDim.z; }

static __device__ __forceinline__ void coll_signal(const ga_desc* h, CollState* R, uint32_t A, int c, uint32_t n) {
    if (A == R->arena / class_share(c)) atomicAdd(&R->sig[c], n);
    else bsem_signal_after_rmw(sem_ptr(h, A, c), n);
}

template <bool kCluster>
static __device__ __noinline__ void coll_begin(const ga_desc* h) {
    CollState* L = coll_local();
    const uint32_t t = cta_tid();
    if (t < 2 * kNcls) (&L->cnt[0][0])[t] = 0;
    if (t < kNcls) L->sig[t] = 0;
    if (t == 0) { L->parity = 0; L->arena = arena_of(h); }
    Coll<kCluster>::sync();
}

// One thread decides class c for the whole collective: ONE Alg. 1 wait for
// the collective's demand Nc (B' = slots * ceil(Nc / slots), R-8).  ACQUIRED:
// every requesting group then claims with its units already held.  GROW is
// retracted (signal(0, B'-N)) and the groups run their own waits
// and growth; a blocked wait spins here first (delegating reclamation).
static __device__ __noinline__ void coll_decide_class(const ga_desc* h, CollState* R, uint32_t par, int c) {
    R->cnt[par ^ 1][c] = 0;                                          // the previous call's counter
    const uint32_t Nc = R->cnt[par][c];
    uint32_t held = 0;
    if (Nc) {
        const uint32_t A = R->arena / class_share(c);
        const uint32_t slots = slots_of(c);
        const uint32_t Bp = slots * ((Nc + slots - 1) / slots);
        uint64_t* sp = sem_ptr(h, A, c);
        uint64_t w = 0;
        int r = bsem_decide(sp, a_add(sp, dCD(-(int32_t)Nc, (int32_t)Bp)), Nc, Bp, &w);
        if (r == kBlocked) r = bsem_wait_slow<2048>(sp, Nc, Bp, ArenaSpin{h, A}, w);
        if (r == kGrow) bsem_signal(sp, 0, Bp - Nc);
        held = r == kAcquired;
    }
    R->held[c] = held;
}

template <bool kCluster>
static __device__ __noinline__ uint64_t malloc_coll_off(const ga_desc* h, uint64_t n) {
    using CC = Coll<kCluster>;
    CollState* R = CC::root();
    const unsigned act = active_lanes();
    const uint32_t lane = lane_id();
    if ((int)lane == __ffs(act) - 1) red_rlx(arena_ctr(h, 0), __popc(act));       // n_malloc, per warp
    const int key = size_key(h, n);
    const bool bin = key >= 0 && key < kNcls;
    const unsigned grp = __match_any_sync(act, key);
    const unsigned bl = __match_any_sync(act, (unsigned)bin);                      // valid in bin/span lanes
    const uint32_t par = R->parity;
    if (bin && (int)lane == __ffs(grp) - 1) atomicAdd(&R->cnt[par][key], (uint32_t)__popc(grp));
    CC::sync();                                                                     // demand complete
    const uint32_t t = cta_tid(), nc = CC::ncta(), me = CC::rank();
    if (me == 0 && t == 0) R->parity = par ^ 1;
    if (t * nc + me < (uint32_t)kNcls) coll_decide_class(h, R, par, (int)(t * nc + me));   // class c: CTA c % nc
    CC::sync();                                                                     // every decision made
    if (key < 0) return kNull;
    uint64_t my;
    if (bin) {
        const uint32_t A = R->arena / class_share(key);
        my = malloc_lockstep(h, bl, grp, key, A, R->held[key] != 0);
        const unsigned rest = __match_any_sync(bl, ((unsigned)key << 1) | (unsigned)(my == kNull));
        if (my == kNull) {
            if ((int)lane == __ffs(rest) - 1) stat_add(h, kStatFallback, 1);
            my = group_fallback(h, rest, A, key);
        }
        return my;
    }
    const int o = key - kNcls;                                                      // TBuddy: the warp path
    my = tree_malloc_group(h, grp, o);
    if (my == kNull) {
        int64_t x = tree_alloc_one_retry(h, o, false);
        if (x >= 0) {
            uint64_t pgt = (uint64_t)x << o;
            st_rlx32(&h->kind[pgt], kKindTree | (uint32_t)o);
            my = pgt << kPageShift;
        } else stat_add(h, kStatFail, 1);
    }
    return my;
}

template <bool kCluster>
static __device__ __noinline__ void free_coll_off(const ga_desc* h, uint64_t off) {
    using CC = Coll<kCluster>;
    CollState* R = CC::root();
    free_body<true>(h, off, R);
    CC::sync();                                                                     // every unit counted
    const uint32_t t = cta_tid();
    if (CC::rank() == 0 && t < kNcls) {
        const uint32_t v = atomicExch(&R->sig[t], 0u);
        if (v) bsem_signal_after_rmw(sem_ptr(h, R->arena / class_share((int)t), (int)t), v);
    }
}

}  // namespace ga
