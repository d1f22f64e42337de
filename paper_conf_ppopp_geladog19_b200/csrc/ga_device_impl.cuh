// ga_device_impl.cuh -- device implementation of the B200-native allocator.
//
// Method: Gelado & Garland, "Throughput-Oriented GPU Memory Allocation", PPoPP'19
// (PAPER.md, cited P:Lnnn).  Written for sm_100a from the paper's description;
// the paper's Volta design is prior art.
//
// Sections:
//   1. constants, PTX helpers
//   2. bulk semaphore (Alg. 1 / Alg. 2) packed as (C, D = E - R) in
//      one 64-bit word (reading R-6); wait is one CAS per attempt, signal one
//      red.release.add
//   3. hierarchical bitsets (find-any-set with scattered starts)
//   4. TBuddy over per-level availability bitmaps; lock-free merge
//      via a CAS on the word holding both siblings (reading R-21)
//   5. UAlloc: per-SM arenas, 64-page chunks, one-page bins with
//      out-of-band 256-bit slot bitmaps, per-class bulk semaphores
//   6. deferred reclamation delegated to waiting threads
//   7. warp-collective front end: __match_any_sync groups a warp's lanes by size
//      class; one leader performs the semaphore operation and the bitmap claim
//      for the whole group (collective critical section)
//
// Invariants the code relies on:
//   * bits[p][*] == all ones whenever page p is not a live bin, so a stale
//     claimer's atomicOr can never take a slot in a recycled page;
//   * kind[p] is written only while bits[p] is all ones; claimers re-validate it;
//   * chunk_used[k] == all ones whenever chunk k is not owned by an arena;
//   * at quiescence: class semaphore C == free slots of the arena's class bins,
//     page semaphore C == free pages of the arena's chunks, tree C[n] ==
//     available nodes of order n, every D == 0.
#pragma once
#include <cstdint>
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
constexpr int kNcls = 8;                        // classes 16 .. 2048 B
constexpr int kMinShift = 4;                    // 16 B minimum class (R-13)
constexpr int kBinWords = 4;                    // 256-bit slot bitmap per page
constexpr uint64_t kNull = ~0ull;
constexpr uint32_t kKindBin = 0x40000000u;      // | arena << 8 | class
constexpr uint32_t kKindTree = 0x80000000u;     // | order
constexpr int kSemStride = 4;                   // u64 words between semaphores (32 B)
constexpr int kMaxLevels = 48;

enum { kStatBinGrow = 0, kStatChunkGrow, kStatBinReclaim, kStatChunkReclaim, kStatFallback,
       kStatFail, kNumStats };

static __device__ __forceinline__ uint32_t lane_id() { uint32_t r; asm volatile("mov.u32 %0, %%laneid;" : "=r"(r)); return r; }
static __device__ __forceinline__ uint32_t lanemask_lt() { uint32_t r; asm volatile("mov.u32 %0, %%lanemask_lt;" : "=r"(r)); return r; }
static __device__ __forceinline__ uint32_t smid() { uint32_t r; asm volatile("mov.u32 %0, %%smid;" : "=r"(r)); return r; }

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
static __device__ __forceinline__ void stat_add(const ga_desc* h, int i, uint64_t v) { a_add(&h->stats[i], v); }

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
static __device__ __forceinline__ uint64_t lowest_bits(uint64_t x, int k) {
    uint64_t m = 0;
    while (k-- > 0 && x) { uint64_t b = x & (~x + 1); m |= b; x ^= b; }
    return m;
}
// position of the n-th (0-based) set bit of x
static __device__ __forceinline__ uint32_t nth_set(uint64_t x, uint32_t n) {
    uint32_t lo = __popc((uint32_t)x);
    if (n >= lo) { return 32 + __fns((uint32_t)(x >> 32), 0, (int)(n - lo) + 1); }
    return __fns((uint32_t)x, 0, (int)n + 1);
}

static __device__ __forceinline__ uint32_t slots_of(int c) { return 256u >> c; }
static __device__ __forceinline__ int words_of(int c) { return c == 0 ? 4 : c == 1 ? 2 : 1; }
static __device__ __forceinline__ uint64_t valid_mask(int c, int w) {
    int s = (int)slots_of(c) - 64 * w;
    return s >= 64 ? ~0ull : s <= 0 ? 0ull : ((1ull << s) - 1);
}
static __device__ __forceinline__ uint32_t arena_of(const ga_desc* h) { return smid() % h->n_arenas; }
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

// try-wait (R-7): C -= N iff C >= N.  One fetch-add: subtract,
// and give the units back if the pre-image was short.
static __device__ __forceinline__ bool bsem_trywait(uint64_t* s, uint32_t N) {
    if (sem_C(ld_rlx(s)) < (int32_t)N) return false;
    const uint64_t dn = (uint64_t)N << 32;
    uint64_t old = a_add(s, (uint64_t)0 - dn);
    if (sem_C(old) >= (int32_t)N) return true;
    a_add(s, dn);
    return false;
}

// Alg. 1 core (documentation at bsem_wait below).
template <bool kExact, class Spin>
static __device__ __noinline__ int bsem_wait_impl(uint64_t* s, uint32_t N, uint32_t B, Spin spin) {
    const uint64_t dn = (uint64_t)N << 32;
    uint64_t w;
    if (kExact) {
        // Fast path: a plain load says the units are there -> one fetch-add.
        // If it raced (pre-image short), give them back and run the exact form.
        w = ld_rlx(s);
        if (sem_C(w) >= (int32_t)N) {
            uint64_t old = a_add(s, (uint64_t)0 - dn);
            if (sem_C(old) >= (int32_t)N) return kAcquired;
            w = a_add(s, dn) + dn;
        }
        // Exact Alg. 1: one CAS decides among the three branches on the current word.
        for (;;) {
            int32_t C = sem_C(w), D = sem_D(w);
            uint64_t nw;
            int res;
            if ((int64_t)C + D < (int64_t)N) { nw = w + (uint64_t)(B - N); res = kGrow; }         // E += B - N
            else if (C >= (int32_t)N) { nw = w - dn; res = kAcquired; }                        // C -= N
            else { nw = w - (uint64_t)N; res = kBlocked; }                                      // R += N
            uint64_t old = a_cas(s, w, nw);
            if (old != w) { w = old; continue; }
            if (res != kBlocked) return res;
            uint32_t ns = 64;
            for (;;) {                                                                          // R-2
                w = ld_rlx(s);
                if (!(sem_C(w) < (int32_t)N && (int64_t)sem_C(w) + sem_D(w) >= 0)) break;
                spin();
                __nanosleep(ns);
                if (ns < 2048) ns <<= 1;
            }
            w = a_add(s, (uint64_t)N) + (uint64_t)N;                                            // R -= N
        }
    }
    // Optimistic form: one fetch-add C -= N decides on the pre-image.
    //   pre C >= N           -> ACQUIRED (one atomic, no retry)
    //   pre C + D < N        -> GROW: give C back, E += B - N
    //   otherwise            -> reserve: give C back, R += N (C + D unchanged), spin
    // Reservation conversions keep C + D exact; an in-flight GROW conversion hides
    // its units for one round trip, so others may over-produce (never over-grant).
    for (;;) {
        uint64_t old = a_add(s, (uint64_t)0 - dn);
        int32_t C = sem_C(old), D = sem_D(old);
        if (C >= (int32_t)N) return kAcquired;
        if ((int64_t)C + D < (int64_t)N) {
            a_add(s, dn + (uint64_t)(B - N));                                                   // C += N, E += B - N
            return kGrow;
        }
        w = a_add(s, dn - (uint64_t)N) + dn - (uint64_t)N;                                     // C += N, R += N
        uint32_t ns = 64;
        while (sem_C(w) < (int32_t)N && (int64_t)sem_C(w) + sem_D(w) >= 0) {                    // R-2
            spin();
            __nanosleep(ns);
            if (ns < 2048) ns <<= 1;
            w = ld_rlx(s);
        }
        a_add(s, (uint64_t)N);                                                                  // R -= N
    }
}
// Alg. 1.  Returns kAcquired (0) or kGrow (-1; the caller must
// produce B units, keep N and signal(B - N, B - N), or signal(0, B - N) on
// failure).  While blocked it runs `spin()` -- the delegated work
// of Sec. 4.2.1 -- between polls.  Reading R-2: keep waiting while
// C < N and R <= C + E, i.e. C < N and C + D >= 0.
// bsem_wait: exact growth decisions (arena class / page semaphores: an extra
//   batch costs real pages); bsem_wait_fast: optimistic (TBuddy orders: an extra
//   split stays available inside the tree).  DESIGN.md "Semaphore word".
template <class Spin>
static __device__ __forceinline__ int bsem_wait(uint64_t* s, uint32_t N, uint32_t B, Spin spin) { return bsem_wait_impl<true>(s, N, B, spin); }
template <class Spin>
static __device__ __forceinline__ int bsem_wait_fast(uint64_t* s, uint32_t N, uint32_t B, Spin spin) { return bsem_wait_impl<false>(s, N, B, spin); }
struct NoSpin { __device__ void operator()() const {} };

// ---------------------------------------------------------------------------
// 3. hierarchical bitsets: level 0 holds the data bits, level k+1 has one bit per
// non-zero word of level k.  Summary bits may be transiently stale in either
// direction; finders tolerate false positives, callers that hold semaphore
// units retry on a false negative (a setter is about to publish its bit).
// ---------------------------------------------------------------------------
struct HB {
    uint64_t* w;          // level 0 at w[0], then the summaries
    uint32_t n[4];        // words per level
    uint32_t off[4];      // word offset of each level
    int nl;               // number of levels
};
__host__ __device__ inline HB hb_make(uint64_t* base, uint32_t n0) {
    HB b; b.w = base; b.nl = 0;
    uint32_t n = n0 ? n0 : 1, o = 0;
    for (;;) {
        b.n[b.nl] = n; b.off[b.nl] = o; b.nl++; o += n;
        if (n == 1 || b.nl == 4) break;
        n = (n + 63) / 64;
    }
    return b;
}
__host__ __device__ inline uint32_t hb_total_words(uint32_t n0) {
    HB b = hb_make(nullptr, n0); return b.off[b.nl - 1] + b.n[b.nl - 1];
}
// propagate "word j of level k became non-zero" upwards
static __device__ __forceinline__ void hb_up_set(const HB& b, int k, uint32_t j) {
    for (; k + 1 < b.nl; k++) {
        uint64_t old = a_or(&b.w[b.off[k + 1] + (j >> 6)], 1ull << (j & 63));
        if (old) return;
        j >>= 6;
    }
}
// propagate "word j of level k became zero" upwards, with clear-then-recheck
static __device__ __noinline__ void hb_up_clear(const HB& b, int k, uint32_t j) {
    for (; k + 1 < b.nl; k++) {
        uint64_t* sw = &b.w[b.off[k + 1] + (j >> 6)];
        uint64_t bit = 1ull << (j & 63);
        uint64_t old = a_and(sw, ~bit);
        fence_sc();
        if (ld_rlx(&b.w[b.off[k] + j]) != 0) {          // re-set: a setter raced with us
            uint64_t o2 = a_or(sw, bit);
            if (o2 == 0) hb_up_set(b, k + 1, j >> 6);
            return;
        }
        if ((old & ~bit) != 0) return;                   // summary word still non-zero
        j >>= 6;
    }
}
// set bit i (level 0); returns the previous level-0 word
static __device__ __forceinline__ uint64_t hb_set(const HB& b, uint64_t i) {
    uint64_t old = a_or(&b.w[i >> 6], 1ull << (i & 63));
    if (old == 0) hb_up_set(b, 0, (uint32_t)(i >> 6));
    return old;
}
// called after an atomic made level-0 word j zero
static __device__ __forceinline__ void hb_word_zeroed(const HB& b, uint32_t j) { if (b.nl > 1) hb_up_clear(b, 0, j); }
// find a level-0 word that looks non-zero, starting the search at a scattered
// position; returns its index or -1
static __device__ __noinline__ int64_t hb_find(const HB& b, uint32_t seed) {
    int top = b.nl - 1;
    uint32_t nt = b.n[top];
    for (uint32_t t = 0; t < nt; t++) {
        uint32_t j = (seed + t) % nt;
        uint64_t x = ld_rlx(&b.w[b.off[top] + j]);
        // depth-first descent through candidate bits (at most 4 levels)
        uint32_t idx[4]; uint64_t rem[4];
        int k = top; idx[k] = j; rem[k] = x;
        while (k <= top) {
            if (rem[k] == 0) { k++; continue; }
            if (k == 0) return (int64_t)idx[0];
            uint32_t bit = first_from(rem[k], seed >> (5 * k));
            rem[k] &= ~(1ull << bit);
            uint32_t child = idx[k] * 64 + bit;
            if (child >= b.n[k - 1]) continue;
            uint64_t y = ld_rlx(&b.w[b.off[k - 1] + child]);
            if (y == 0) continue;
            k--; idx[k] = child; rem[k] = y;
            if (k == 0) return (int64_t)child;
        }
    }
    return -1;
}
static __device__ __forceinline__ HB level_hb(const ga_desc* h, int n) { HB b = hb_make(h->avail + h->lvl_off[n], h->lvl_words[n]); return b; }
static __device__ __forceinline__ HB owned_hb(const ga_desc* h, uint32_t A) {
    uint32_t tw = hb_total_words(h->chunk_words);
    return hb_make(h->owned + (uint64_t)A * tw, h->chunk_words);
}

// ---------------------------------------------------------------------------
// 4. TBuddy
// ---------------------------------------------------------------------------
static __device__ __forceinline__ bool node_inside(const ga_desc* h, int n, uint64_t i) { return ((i + 1) << n) <= h->pages; }

// make node i of level n available (a split's right child, a freed root)
static __device__ __forceinline__ void tree_publish(const ga_desc* h, int n, uint64_t i, uint32_t expected) {
    HB b = level_hb(h, n);
    hb_set(b, i);
    bsem_signal(tsem_ptr(h, n), 1, expected);            // C += 1 (and retire E if it was expected)
}

// claim up to `need` available nodes of level n (caller holds `need` units of
// tsem[n]); claims from one word; returns the word index and the claimed mask
static __device__ __noinline__ uint64_t tree_claim_word(const ga_desc* h, int n, int need, uint32_t seed, uint64_t* word_out) {
    HB b = level_hb(h, n);
    uint32_t ns = 32;
    for (;;) {
        int64_t j = hb_find(b, seed);
        if (j >= 0) {
            uint64_t* wp = &b.w[j];
            uint64_t x = ld_rlx(wp);
            while (x) {
                uint64_t m = lowest_bits(x, need);
                uint64_t old = a_and(wp, ~m);
                uint64_t got = old & m;
                if ((old & ~m) == 0 && old != 0) hb_word_zeroed(b, (uint32_t)j);
                if (got) { *word_out = (uint64_t)j; return got; }
                x = old & ~m;
            }
        }
        __nanosleep(ns); if (ns < 1024) ns <<= 1;
        seed = hash32(seed + 1);
    }
}

// Single-thread allocation of one order-o block, iterative:
// climb while wait says GROW, claim at the first level that grants, split down.
// Returns the node index at level o, or -1 (every E retracted).
static __device__ __noinline__ int64_t tree_alloc_one(const ga_desc* h, int o) {
    int m = o;
    for (;;) {
        if (m > (int)h->L) {                               // no parent: fail, retract E below
            for (int k = o; k < m; k++) bsem_signal(tsem_ptr(h, k), 0, 1);
            return -1;
        }
        if (bsem_wait_fast(tsem_ptr(h, m), 1, 2, NoSpin()) == kAcquired) break;   // batch size two
        m++;
    }
    uint64_t wj;
    uint64_t got = tree_claim_word(h, m, 1, scatter_seed(), &wj);
    uint64_t x = wj * 64 + (uint64_t)(__ffsll((long long)got) - 1);
    for (int k = m - 1; k >= o; k--) {                    // split: keep left, publish right
        x = 2 * x;
        tree_publish(h, k, x + 1, 1);
    }
    return (int64_t)x;
}

// Free node x of level n: merge with the buddy when try-wait and
// the buddy's available->busy transition both succeed, cascading (R-19);
// otherwise mark it available with one CAS on the word that holds both
// siblings (R-21), so two siblings never both end up available.
static __device__ __noinline__ void tree_free(const ga_desc* h, int n, uint64_t x) {
    uint32_t ns = 32;
    for (;;) {
        HB b = level_hb(h, n);
        uint64_t* wp = &b.w[x >> 6];
        uint64_t xb = 1ull << (x & 63), yb = 1ull << ((x ^ 1) & 63);
        bool root = (n >= (int)h->L) || !node_inside(h, n, x ^ 1);
        uint64_t w = ld_rlx(wp);
        if (!root && (w & yb)) {
            if (bsem_trywait(tsem_ptr(h, n), 1)) {
                uint64_t old = a_and(wp, ~yb);
                if (old & yb) {                           // merged: free the parent at n + 1
                    if ((old & ~yb) == 0) hb_word_zeroed(b, (uint32_t)(x >> 6));
                    x >>= 1; n++;
                    ns = 32;
                    continue;
                }
                bsem_signal(tsem_ptr(h, n), 1, 0);        // buddy claimed meanwhile: give back
            } else {
                __nanosleep(ns); if (ns < 1024) ns <<= 1; // buddy's unit is held by a claimer
            }
            continue;
        }
        uint64_t old = a_cas(wp, w, w | xb);
        if (old != w) continue;                           // the pair changed: re-evaluate
        if (w == 0) hb_up_set(b, 0, (uint32_t)(x >> 6));
        bsem_signal(tsem_ptr(h, n), 1, 0);
        return;
    }
}

// Does any order >= o show a unit (C >= 1) or growth / reservations in flight
// (D != 0)?  At true exhaustion every such word is (0, 0).
static __device__ __noinline__ bool tree_has_supply(const ga_desc* h, int o) {
    for (int k = o; k <= (int)h->L; k++) {
        uint64_t w = ld_rlx(tsem_ptr(h, k));
        if (sem_C(w) >= 1 || sem_D(w) != 0) return true;
    }
    return false;
}
// Per-lane TBuddy allocation with the no-false-starvation retry: the optimistic
// order semaphores can send a lane up the tree while another lane's split is
// still being published (R-27 analogue).  Retry while the tree shows supply;
// before giving up, drain deferred reclamation once (empty chunks go back).
static __device__ __noinline__ int64_t tree_alloc_one_retry(const ga_desc* h, int o);

// ---------------------------------------------------------------------------
// 5. UAlloc: chunks, pages, bins
// ---------------------------------------------------------------------------
static __device__ __forceinline__ uint32_t kind_bin(uint32_t A, int c) { return kKindBin | (A << 8) | (uint32_t)c; }

// Reclamation (section 6) forward declarations
static __device__ void reclaim_arena(const ga_desc* h, uint32_t A, int budget);
struct ArenaSpin {
    const ga_desc* h; uint32_t A;
    __device__ void operator()() const { reclaim_arena(h, A, 4); }
};

// Take a new chunk from TBuddy for arena A, keep the first k pages, open the
// rest.  Returns the chunk index or -1.
static __device__ __noinline__ int64_t chunk_acquire(const ga_desc* h, uint32_t A, uint32_t k) {
    int64_t ch = tree_alloc_one(h, kChunkOrder);
    if (ch < 0) return -1;
    st_rlx32(&h->chunk_owner[ch], A + 1);
    fence();
    hb_set(owned_hb(h, A), (uint64_t)ch);
    uint64_t keep = k >= 64 ? ~0ull : ((1ull << k) - 1);
    a_and(&h->chunk_used[ch], keep);                       // open pages k..63
    stat_add(h, kStatChunkGrow, 1);
    return ch;
}

// Claim up to `need` free pages of one chunk owned by A (caller holds `need`
// units of psem[A]).  Returns the mask of pages claimed, chunk in *ch_out.
static __device__ __noinline__ uint64_t page_claim(const ga_desc* h, uint32_t A, int need, uint64_t* ch_out) {
    HB ob = owned_hb(h, A);
    uint32_t seed = scatter_seed();
    uint32_t ns = 32;
    for (;;) {
        // scan every owned chunk word
        for (uint32_t t = 0; t < ob.n[0]; t++) {
            uint32_t j = (seed + t) % ob.n[0];
            uint64_t ow = ld_rlx(&ob.w[j]);
            while (ow) {
                uint32_t bit = (uint32_t)(__ffsll((long long)ow) - 1);
                ow &= ow - 1;
                uint64_t ch = (uint64_t)j * 64 + bit;
                uint64_t u = ld_rlx(&h->chunk_used[ch]);
                while (~u) {
                    uint64_t m = lowest_bits(~u, need);
                    uint64_t old = a_or(&h->chunk_used[ch], m);
                    uint64_t got = m & ~old;
                    if (got) {
                        if (ld_rlx32(&h->chunk_owner[ch]) != A + 1) {   // recycled chunk: undo
                            a_and(&h->chunk_used[ch], ~got);
                            break;
                        }
                        *ch_out = ch;
                        return got;
                    }
                    u = old | m;
                }
            }
        }
        __nanosleep(ns); if (ns < 1024) ns <<= 1;
    }
}

// Return page p (chunk ch, owner A) to its chunk: C += 1 on psem[A].  An empty
// chunk goes back to TBuddy (R-23).
static __device__ void chunk_release(const ga_desc* h, uint64_t ch);
static __device__ __noinline__ void page_release(const ga_desc* h, uint64_t p) {
    uint64_t ch = p >> kChunkShift;
    uint32_t A = ld_rlx32(&h->chunk_owner[ch]) - 1;
    uint64_t bit = 1ull << (p & (kChunkPages - 1));
    uint64_t old = a_and(&h->chunk_used[ch], ~bit);
    bsem_signal(psem_ptr(h, A), 1, 0);
    if ((old & ~bit) == 0) chunk_release(h, ch);
}

// An empty chunk back to the tree: try-wait all 64 page units, then take every
// page with one CAS (0 -> all ones).  Failure leaves the chunk owned.
static __device__ __noinline__ void chunk_release(const ga_desc* h, uint64_t ch) {
    uint32_t A = ld_rlx32(&h->chunk_owner[ch]) - 1;
    if (A >= h->n_arenas) return;
    if (!bsem_trywait(psem_ptr(h, A), kChunkPages)) return;
    if (a_cas(&h->chunk_used[ch], 0ull, ~0ull) != 0ull) { bsem_signal(psem_ptr(h, A), kChunkPages, 0); return; }
    HB ob = owned_hb(h, A);
    uint64_t old = a_and(&ob.w[ch >> 6], ~(1ull << (ch & 63)));
    if ((old & ~(1ull << (ch & 63))) == 0) hb_word_zeroed(ob, (uint32_t)(ch >> 6));
    a_exch(&h->chunk_cand[ch], 0);
    for (int c = 0; c < kNcls; c++) a_exch(&h->chunk_nonfull[ch * kNcls + c], 0);
    st_rlx32(&h->chunk_owner[ch], 0);
    fence();
    stat_add(h, kStatChunkReclaim, 1);
    tree_free(h, kChunkOrder, ch);
}

// Make page p a bin of class c for arena A.  The group keeps slots [0, take);
// the others are opened (bitmap was all ones).  Returns true if slots remain.
static __device__ __forceinline__ bool bin_init(const ga_desc* h, uint64_t p, uint32_t A, int c, uint32_t take) {
    st_rlx32(&h->kind[p], kind_bin(A, c));
    fence();
    uint64_t* bw = page_bits(h, p);
    for (int w = 0; w < words_of(c); w++) {
        uint64_t v = valid_mask(c, w);
        int lo = (int)take - 64 * w;                      // kept slots in this word
        uint64_t keep = lo >= 64 ? ~0ull : lo <= 0 ? 0ull : ((1ull << lo) - 1);
        uint64_t open = v & ~keep;
        if (open) a_and(&bw[w], ~open);
    }
    return take < slots_of(c);
}

static __device__ __forceinline__ void nonfull_set(const ga_desc* h, uint64_t p, int c) {
    uint64_t* nf = &h->chunk_nonfull[(p >> kChunkShift) * kNcls + c];
    uint64_t bit = 1ull << (p & (kChunkPages - 1));
    if (!(ld_rlx(nf) & bit)) a_or(nf, bit);
}
static __device__ __forceinline__ bool page_full(const uint64_t w[4], int c) {
    for (int i = 0; i < words_of(c); i++) if ((w[i] | ~valid_mask(c, i)) != ~0ull) return false;
    return true;
}
// clear-then-recheck: drop p from the nonfull set only if it is really full
static __device__ __noinline__ void nonfull_clear_if_full(const ga_desc* h, uint64_t p, int c, uint32_t A) {
    uint64_t* nf = &h->chunk_nonfull[(p >> kChunkShift) * kNcls + c];
    uint64_t bit = 1ull << (p & (kChunkPages - 1));
    a_and(nf, ~bit);
    fence_sc();
    uint64_t w[4];
    ld_bitmap(page_bits(h, p), w);
    if (ld_rlx32(&h->kind[p]) == kind_bin(A, c) && !page_full(w, c)) a_or(nf, bit);
}

// Try to claim up to `need` slots of page p (must be an (A, c) bin) from one
// word.  Returns the claimed mask and word index; 0 if the page had none.
static __device__ __noinline__ uint64_t bin_claim_page(const ga_desc* h, uint64_t p, uint32_t A, int c, int need, int* word_out) {
    if (ld_rlx32(&h->kind[p]) != kind_bin(A, c)) return 0;
    uint64_t* bw = page_bits(h, p);
    uint64_t w[4];
    ld_bitmap(bw, w);
    for (int i = 0; i < words_of(c); i++) {
        uint64_t fr = ~w[i] & valid_mask(c, i);
        while (fr) {
            uint64_t m = lowest_bits(fr, need);
            uint64_t old = a_or(&bw[i], m);
            uint64_t got = m & ~old;
            if (got) {
                if (ld_rlx32(&h->kind[p]) != kind_bin(A, c)) {     // recycled page: undo as a free
                    a_and(&bw[i], ~got);
                    return 0;
                }
                w[i] = old | m;
                if ((w[i] | ~valid_mask(c, i)) == ~0ull) {       // this word is full now
                    ld_bitmap(bw, w);
                    if (page_full(w, c)) nonfull_clear_if_full(h, p, c, A);
                }
                *word_out = i;
                return got;
            }
            fr = ~(old | m) & valid_mask(c, i);
        }
    }
    return 0;
}

// Find a bin of (A, c) with a free slot: the arena hint first, then every
// owned chunk's nonfull mask.  Returns the page or kNull.
static __device__ __noinline__ uint64_t bin_find(const ga_desc* h, uint32_t A, int c, uint32_t seed) {
    HB ob = owned_hb(h, A);
    for (uint32_t t = 0; t < ob.n[0]; t++) {
        uint32_t j = (seed + t) % ob.n[0];
        uint64_t ow = ld_rlx(&ob.w[j]);
        while (ow) {
            uint32_t bit = (uint32_t)(__ffsll((long long)ow) - 1);
            ow &= ow - 1;
            uint64_t ch = (uint64_t)j * 64 + bit;
            uint64_t nf = ld_rlx(&h->chunk_nonfull[ch * kNcls + c]);
            while (nf) {
                uint32_t pb = (uint32_t)(__ffsll((long long)nf) - 1);
                nf &= nf - 1;
                uint64_t p = ch * kChunkPages + pb;
                uint64_t w[4];
                ld_bitmap(page_bits(h, p), w);
                if (ld_rlx32(&h->kind[p]) == kind_bin(A, c) && !page_full(w, c)) return p;
                nonfull_clear_if_full(h, p, c, A);        // stale bit
            }
        }
    }
    return kNull;
}

// ---------------------------------------------------------------------------
// 6. deferred reclamation: frees that empty a bin only mark it;
// threads blocked in a semaphore wait, growers and failing mallocs reclaim.
// ---------------------------------------------------------------------------
// Reclaim page p if it is an empty bin: try-wait all its slots (R-22), then
// take every slot word with a CAS (all free -> all ones).
static __device__ __noinline__ bool bin_reclaim(const ga_desc* h, uint64_t p) {
    uint32_t k = ld_rlx32(&h->kind[p]);
    if ((k & 0xC0000000u) != kKindBin) return false;
    uint32_t A = (k >> 8) & 0xFFFFu;
    int c = (int)(k & 0xFF);
    uint64_t* bw = page_bits(h, p);
    uint64_t w[4];
    ld_bitmap(bw, w);
    for (int i = 0; i < words_of(c); i++) if (w[i] & valid_mask(c, i)) return false;
    uint32_t slots = slots_of(c);
    if (!bsem_trywait(sem_ptr(h, A, c), slots)) return false;
    int i = 0;
    for (; i < words_of(c); i++) {
        uint64_t v = valid_mask(c, i);
        if (a_cas(&bw[i], ~v, ~0ull) != ~v) break;
    }
    if (i < words_of(c)) {                                // a slot was claimed meanwhile: undo
        for (int q = 0; q < i; q++) a_and(&bw[q], ~valid_mask(c, q));
        bsem_signal(sem_ptr(h, A, c), slots, 0);
        return false;
    }
    a_and(&h->chunk_nonfull[(p >> kChunkShift) * kNcls + c], ~(1ull << (p & (kChunkPages - 1))));
    st_rlx32(&h->kind[p], 0);
    fence();
    stat_add(h, kStatBinReclaim, 1);
    page_release(h, p);
    return true;
}

static __device__ __forceinline__ void mark_candidate(const ga_desc* h, uint64_t p, uint32_t A) {
    uint64_t* cw = &h->chunk_cand[p >> kChunkShift];
    uint64_t bit = 1ull << (p & (kChunkPages - 1));
    if (!(ld_rlx(cw) & bit)) a_or(cw, bit);
    fence_sc();
    if (!ld_rlx(&h->cand_any[A * kSemStride])) a_or(&h->cand_any[A * kSemStride], 1);
}

// Reclaim up to `budget` candidate bins of arena A (budget < 0: all).
static __device__ __noinline__ void reclaim_arena(const ga_desc* h, uint32_t A, int budget) {
    uint64_t* any = &h->cand_any[A * kSemStride];
    if (!ld_rlx(any)) return;
    a_exch(any, 0);
    fence_sc();
    HB ob = owned_hb(h, A);
    bool left = false;
    for (uint32_t j = 0; j < ob.n[0]; j++) {
        uint64_t ow = ld_rlx(&ob.w[j]);
        while (ow) {
            uint32_t bit = (uint32_t)(__ffsll((long long)ow) - 1);
            ow &= ow - 1;
            uint64_t ch = (uint64_t)j * 64 + bit;
            if (!ld_rlx(&h->chunk_cand[ch])) continue;
            if (budget == 0) { left = true; break; }
            uint64_t cm = a_exch(&h->chunk_cand[ch], 0);
            while (cm) {
                uint32_t pb = (uint32_t)(__ffsll((long long)cm) - 1);
                cm &= cm - 1;
                if (budget == 0) { a_or(&h->chunk_cand[ch], 1ull << pb); left = true; continue; }
                bin_reclaim(h, ch * kChunkPages + pb);
                if (budget > 0) budget--;
            }
        }
        if (left) break;
    }
    if (left) { fence(); a_or(any, 1); }
}
static __device__ __noinline__ void reclaim_all(const ga_desc* h) {
    for (uint32_t A = 0; A < h->n_arenas; A++) reclaim_arena(h, A, -1);
}

static __device__ __noinline__ int64_t tree_alloc_one_retry(const ga_desc* h, int o) {
    bool drained = false;
    uint32_t ns = 64;
    for (int attempt = 0; attempt < 256; attempt++) {
        int64_t x = tree_alloc_one(h, o);
        if (x >= 0) return x;
        if (!tree_has_supply(h, o)) {
            if (drained) return -1;
            reclaim_all(h);
            drained = true;
            continue;
        }
        __nanosleep(ns); if (ns < 4096) ns <<= 1;
    }
    return -1;
}

// ---------------------------------------------------------------------------
// 7. front end
// ---------------------------------------------------------------------------
// size -> key: 0..7 bin class, 8 + order for TBuddy, -1 for NULL
static __device__ __forceinline__ int size_key(const ga_desc* h, uint64_t n) {
    if (n == 0 || n > (h->pages << kPageShift)) return -1;                  // R-15
    if (n <= 16) return 0;
    int lg = 64 - __clzll((long long)(n - 1));                            // ceil(log2 n), R-14
    if (lg <= 11) return lg - kMinShift;                                  // <= 2048 B: bins (R-12)
    int o = lg - kPageShift;
    if (o > (int)h->L) return -1;
    return kNcls + o;
}

// A grant tells the group which slots / nodes it received in one round.
struct Grant {
    uint64_t unit;      // bins: page; tree: word index at level m
    uint64_t mask;      // bins: slot mask within word `word`; pages grant: page mask in chunk
    uint32_t base;      // first group rank served
    uint32_t count;     // ranks served
    int word;           // bins: word of the page bitmap; tree: shift m - o
    int kind;           // 0 slots, 1 fresh pages of a chunk, 2 tree nodes, 3 done, 4 failed
};

static __device__ __forceinline__ Grant shfl_grant(unsigned grp, Grant g, int src) {
    Grant r;
    r.unit = __shfl_sync(grp, g.unit, src);
    r.mask = __shfl_sync(grp, g.mask, src);
    r.base = __shfl_sync(grp, g.base, src);
    r.count = __shfl_sync(grp, g.count, src);
    r.word = __shfl_sync(grp, g.word, src);
    r.kind = __shfl_sync(grp, g.kind, src);
    return r;
}

// ---- bins, group path ------------------------------------------------------
struct BinLeader {
    uint32_t A; int c; uint32_t N;
    uint32_t served;       // ranks served so far
    int phase;             // 0 account, 1 claim existing, 2 fresh pages, 3 done
    uint32_t pages_left;   // fresh pages still to track (phase 2)
    uint32_t Bp;
    uint64_t hint;
    uint32_t seed;
};

static __device__ __noinline__ Grant bin_leader_step(const ga_desc* h, BinLeader& L) {
    Grant g; g.kind = 3; g.base = L.served; g.count = 0; g.unit = 0; g.mask = 0; g.word = 0;
    uint32_t slots = slots_of(L.c);
    if (L.phase == 0) {
        L.Bp = slots * ((L.N + slots - 1) / slots);                          // R-8
        int r = bsem_wait(sem_ptr(h, L.A, L.c), L.N, L.Bp, ArenaSpin{h, L.A});
        if (r == kAcquired) { L.phase = 1; L.hint = ld_rlx32(&h->hint[L.A * kNcls + L.c]); }
        else {
            // GROW: B'/slots new bins; pages accounted on the arena's page semaphore
            uint32_t k = L.Bp / slots;
            int rp = bsem_wait(psem_ptr(h, L.A), k, kChunkPages, ArenaSpin{h, L.A});
            if (rp == kGrow) {
                reclaim_arena(h, L.A, -1);                 // delegated work before a new chunk
                int64_t ch = chunk_acquire(h, L.A, k);
                if (ch < 0) {
                    bsem_signal(psem_ptr(h, L.A), 0, kChunkPages - k);
                    bsem_signal(sem_ptr(h, L.A, L.c), 0, L.Bp - L.N);
                    g.kind = 4;
                    return g;
                }
                bsem_signal(psem_ptr(h, L.A), kChunkPages - k, kChunkPages - k);
                L.phase = 2; L.pages_left = 0;
                // the whole batch sits in this chunk: pages 0..k-1
                uint64_t pm = k >= 64 ? ~0ull : ((1ull << k) - 1);
                uint32_t take_total = L.N;
                for (uint32_t i = 0; i < k; i++) {
                    uint32_t take = take_total > slots ? slots : take_total;
                    take_total -= take;
                    if (bin_init(h, (uint64_t)ch * kChunkPages + i, L.A, L.c, take))
                        nonfull_set(h, (uint64_t)ch * kChunkPages + i, L.c);
                }
                stat_add(h, kStatBinGrow, k);
                g.kind = 1; g.unit = (uint64_t)ch; g.mask = pm; g.count = L.N; g.word = (int)slots;
                L.served = L.N;
                L.hint = (uint64_t)ch * kChunkPages + k - 1;
                st_rlx32(&h->hint[L.A * kNcls + L.c], (uint32_t)L.hint);
                bsem_signal(sem_ptr(h, L.A, L.c), L.Bp - L.N, L.Bp - L.N);
                L.phase = 3;
                return g;
            }
            L.phase = 2; L.pages_left = k;
        }
    }
    if (L.phase == 2) {
        // track pages_left pages from the arena's chunks (units already held)
        uint64_t ch;
        uint64_t pm = page_claim(h, L.A, (int)L.pages_left, &ch);
        uint32_t np = __popcll(pm);
        uint32_t rem = L.N - L.served;
        uint32_t serve = np * slots < rem ? np * slots : rem;
        uint32_t left = serve;
        for (uint32_t i = 0; i < np; i++) {
            uint64_t p = ch * kChunkPages + nth_set(pm, i);
            uint32_t take = left > slots ? slots : left;
            left -= take;
            if (bin_init(h, p, L.A, L.c, take)) nonfull_set(h, p, L.c);
            L.hint = p;
        }
        stat_add(h, kStatBinGrow, np);
        L.pages_left -= np;
        g.kind = 1; g.unit = ch; g.mask = pm; g.count = serve; g.word = (int)slots;
        L.served += serve;
        if (L.pages_left == 0) {
            st_rlx32(&h->hint[L.A * kNcls + L.c], (uint32_t)L.hint);
            bsem_signal(sem_ptr(h, L.A, L.c), L.Bp - L.N, L.Bp - L.N);
            L.phase = 3;
        }
        return g;
    }
    if (L.phase == 1) {
        uint32_t ns = 32;
        for (;;) {
            uint64_t p = L.hint;
            if (p < h->pages) {
                int wi;
                uint64_t got = bin_claim_page(h, p, L.A, L.c, (int)(L.N - L.served), &wi);
                if (got) {
                    uint32_t n = __popcll(got);
                    g.kind = 0; g.unit = p; g.mask = got; g.word = wi; g.count = n;
                    L.served += n;
                    if (L.served == L.N) {
                        L.phase = 3;
                        if (ld_rlx32(&h->hint[L.A * kNcls + L.c]) != (uint32_t)p) st_rlx32(&h->hint[L.A * kNcls + L.c], (uint32_t)p);
                    }
                    return g;
                }
            }
            uint64_t q = bin_find(h, L.A, L.c, L.seed);
            if (q != kNull) { L.hint = q; continue; }
            // units are held but no bin is visible yet: a free / grower is publishing
            L.hint = kNull;
            __nanosleep(ns); if (ns < 1024) ns <<= 1;
            L.seed = hash32(L.seed + 7);
        }
    }
    return g;
}

// Per-lane slow path (R-26, R-27): N = 1 waits; after local growth fails,
// drain reclamation, then take pages and slots from other arenas before NULL.
static __device__ __noinline__ uint64_t bin_malloc_lane(const ga_desc* h, uint32_t A0, int c) {
    uint32_t slots = slots_of(c);
    uint64_t csz = 16ull << c;
    for (int attempt = 0; attempt < 2; attempt++) {
        int r = bsem_wait(sem_ptr(h, A0, c), 1, slots, ArenaSpin{h, A0});
        if (r == kAcquired) {
            uint32_t seed = scatter_seed();
            uint32_t ns = 32;
            uint64_t p = ld_rlx32(&h->hint[A0 * kNcls + c]);
            for (;;) {
                if (p < h->pages) {
                    int wi;
                    uint64_t got = bin_claim_page(h, p, A0, c, 1, &wi);
                    if (got) return (p << kPageShift) + (uint64_t)(wi * 64 + __ffsll((long long)got) - 1) * csz;
                }
                p = bin_find(h, A0, c, seed);
                if (p == kNull) { __nanosleep(ns); if (ns < 1024) ns <<= 1; seed = hash32(seed + 3); }
            }
        }
        int rp = bsem_wait(psem_ptr(h, A0), 1, kChunkPages, ArenaSpin{h, A0});
        uint64_t p = kNull;
        if (rp == kAcquired) {
            uint64_t ch;
            uint64_t pm = page_claim(h, A0, 1, &ch);
            p = ch * kChunkPages + (uint64_t)(__ffsll((long long)pm) - 1);
        } else {
            reclaim_arena(h, A0, -1);
            int64_t ch = chunk_acquire(h, A0, 1);
            if (ch >= 0) { bsem_signal(psem_ptr(h, A0), kChunkPages - 1, kChunkPages - 1); p = (uint64_t)ch * kChunkPages; }
            else bsem_signal(psem_ptr(h, A0), 0, kChunkPages - 1);
        }
        if (p != kNull) {
            if (bin_init(h, p, A0, c, 1)) nonfull_set(h, p, c);
            stat_add(h, kStatBinGrow, 1);
            st_rlx32(&h->hint[A0 * kNcls + c], (uint32_t)p);
            bsem_signal(sem_ptr(h, A0, c), slots - 1, slots - 1);
            return p << kPageShift;
        }
        bsem_signal(sem_ptr(h, A0, c), 0, slots - 1);
        if (attempt == 0) reclaim_all(h);
    }
    // every page source first (they only shrink in malloc-only phases), then
    // every arena's bins of this class: a malloc fails only if no arena can
    // serve it (R-26)
    for (uint32_t t = 1; t <= h->n_arenas; t++) {
        uint32_t B = (A0 + t) % h->n_arenas;
        if (bsem_wait(psem_ptr(h, B), 1, 1, NoSpin()) == kAcquired) {
            uint64_t ch;
            uint64_t pm = page_claim(h, B, 1, &ch);
            uint64_t p = ch * kChunkPages + (uint64_t)(__ffsll((long long)pm) - 1);
            if (bin_init(h, p, B, c, 1)) nonfull_set(h, p, c);
            stat_add(h, kStatBinGrow, 1);
            bsem_signal(sem_ptr(h, B, c), slots - 1, 0);
            return p << kPageShift;
        }
    }
    for (uint32_t t = 1; t <= h->n_arenas; t++) {
        uint32_t B = (A0 + t) % h->n_arenas;
        if (bsem_wait(sem_ptr(h, B, c), 1, 1, NoSpin()) == kAcquired) {
            uint32_t seed = scatter_seed();
            uint32_t ns = 32;
            uint64_t p = ld_rlx32(&h->hint[B * kNcls + c]);
            for (;;) {
                if (p < h->pages) {
                    int wi;
                    uint64_t got = bin_claim_page(h, p, B, c, 1, &wi);
                    if (got) return (p << kPageShift) + (uint64_t)(wi * 64 + __ffsll((long long)got) - 1) * csz;
                }
                p = bin_find(h, B, c, seed);
                if (p == kNull) { __nanosleep(ns); if (ns < 1024) ns <<= 1; seed = hash32(seed + 3); }
            }
        }
    }
    stat_add(h, kStatFail, 1);
    return kNull;
}

// ---- TBuddy, group path ----------------------------------------------------
struct TreeLeader {
    int o; int m; uint32_t N; uint32_t Nm; uint32_t served; uint32_t seed; int phase;
};
static __device__ __forceinline__ uint32_t ceil_half(uint32_t x) { return (x + 1) >> 1; }

static __device__ __noinline__ Grant tree_leader_step(const ga_desc* h, TreeLeader& L) {
    Grant g; g.kind = 3; g.base = L.served; g.count = 0; g.unit = 0; g.mask = 0; g.word = 0;
    if (L.phase == 0) {
        uint32_t Nk = L.N;
        int m = L.o;
        for (;;) {
            if (m > (int)h->L) {                              // nothing to grow from: retract E
                uint32_t nk = L.N;
                for (int k = L.o; k < m; k++) { bsem_signal(tsem_ptr(h, k), 0, 2 * ceil_half(nk) - nk); nk = ceil_half(nk); }
                g.kind = 4;
                return g;
            }
            int r = bsem_wait_fast(tsem_ptr(h, m), Nk, 2 * ceil_half(Nk), NoSpin());
            if (r == kAcquired) break;
            Nk = ceil_half(Nk);
            m++;
        }
        L.m = m; L.Nm = Nk; L.phase = 1;
    }
    if (L.phase == 1) {
        int s = L.m - L.o;
        uint32_t need_nodes = L.Nm - ((L.served + (1u << s) - 1) >> s);
        uint64_t wj;
        uint64_t got = tree_claim_word(h, L.m, (int)need_nodes, L.seed, &wj);
        uint32_t nn = __popcll(got);
        uint32_t rem = L.N - L.served;
        uint32_t cap = nn << s;
        uint32_t serve = cap < rem ? cap : rem;
        if (serve == rem && s > 0) {
            // the last node is split: publish the unused right parts (E at each level)
            uint64_t xlast = wj * 64 + (63 - __clzll((long long)got));
            uint32_t keep_last = serve - ((nn - 1) << s);
            uint64_t pos = keep_last;
            for (int j = 0; j < s; j++) {
                if ((pos >> j) & 1) {
                    tree_publish(h, L.o + j, ((xlast << s) + pos) >> j, 1);
                    pos += 1ull << j;
                }
            }
        }
        g.kind = 2; g.unit = wj; g.mask = got; g.count = serve; g.word = s;
        L.served += serve;
        if (L.served == L.N) L.phase = 3;
        return g;
    }
    return g;
}

// ---- the group driver --------------------------------------------------------
// Every lane of `grp` calls this with the same key; returns this lane's offset.
static __device__ __forceinline__ uint64_t group_malloc(const ga_desc* h, unsigned grp, int key) {
    const int lane = (int)lane_id();
    const int leader = __ffs(grp) - 1;
    const uint32_t N = __popc(grp);
    const uint32_t rank = __popc(grp & lanemask_lt());
    uint64_t my = kNull;
    BinLeader bl; TreeLeader tl;
    bool is_bin = key < kNcls;
    if (lane == leader) {
        if (is_bin) { bl.A = arena_of(h); bl.c = key; bl.N = N; bl.served = 0; bl.phase = 0; bl.pages_left = 0; bl.Bp = 0; bl.hint = kNull; bl.seed = scatter_seed(); }
        else { tl.o = key - kNcls; tl.m = tl.o; tl.N = N; tl.Nm = 0; tl.served = 0; tl.seed = scatter_seed(); tl.phase = 0; }
    }
    for (;;) {
        Grant g;
        if (lane == leader) g = is_bin ? bin_leader_step(h, bl) : tree_leader_step(h, tl);
        g = shfl_grant(grp, g, leader);
        if (g.kind >= 3) {
            if (g.kind == 4) {
                // R-27: the group could not be served as a whole -> per lane
                if (lane == leader) stat_add(h, kStatFallback, 1);
                if (my == kNull) {
                    if (is_bin) my = bin_malloc_lane(h, arena_of(h), key);
                    else {
                        int o = key - kNcls;
                        int64_t x = tree_alloc_one_retry(h, o);
                        if (x >= 0) {
                            uint64_t pg = (uint64_t)x << o;
                            st_rlx32(&h->kind[pg], kKindTree | (uint32_t)o);
                            my = pg << kPageShift;
                        } else stat_add(h, kStatFail, 1);
                    }
                }
            }
            break;
        }
        if (rank >= g.base && rank < g.base + g.count) {
            uint32_t r = rank - g.base;
            if (g.kind == 0) {
                uint32_t b = nth_set(g.mask, r);
                my = (g.unit << kPageShift) + (uint64_t)(g.word * 64 + b) * (16ull << key);
            } else if (g.kind == 1) {
                uint32_t slots = (uint32_t)g.word;
                uint64_t p = g.unit * kChunkPages + nth_set(g.mask, r / slots);
                my = (p << kPageShift) + (uint64_t)(r % slots) * (16ull << key);
            } else {
                int s = g.word, o = key - kNcls;
                uint64_t x = g.unit * 64 + nth_set(g.mask, r >> s);
                uint64_t node = (x << s) + (r & ((1u << s) - 1));
                uint64_t pg = node << o;
                st_rlx32(&h->kind[pg], kKindTree | (uint32_t)o);
                my = pg << kPageShift;
            }
        }
    }
    return my;
}

static __device__ __noinline__ uint64_t ga_malloc_off(const ga_desc* h, uint64_t n) {
    unsigned act = __activemask();
    int key = size_key(h, n);
    unsigned grp = __match_any_sync(act, key);
    if (key < 0) return kNull;
    return group_malloc(h, grp, key);
}

// free: TBuddy blocks per lane; bin slots grouped per bitmap word (one
// atomicAnd) and per (arena, class) (one signal)
static __device__ __noinline__ void ga_free_off(const ga_desc* h, uint64_t off) {
    unsigned act = __activemask();
    uint32_t k = 0;
    uint64_t p = 0;
    if (off != kNull) { p = off >> kPageShift; k = ld_rlx32(&h->kind[p]); }
    bool is_bin = (off != kNull) && ((k & 0xC0000000u) == kKindBin);
    unsigned bins = __ballot_sync(act, is_bin);
    if (off != kNull && !is_bin) {
        // TBuddy block (page aligned); order from the page kind (R-18)
        int o = (int)(k & 0xFF);
        st_rlx32(&h->kind[p], 0);
        fence();
        tree_free(h, o, p >> o);
    }
    if (!is_bin) return;
    uint32_t A = (k >> 8) & 0xFFFFu;
    int c = (int)(k & 0xFF);
    uint32_t slot = (uint32_t)((off & (kPage - 1)) >> (c + kMinShift));
    int w = (int)(slot >> 6);
    uint64_t key1 = (p << 2) | (uint64_t)w;
    unsigned g1 = __match_any_sync(bins, key1);
    uint64_t bit = 1ull << (slot & 63);
    uint32_t lo = __reduce_or_sync(g1, (uint32_t)bit), hi = __reduce_or_sync(g1, (uint32_t)(bit >> 32));
    uint64_t mask = ((uint64_t)hi << 32) | lo;
    if ((int)lane_id() == __ffs(g1) - 1) {
        uint64_t* bw = page_bits(h, p);
        uint64_t old = a_and(&bw[w], ~mask);
        uint64_t v = valid_mask(c, w);
        if ((old | ~v) == ~0ull) nonfull_set(h, p, c);    // the word was full: bin back in the list
        if (((old & ~mask) & v) == 0) {                    // this word is empty: is the bin?
            uint64_t ww[4];
            ld_bitmap(bw, ww);
            bool empty = true;
            for (int i = 0; i < words_of(c); i++) if (ww[i] & valid_mask(c, i)) empty = false;
            if (empty) mark_candidate(h, p, A);
        }
    }
    __syncwarp(bins);
    uint32_t key2 = (A << 3) | (uint32_t)c;
    unsigned g2 = __match_any_sync(bins, key2);
    if ((int)lane_id() == __ffs(g2) - 1) bsem_signal_after_rmw(sem_ptr(h, A, c), __popc(g2));
}

}  // namespace ga
