/*
 * oracle/ga_oracle.c -- sequential CPU ORACLE for Gelado & Garland,
 * "Throughput-Oriented GPU Memory Allocation", PPoPP'19 (/root/reference/PAPER.md,
 * cited below as P:Lnnn = PAPER.md line nnn).
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / `--impl reference` legs may load this library.  It shares no
 * code, header, table or constant with the CUDA path
 * (paper_conf_ppopp_geladog19_b200/csrc); neither side includes the other.
 *
 * What it computes (plain, sequential, one operation at a time, canonical order):
 *   - bulk semaphores, Alg. 1 / Alg. 2 -- sequentially
 *     E = R = 0 between calls, so wait() is "ACQUIRED iff C >= N, else GROW";
 *   - TBuddy: a static binary tree whose nodes are Available /
 *     Busy / Partial, one bulk semaphore per order with batch 2, split on GROW,
 *     merge-on-free with try-wait + buddy transition and (reading R-19) cascade;
 *   - UAlloc with ONE arena: chunks of CHUNK_PAGES pages taken
 *     from TBuddy, bins of one page holding one size class, per-bin bitmaps and
 *     free counters, per-class bulk semaphores (batch = slots per bin) and one
 *     page semaphore (batch = usable pages per chunk), eager reclamation of an
 *     empty bin / empty chunk (readings R-22, R-23);
 *   - the front end: round up to a power of two, route by size;
 *   - a trace runner, an allocation-log checker, a canonical snapshot writer and
 *     an invariant checker.
 *
 * Where the paper is silent or garbled the DESIGN.md readings R-1..R-31 apply;
 * each use is tagged below.  Choice among several legal blocks (R-20): the
 * oracle always takes the LOWEST address -- addresses are never compared with
 * the GPU, only counts, the empty-heap snapshot and log validity.
 *
 * Parity pins (tests/test_oracle_*.py): Fig. 1(b)/(a) traces (semaphore
 * stepper, oracle/bsem.py), buddy properties, brute force on tiny
 * heaps, closed-form capacities, the paper-layout failure rates of P:L1655-1698,
 * free-all == fresh snapshot.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <stdio.h>

#define ORA_NULL (~(uint64_t)0)

/* ------------------------------------------------------------------------- */
/* Bulk semaphore, sequential form of Alg. 1 / Alg. 2.                         */
/* ------------------------------------------------------------------------- */
typedef struct { int64_t C, E, R; } bsem;   /* value, expected, reserved */
enum { ACQUIRED = 0, GROW = -1 };

/* Alg. 1.  R-1: the garbled "Sem.C >= I" reads "Sem.C >= N".
 * R-8: B is the batch B' = B*ceil(N/B) the caller will produce on GROW.
 * Sequentially the third (reserve-and-block) branch is unreachable because
 * E = R = 0 between operations: C+E-R >= N and C < N cannot both hold. */
static int bsem_wait(bsem* s, int64_t N, int64_t B) {
    if (s->C + s->E - s->R < N) { s->E += B - N; return GROW; }
    if (s->C >= N) { s->C -= N; return ACQUIRED; }
    fprintf(stderr, "oracle: bsem_wait would block in a sequential run\n");
    abort();
}
/* Alg. 2; R-3: the box (C += N, E -= B) wins over the prose. */
static void bsem_signal(bsem* s, int64_t N, int64_t B) { s->C += N; s->E -= B; }
/* try-wait; R-7: decrement by N if C >= N, else fail. */
static int bsem_trywait(bsem* s, int64_t N) {
    if (s->C >= N) { s->C -= N; return 1; }
    return 0;
}

/* ------------------------------------------------------------------------- */
/* Indexed bitset: find the lowest set bit quickly.  Used only to find "the   */
/* lowest-address X" (R-20) without an O(n) scan; semantics = a plain set.    */
/* ------------------------------------------------------------------------- */
typedef struct { int nlev; uint64_t len[8]; uint64_t* w[8]; } bset;

static void bset_init(bset* b, uint64_t nbits) {
    memset(b, 0, sizeof *b);
    uint64_t n = nbits ? nbits : 1;
    do {
        uint64_t words = (n + 63) / 64;
        b->len[b->nlev] = words;
        b->w[b->nlev] = (uint64_t*)calloc(words, 8);
        b->nlev++;
        n = words;
    } while (n > 1);
}
static void bset_free(bset* b) { for (int i = 0; i < b->nlev; i++) free(b->w[i]); }
static void bset_set(bset* b, uint64_t i) {
    for (int l = 0; l < b->nlev; l++) {
        uint64_t wi = i >> 6, old = b->w[l][wi];
        b->w[l][wi] = old | (1ull << (i & 63));
        if (old) return;             /* upper levels already mark this word */
        i = wi;
    }
}
static void bset_clear(bset* b, uint64_t i) {
    for (int l = 0; l < b->nlev; l++) {
        uint64_t wi = i >> 6;
        b->w[l][wi] &= ~(1ull << (i & 63));
        if (b->w[l][wi]) return;     /* word still non-empty */
        i = wi;
    }
}
static int bset_test(const bset* b, uint64_t i) { return (b->w[0][i >> 6] >> (i & 63)) & 1; }
static int64_t bset_first(const bset* b) {
    int l = b->nlev - 1;
    uint64_t wi = 0;
    /* top level has exactly one word */
    if (!b->w[l][0]) return -1;
    for (;;) {
        uint64_t bit = (uint64_t)__builtin_ctzll(b->w[l][wi]);
        uint64_t idx = wi * 64 + bit;
        if (l == 0) return (int64_t)idx;
        l--; wi = idx;
    }
}

/* ------------------------------------------------------------------------- */
/* Layout (paper values P:L1026-1040, R-9..R-13).          */
/* ------------------------------------------------------------------------- */
typedef struct {
    uint32_t page;          /* bytes per page / bin (4096; R-9)          */
    uint32_t chunk_pages;   /* pages per chunk (64 bins; R-10)      */
    uint32_t min_class;     /* smallest class (build 16 B, R-13; paper 8 B)        */
    uint32_t bin_max;       /* largest bin class (build 2048 B; paper 1024 B, R-12)*/
    uint32_t paper_layout;  /* 1: in-band 128 B bin headers + 2 header bins per
                               chunk + 62 tails (R-11); 0: build     */
    uint32_t snap_max_class;/* snapshot FORMAT only (include/ga.h): the class
                               section has one counter pair per power of two from
                               min_class up to this size (65536 = the top of the
                               16 B - 64 KB mixed range, BASELINE.json configs[3]),
                               0 = bin classes only.  The oracle serves sizes above
                               bin_max from TBuddy, as the paper does
                               (P:L1655-1674), and writes zeros for those entries. */
} ora_layout;

enum { ST_BUSY = 0, ST_AVAIL = 1, ST_PARTIAL = 2 };   /* node states */
enum { PK_TREE = 0, PK_TREE_HEAD = 1, PK_CHUNK_FREE = 2, PK_CHUNK_HDR = 3, PK_BIN = 4 };

typedef struct {
    ora_layout lay;
    uint64_t heap_bytes, pages, nchunks;
    int L;                       /* tree height: 2^L >= pages                  */
    int chunk_order;             /* log2(chunk_pages)                          */
    int ncls;                    /* number of bin classes                      */
    uint32_t slots[32];          /* slots per bin, per class                   */
    uint32_t body_slots[32];     /* paper layout: slots in the bin body        */
    uint32_t words;              /* u64 bitmap words per bin                   */
    uint32_t usable_pages;       /* bin-capable pages per chunk                */
    uint32_t hdr_pages;          /* paper layout: 2 header bins per chunk      */
    /* TBuddy */
    uint8_t* st[64];             /* node state per level                       */
    bset av[64];                 /* index of AVAILABLE nodes per level         */
    bsem tsem[64];               /* one bulk semaphore per order  */
    /* UAlloc, one arena */
    bsem csem[32];               /* one bulk semaphore per size class          */
    bsem psem;                   /* free pages in the arena's chunks           */
    uint8_t* kind;               /* page kind (R-18)                           */
    uint8_t* aux;                /* order (tree head) or class (bin)           */
    uint64_t* bits;              /* bin bitmaps, words per page                */
    uint32_t* freecnt;           /* bin free counter            */
    uint8_t* chunk_owned;
    uint64_t* chunk_used;        /* used pages of the chunk (chunk header bitmap) */
    bset nonfull[32];            /* bins of class c with a free slot (the per-size
                                    bin free-list of P:L1040-1042, kept ordered)   */
    bset chunk_free;             /* owned chunks with a free usable page        */
    /* statistics */
    uint64_t reserved_pages, peak_reserved_pages;
    uint64_t n_malloc, n_fail, n_free, n_bin_grow, n_chunk_grow, n_bin_reclaim, n_chunk_reclaim;
} ora_heap;

static int ilog2_u64(uint64_t x) { return 63 - __builtin_clzll(x); }
static uint64_t ceil_pow2(uint64_t x) { uint64_t c = 1; while (c < x) c <<= 1; return c; }

/* Node (level n, index i) lies fully inside the usable heap. */
static int node_inside(const ora_heap* h, int n, uint64_t i) { return ((i + 1) << n) <= h->pages; }

static void set_state(ora_heap* h, int n, uint64_t i, int s) {
    uint8_t old = h->st[n][i];
    h->st[n][i] = (uint8_t)s;
    if (old == ST_AVAIL && s != ST_AVAIL) bset_clear(&h->av[n], i);
    if (old != ST_AVAIL && s == ST_AVAIL) bset_set(&h->av[n], i);
}

/* Propagation to the parents: a non-available node is Partial
 * iff its sub-tree holds an available block, else Busy. */
static void fix_up(ora_heap* h, int n, uint64_t i) {
    for (int k = n + 1; k <= h->L; k++) {
        i >>= 1;
        if (h->st[k][i] == ST_AVAIL) { fprintf(stderr, "oracle: available ancestor\n"); abort(); }
        uint8_t l = h->st[k - 1][2 * i], r = h->st[k - 1][2 * i + 1];
        set_state(h, k, i, (l != ST_BUSY || r != ST_BUSY) ? ST_PARTIAL : ST_BUSY);
    }
}

static void reserve_add(ora_heap* h, int64_t pages) {
    h->reserved_pages += (uint64_t)pages;
    if (h->reserved_pages > h->peak_reserved_pages) h->peak_reserved_pages = h->reserved_pages;
}

/* TBuddy allocation of order n.  Returns the node index or -1. */
static int64_t tree_alloc(ora_heap* h, int n) {
    if (n > h->L) return -1;
    if (bsem_wait(&h->tsem[n], 1, 2) == ACQUIRED) {          /* batch size two */
        int64_t i = bset_first(&h->av[n]);                    /* R-20: lowest address */
        if (i < 0) { fprintf(stderr, "oracle: semaphore/tree mismatch\n"); abort(); }
        set_state(h, n, (uint64_t)i, ST_BUSY);                /* available -> busy */
        fix_up(h, n, (uint64_t)i);
        return i;
    }
    /* wait returned -1: allocate a block of order n+1 and split it */
    int64_t p = tree_alloc(h, n + 1);
    if (p < 0) {
        bsem_signal(&h->tsem[n], 0, 1);                       /* failure must be signalled */
        return -1;
    }
    set_state(h, n + 1, (uint64_t)p, ST_PARTIAL);            /* busy -> partial */
    set_state(h, n, 2 * (uint64_t)p + 1, ST_AVAIL);          /* one child busy -> available */
    fix_up(h, n + 1, (uint64_t)p);
    bsem_signal(&h->tsem[n], 1, 1);                           /* notify the new available block */
    return 2 * p;                                             /* the other child is ours (busy) */
}

/* TBuddy free of node i at order n with the cascade of R-19. */
static void tree_free(ora_heap* h, int n, uint64_t i) {
    for (;;) {
        uint64_t b = i ^ 1;
        int has_buddy = (n < h->L) && node_inside(h, n, b);  /* R-30: forest roots have no buddy */
        if (has_buddy && bsem_trywait(&h->tsem[n], 1)) {     /* merge only if try-wait succeeds */
            if (h->st[n][b] == ST_AVAIL) {                    /* buddy available -> busy */
                set_state(h, n, b, ST_BUSY);
                i >>= 1; n += 1;                              /* merged: free the parent (cascade) */
                set_state(h, n, i, ST_BUSY);
                continue;
            }
            bsem_signal(&h->tsem[n], 1, 0);                   /* transition failed: signal back */
        }
        set_state(h, n, i, ST_AVAIL);                         /* busy -> available */
        fix_up(h, n, i);
        bsem_signal(&h->tsem[n], 1, 0);
        return;
    }
}

/* ------------------------------------------------------------------------- */
/* Heap creation.                                                            */
/* ------------------------------------------------------------------------- */
static void ora_heap_destroy_impl(ora_heap* h);

ora_heap* ora_heap_create(const ora_layout* lay, uint64_t bytes) {
    if (!lay || lay->page == 0 || (lay->page & (lay->page - 1)) || lay->chunk_pages == 0 ||
        lay->chunk_pages > 64 || (lay->chunk_pages & (lay->chunk_pages - 1)) ||
        lay->min_class == 0 || (lay->min_class & (lay->min_class - 1)) ||
        lay->bin_max < lay->min_class || (lay->bin_max & (lay->bin_max - 1)) ||
        lay->bin_max > lay->page)
        return NULL;
    if (lay->paper_layout && (lay->page != 4096 || lay->chunk_pages != 64 || lay->bin_max > 1024))
        return NULL;
    ora_heap* h = (ora_heap*)calloc(1, sizeof *h);
    h->lay = *lay;
    /* R-30: usable size = bytes rounded down to a whole number of chunks */
    uint64_t cbytes = (uint64_t)lay->page * lay->chunk_pages;
    h->nchunks = bytes / cbytes;
    if (h->nchunks == 0) { free(h); return NULL; }
    h->pages = h->nchunks * lay->chunk_pages;
    h->heap_bytes = h->pages * lay->page;
    h->L = 0;
    while ((1ull << h->L) < h->pages) h->L++;
    h->chunk_order = ilog2_u64(lay->chunk_pages);
    h->ncls = ilog2_u64(lay->bin_max) - ilog2_u64(lay->min_class) + 1;
    uint32_t maxslots = 0;
    for (int c = 0; c < h->ncls; c++) {
        uint32_t sz = lay->min_class << c;
        if (lay->paper_layout) {
            /* 128 B in-band header; body = page - 128; sizes <= 128 also use
               the 128 B tail appended to the bin (R-11) */
            h->body_slots[c] = (lay->page - 128) / sz;
            h->slots[c] = h->body_slots[c] + (sz <= 128 ? 128 / sz : 0);
        } else {
            h->body_slots[c] = h->slots[c] = lay->page / sz;
        }
        if (h->slots[c] > maxslots) maxslots = h->slots[c];
    }
    h->words = (maxslots + 63) / 64;
    h->hdr_pages = lay->paper_layout ? 2 : 0;
    h->usable_pages = lay->chunk_pages - h->hdr_pages;
    for (int n = 0; n <= h->L; n++) {
        uint64_t cnt = 1ull << (h->L - n);
        h->st[n] = (uint8_t*)calloc(cnt, 1);        /* all BUSY */
        bset_init(&h->av[n], cnt);
    }
    /* R-30: binary decomposition of the usable pages into maximal aligned roots */
    uint64_t off = 0;
    for (int n = h->L; n >= 0; n--) {
        if (h->pages - off >= (1ull << n)) {
            set_state(h, n, off >> n, ST_AVAIL);
            h->tsem[n].C += 1;
            fix_up(h, n, off >> n);
            off += 1ull << n;
        }
    }
    h->kind = (uint8_t*)calloc(h->pages, 1);
    h->aux = (uint8_t*)calloc(h->pages, 1);
    h->bits = (uint64_t*)calloc(h->pages * h->words, 8);
    h->freecnt = (uint32_t*)calloc(h->pages, 4);
    h->chunk_owned = (uint8_t*)calloc(h->nchunks, 1);
    h->chunk_used = (uint64_t*)calloc(h->nchunks, 8);
    for (int c = 0; c < h->ncls; c++) bset_init(&h->nonfull[c], h->pages);
    bset_init(&h->chunk_free, h->nchunks);
    return h;
}

static void ora_heap_destroy_impl(ora_heap* h) {
    if (!h) return;
    for (int n = 0; n <= h->L; n++) { free(h->st[n]); bset_free(&h->av[n]); }
    for (int c = 0; c < h->ncls; c++) bset_free(&h->nonfull[c]);
    bset_free(&h->chunk_free);
    free(h->kind); free(h->aux); free(h->bits); free(h->freecnt);
    free(h->chunk_owned); free(h->chunk_used);
    free(h);
}
void ora_heap_destroy(ora_heap* h) { ora_heap_destroy_impl(h); }

/* ------------------------------------------------------------------------- */
/* UAlloc: chunk pages and bins.                              */
/* ------------------------------------------------------------------------- */
static uint64_t usable_mask(const ora_heap* h) {
    uint64_t all = h->lay.chunk_pages == 64 ? ~0ull : ((1ull << h->lay.chunk_pages) - 1);
    uint64_t hdr = (1ull << h->hdr_pages) - 1;
    return all & ~hdr;
}

/* A bin page from the arena's chunks; on GROW a new chunk from TBuddy
 * (P:L1076-1092).  Returns the page index or -1. */
static int64_t page_alloc(ora_heap* h) {
    uint32_t upc = h->usable_pages;
    if (bsem_wait(&h->psem, 1, upc) == ACQUIRED) {
        int64_t k = bset_first(&h->chunk_free);                 /* lowest chunk with a free bin */
        if (k < 0) { fprintf(stderr, "oracle: page semaphore mismatch\n"); abort(); }
        uint64_t freem = usable_mask(h) & ~h->chunk_used[k];
        uint64_t j = (uint64_t)__builtin_ctzll(freem);          /* lowest free page of that chunk */
        h->chunk_used[k] |= 1ull << j;
        if (!(usable_mask(h) & ~h->chunk_used[k])) bset_clear(&h->chunk_free, (uint64_t)k);
        return (int64_t)((uint64_t)k * h->lay.chunk_pages + j);
    }
    int64_t node = tree_alloc(h, h->chunk_order);               /* a new chunk from TBuddy */
    if (node < 0) { bsem_signal(&h->psem, 0, upc - 1); return -1; }
    reserve_add(h, h->lay.chunk_pages);
    h->n_chunk_grow++;
    uint64_t k = (uint64_t)node;                                /* chunk index == node index at chunk order */
    h->chunk_owned[k] = 1;
    uint64_t base = k * h->lay.chunk_pages;
    for (uint32_t j = 0; j < h->lay.chunk_pages; j++)
        h->kind[base + j] = (j < h->hdr_pages) ? PK_CHUNK_HDR : PK_CHUNK_FREE;
    uint64_t j = h->hdr_pages;                                  /* take the lowest usable page */
    h->chunk_used[k] = ((1ull << h->hdr_pages) - 1) | (1ull << j);
    if (usable_mask(h) & ~h->chunk_used[k]) bset_set(&h->chunk_free, k);
    bsem_signal(&h->psem, upc - 1, upc - 1);
    return (int64_t)(base + j);
}

/* Return a page to its chunk; an empty chunk goes back to TBuddy (R-23). */
static void page_free(ora_heap* h, uint64_t p) {
    uint64_t k = p / h->lay.chunk_pages, j = p % h->lay.chunk_pages;
    h->kind[p] = PK_CHUNK_FREE;
    h->chunk_used[k] &= ~(1ull << j);
    bset_set(&h->chunk_free, k);
    bsem_signal(&h->psem, 1, 0);
    if ((h->chunk_used[k] & usable_mask(h)) == 0) {
        if (!bsem_trywait(&h->psem, h->usable_pages)) { fprintf(stderr, "oracle: chunk trywait\n"); abort(); }
        bset_clear(&h->chunk_free, k);
        h->chunk_owned[k] = 0;
        h->chunk_used[k] = 0;
        uint64_t base = k * h->lay.chunk_pages;
        for (uint32_t q = 0; q < h->lay.chunk_pages; q++) h->kind[base + q] = PK_TREE;
        h->n_chunk_reclaim++;
        h->reserved_pages -= h->lay.chunk_pages;
        tree_free(h, h->chunk_order, k);
    }
}

static uint64_t slot_offset(const ora_heap* h, uint64_t p, int c, uint32_t s) {
    uint32_t sz = h->lay.min_class << c;
    if (!h->lay.paper_layout) return p * h->lay.page + (uint64_t)s * sz;
    if (s < h->body_slots[c]) return p * h->lay.page + 128 + (uint64_t)s * sz;
    /* R-11: tail t (bin t+2) sits at chunk offset 128+128t (t<31) or 4096+128+128(t-31) */
    uint64_t k = p / h->lay.chunk_pages, t = p % h->lay.chunk_pages - 2;
    uint64_t cbase = k * h->lay.chunk_pages * h->lay.page;
    uint64_t toff = t < 31 ? 128 + 128 * t : h->lay.page + 128 + 128 * (t - 31);
    return cbase + toff + (uint64_t)(s - h->body_slots[c]) * sz;
}

static int bit_get(const ora_heap* h, uint64_t p, uint32_t s) { return (h->bits[p * h->words + s / 64] >> (s % 64)) & 1; }
static void bit_put(ora_heap* h, uint64_t p, uint32_t s, int v) {
    uint64_t* w = &h->bits[p * h->words + s / 64];
    if (v) *w |= 1ull << (s % 64); else *w &= ~(1ull << (s % 64));
}

/* Bin allocation of class c: two-stage. */
static uint64_t bin_alloc(ora_heap* h, int c) {
    uint32_t slots = h->slots[c];
    if (bsem_wait(&h->csem[c], 1, slots) == ACQUIRED) {
        int64_t p = bset_first(&h->nonfull[c]);                 /* R-20: lowest-address bin */
        if (p < 0) { fprintf(stderr, "oracle: class semaphore mismatch\n"); abort(); }
        uint32_t s = 0;
        while (bit_get(h, (uint64_t)p, s)) s++;                 /* lowest zero bit */
        bit_put(h, (uint64_t)p, s, 1);
        if (--h->freecnt[p] == 0) bset_clear(&h->nonfull[c], (uint64_t)p);
        return slot_offset(h, (uint64_t)p, c, s);
    }
    int64_t p = page_alloc(h);                                  /* wait returned -1: a new bin */
    if (p < 0) { bsem_signal(&h->csem[c], 0, slots - 1); return ORA_NULL; }
    h->n_bin_grow++;
    h->kind[p] = PK_BIN;
    h->aux[p] = (uint8_t)c;
    memset(&h->bits[(uint64_t)p * h->words], 0, 8 * h->words);
    bit_put(h, (uint64_t)p, 0, 1);                              /* our slot */
    h->freecnt[p] = slots - 1;
    if (slots > 1) bset_set(&h->nonfull[c], (uint64_t)p);
    bsem_signal(&h->csem[c], slots - 1, slots - 1);
    return slot_offset(h, (uint64_t)p, c, 0);
}

/* Map a bin offset back to (page, class, slot); -1 when it is not a slot. */
static int bin_locate(const ora_heap* h, uint64_t off, uint64_t* pp, int* cc, uint32_t* ss) {
    uint64_t p = off / h->lay.page, in = off % h->lay.page;
    if (p >= h->pages) return -1;
    if (h->kind[p] == PK_BIN) {
        int c = h->aux[p];
        uint32_t sz = h->lay.min_class << c;
        uint64_t hdr = h->lay.paper_layout ? 128 : 0;
        if (in < hdr || (in - hdr) % sz) return -1;
        uint64_t s = (in - hdr) / sz;
        if (s >= h->body_slots[c]) return -1;
        *pp = p; *cc = c; *ss = (uint32_t)s;
        return 0;
    }
    if (h->lay.paper_layout && h->kind[p] == PK_CHUNK_HDR) {
        uint64_t k = p / h->lay.chunk_pages, j = p % h->lay.chunk_pages;
        if (in < 128) return -1;
        uint64_t t = (j == 0 ? 0 : 31) + (in - 128) / 128, w = (in - 128) % 128;
        uint64_t bp = k * h->lay.chunk_pages + 2 + t;
        if (h->kind[bp] != PK_BIN) return -1;
        int c = h->aux[bp];
        uint32_t sz = h->lay.min_class << c;
        if (sz > 128 || w % sz) return -1;
        *pp = bp; *cc = c; *ss = h->body_slots[c] + (uint32_t)(w / sz);
        return 0;
    }
    return -1;
}

/* ------------------------------------------------------------------------- */
/* Front end: malloc / free.                                     */
/* ------------------------------------------------------------------------- */

/* Size -> class (R-12..R-15).  Returns 0 = NULL request, 1 = bin
 * (class index in *cls), 2 = tree (order in *order). */
int ora_classify(const ora_heap* h, uint64_t n, int* cls, int* order) {
    if (n == 0 || n > h->heap_bytes) return 0;                  /* R-15 */
    uint64_t c = ceil_pow2(n < h->lay.min_class ? h->lay.min_class : n);   /* R-14: ceil */
    if (c <= h->lay.bin_max) { *cls = ilog2_u64(c) - ilog2_u64(h->lay.min_class); return 1; }
    int o = ilog2_u64(c) - ilog2_u64(h->lay.page);
    if (o < 0) o = 0;                                           /* R-12: 2 KB -> a 4 KB page (paper layout) */
    if (o > h->L) return 0;
    *order = o;
    return 2;
}

uint64_t ora_malloc(ora_heap* h, uint64_t n) {
    int c = 0, o = 0;
    h->n_malloc++;
    int route = ora_classify(h, n, &c, &o);
    uint64_t off = ORA_NULL;
    if (route == 1) off = bin_alloc(h, c);
    else if (route == 2) {
        int64_t node = tree_alloc(h, o);
        if (node >= 0) {
            uint64_t p = (uint64_t)node << o;
            h->kind[p] = PK_TREE_HEAD;                          /* R-18: order stored at the head page */
            h->aux[p] = (uint8_t)o;
            reserve_add(h, 1ll << o);
            off = p * h->lay.page;
        }
    }
    if (off == ORA_NULL) h->n_fail++;
    return off;
}

/* Returns 0 on success, 1 for free(NULL) (no-op, R-16), negative on an invalid free. */
int ora_free(ora_heap* h, uint64_t off) {
    if (off == ORA_NULL) return 1;
    if (off >= h->heap_bytes) return -1;
    uint64_t p = off / h->lay.page;
    if (h->kind[p] == PK_TREE_HEAD && off % h->lay.page == 0) {  /* page aligned: TBuddy */
        int o = h->aux[p];
        h->kind[p] = PK_TREE;
        h->reserved_pages -= 1ull << o;
        tree_free(h, o, p >> o);
        h->n_free++;
        return 0;
    }
    uint64_t bp; int c; uint32_t s;
    if (bin_locate(h, off, &bp, &c, &s) != 0) return -2;
    if (!bit_get(h, bp, s)) return -3;                          /* double free */
    bit_put(h, bp, s, 0);
    uint32_t slots = h->slots[c];
    if (h->freecnt[bp]++ == 0) bset_set(&h->nonfull[c], bp);   /* exhausted bin back in the list */
    bsem_signal(&h->csem[c], 1, 0);
    h->n_free++;
    if (h->freecnt[bp] == slots) {                              /* last block freed: drop the bin */
        if (!bsem_trywait(&h->csem[c], slots)) { fprintf(stderr, "oracle: bin trywait\n"); abort(); }  /* R-22 */
        bset_clear(&h->nonfull[c], bp);
        h->freecnt[bp] = 0;
        memset(&h->bits[bp * h->words], 0, 8 * h->words);
        h->n_bin_reclaim++;
        page_free(h, bp);
    }
    return 0;
}

/* Pages held outside the free tree (allocated blocks and chunks). */
uint64_t ora_reserved_pages(const ora_heap* h) { return h->reserved_pages; }

/* ------------------------------------------------------------------------- */
/* Invariants at quiescence.                    */
/* Returns 0 when all hold, else a positive code and a message.               */
/* ------------------------------------------------------------------------- */
int ora_check_invariants(const ora_heap* h, char* msg, int msglen) {
#define FAILF(code, ...) do { if (msg) snprintf(msg, (size_t)msglen, __VA_ARGS__); return code; } while (0)
    uint64_t avail_pages = 0;
    for (int n = 0; n <= h->L; n++) {
        uint64_t cnt = 1ull << (h->L - n), navail = 0;
        for (uint64_t i = 0; i < cnt; i++) {
            uint8_t s = h->st[n][i];
            if (s == ST_AVAIL) {
                navail++;
                if (!node_inside(h, n, i)) FAILF(1, "available node outside heap n=%d i=%llu", n, (unsigned long long)i);
                /* property 1: two siblings cannot both be available */
                if (n < h->L && node_inside(h, n, i ^ 1) && h->st[n][i ^ 1] == ST_AVAIL)
                    FAILF(2, "siblings both available n=%d i=%llu", n, (unsigned long long)i);
                /* property 2: the sub-tree of an available node is all busy */
                for (int k = n - 1, w = 2; k >= 0; k--, w *= 2)
                    for (uint64_t j = i << (n - k); j < ((i + 1) << (n - k)); j++)
                        if (h->st[k][j] != ST_BUSY) FAILF(3, "non-busy below available n=%d", n);
            } else if (n > 0) {
                uint8_t l = h->st[n - 1][2 * i], r = h->st[n - 1][2 * i + 1];
                int want = (l != ST_BUSY || r != ST_BUSY) ? ST_PARTIAL : ST_BUSY;
                if (s != want) FAILF(4, "partial/busy state wrong n=%d i=%llu", n, (unsigned long long)i);
            }
            if (bset_test(&h->av[n], i) != (s == ST_AVAIL)) FAILF(5, "avail index wrong");
        }
        if (h->tsem[n].C != (int64_t)navail || h->tsem[n].E || h->tsem[n].R)
            FAILF(6, "tree semaphore %d: C=%lld avail=%llu", n, (long long)h->tsem[n].C, (unsigned long long)navail);
        avail_pages += navail << n;
    }
    if (avail_pages + h->reserved_pages != h->pages) FAILF(7, "reserved accounting");
    int64_t freeslots[32] = {0}, freepages = 0;
    for (uint64_t k = 0; k < h->nchunks; k++) {
        uint64_t base = k * h->lay.chunk_pages;
        if (!h->chunk_owned[k]) {
            if (h->chunk_used[k]) FAILF(8, "unowned chunk with used pages");
            if (bset_test(&h->chunk_free, k)) FAILF(9, "unowned chunk indexed");
            continue;
        }
        if (h->st[h->chunk_order][k] != ST_BUSY) FAILF(10, "owned chunk not busy in the tree");
        uint64_t um = usable_mask(h);
        if (bset_test(&h->chunk_free, k) != ((um & ~h->chunk_used[k]) != 0)) FAILF(11, "chunk index");
        if (!(h->chunk_used[k] & um)) FAILF(12, "empty chunk not reclaimed");
        for (uint32_t j = 0; j < h->lay.chunk_pages; j++) {
            uint64_t p = base + j;
            int used = (h->chunk_used[k] >> j) & 1;
            if (j < h->hdr_pages) { if (!used || h->kind[p] != PK_CHUNK_HDR) FAILF(13, "hdr page"); continue; }
            if (!used) { if (h->kind[p] != PK_CHUNK_FREE) FAILF(14, "free page kind"); freepages++; continue; }
            if (h->kind[p] != PK_BIN) FAILF(15, "used page not a bin");
            int c = h->aux[p];
            uint32_t cnt = 0;
            for (uint32_t s = 0; s < h->slots[c]; s++) cnt += !bit_get(h, p, s);
            if (cnt != h->freecnt[p]) FAILF(16, "bin free counter");
            if (cnt == h->slots[c]) FAILF(17, "empty bin not reclaimed");
            if (bset_test(&h->nonfull[c], p) != (cnt > 0)) FAILF(18, "nonfull index");
            freeslots[c] += cnt;
        }
    }
    for (int c = 0; c < h->ncls; c++)
        if (h->csem[c].C != freeslots[c] || h->csem[c].E || h->csem[c].R)
            FAILF(19, "class semaphore %d: C=%lld free=%lld", c, (long long)h->csem[c].C, (long long)freeslots[c]);
    if (h->psem.C != freepages || h->psem.E || h->psem.R) FAILF(20, "page semaphore");
    return 0;
#undef FAILF
}

/* ------------------------------------------------------------------------- */
/* Canonical snapshot (format in include/ga.h, "Canonical snapshot").          */
/* Returns the number of bytes (written only if cap suffices).                */
/* ------------------------------------------------------------------------- */
typedef struct { uint8_t* p; uint64_t n, cap; } wbuf;
static void wput(wbuf* w, const void* src, uint64_t len) {
    if (w->n + len <= w->cap && w->p) memcpy(w->p + w->n, src, len);
    w->n += len;
}
static void wput_u64(wbuf* w, uint64_t v) { wput(w, &v, 8); }
static void wput_i64(wbuf* w, int64_t v) { wput(w, &v, 8); }

uint64_t ora_snapshot(const ora_heap* h, uint8_t* out, uint64_t cap) {
    wbuf w = { out, 0, cap };
    wput_u64(&w, 0x31304e5341534147ull);                        /* "GASNAP01" */
    wput_u64(&w, h->heap_bytes);
    wput_u64(&w, h->pages);
    wput_u64(&w, (uint64_t)h->lay.page | ((uint64_t)(h->L + 1) << 32));
    uint32_t extra = h->lay.snap_max_class > h->lay.bin_max
                     ? (uint32_t)(ilog2_u64(h->lay.snap_max_class) - ilog2_u64(h->lay.bin_max)) : 0;
    wput_u64(&w, (uint64_t)h->lay.min_class | ((uint64_t)h->ncls << 32) | ((uint64_t)extra << 40) |
                 ((uint64_t)h->lay.chunk_pages << 48));
    /* per-page kind byte */
    uint8_t* kb = (uint8_t*)malloc(h->pages);
    memset(kb, 0, h->pages);                                    /* 0x00: inside a free tree node */
    for (int n = 0; n <= h->L; n++)
        for (uint64_t i = 0; i < (1ull << (h->L - n)); i++)
            if (h->st[n][i] == ST_AVAIL) kb[i << n] = (uint8_t)(0x40 | n);
    for (uint64_t p = 0; p < h->pages; p++) {
        if (h->kind[p] == PK_TREE_HEAD) {
            int o = h->aux[p];
            kb[p] = (uint8_t)(0x80 | o);
            for (uint64_t q = p + 1; q < p + (1ull << o); q++) kb[q] = 0x01;
        } else if (h->kind[p] == PK_CHUNK_FREE) kb[p] = 0x02;
        else if (h->kind[p] == PK_CHUNK_HDR) kb[p] = 0x03;
        else if (h->kind[p] == PK_BIN) kb[p] = (uint8_t)(0x10 | h->aux[p]);
    }
    wput(&w, kb, h->pages);
    /* per bin page (ascending): its bitmap, slots bits, LSB first, padded to bytes */
    for (uint64_t p = 0; p < h->pages; p++) {
        if (h->kind[p] != PK_BIN) continue;
        int c = h->aux[p];
        uint32_t nb = (h->slots[c] + 7) / 8;
        uint8_t tmp[64];
        memset(tmp, 0, sizeof tmp);
        for (uint32_t s = 0; s < h->slots[c]; s++) if (bit_get(h, p, s)) tmp[s / 8] |= (uint8_t)(1u << (s % 8));
        wput(&w, tmp, nb);
    }
    free(kb);
    /* per level: availability bitmap, 2^(L-n) bits LSB first, padded to bytes */
    for (int n = 0; n <= h->L; n++) {
        uint64_t cnt = 1ull << (h->L - n), nb = (cnt + 7) / 8;
        uint8_t* tmp = (uint8_t*)calloc(nb, 1);
        for (uint64_t i = 0; i < cnt; i++) if (h->st[n][i] == ST_AVAIL) tmp[i / 8] |= (uint8_t)(1u << (i % 8));
        wput(&w, tmp, nb);
        free(tmp);
    }
    /* semaphores: per class (sum C, max |E-R|), page semaphore, per order (C, E-R) */
    for (int c = 0; c < h->ncls; c++) {
        wput_i64(&w, h->csem[c].C);
        int64_t d = h->csem[c].E - h->csem[c].R;
        wput_i64(&w, d < 0 ? -d : d);
    }
    for (uint32_t s = 0; s < extra; s++) { wput_i64(&w, 0); wput_i64(&w, 0); }
    wput_i64(&w, h->psem.C);
    { int64_t d = h->psem.E - h->psem.R; wput_i64(&w, d < 0 ? -d : d); }
    for (int n = 0; n <= h->L; n++) { wput_i64(&w, h->tsem[n].C); wput_i64(&w, h->tsem[n].E - h->tsem[n].R); }
    wput_u64(&w, 0);                                            /* pending reclamation: eager here */
    return w.n;
}

/* ------------------------------------------------------------------------- */
/* Trace runner.  sizes: u32[R][T], round-major, */
/* 0 = no malloc.  D == 1 (churn): at round r each thread, in thread order,   */
/* frees the block it got at round r-1 and then mallocs size[r][t]; round R   */
/* is a free-all round.  D == 0 (phase split): at round r every thread        */
/* mallocs, then every round-r block is freed.                                */
/* log (optional): 16 B records at 2*(round*T+tid)+op (op 0 malloc, 1 free):  */
/*   u64 off (~0 = NULL / nothing), u32 size_req, u32 tid | round<<20 | op<<31 */
/* Peaks are taken at phase boundaries (after the mallocs of a round).        */
/* ------------------------------------------------------------------------- */
typedef struct {
    uint64_t n_malloc, n_malloc_fail, n_free, calls;
    uint64_t peak_live_bytes, peak_reserved_bytes, peak_reserved_any_bytes;
    uint64_t final_reserved_bytes;
    uint64_t n_bin_grow, n_chunk_grow, n_bin_reclaim, n_chunk_reclaim;
    int64_t invariant_error;
} ora_trace_stats;

typedef struct { uint64_t off; uint32_t size; uint32_t meta; } ora_rec;

static void logrec(ora_rec* log, uint64_t T, uint64_t r, uint64_t tid, int op, uint64_t off, uint32_t sz) {
    if (!log) return;
    ora_rec* e = &log[2 * (r * T + tid) + (uint64_t)op];
    e->off = off; e->size = sz;
    e->meta = (off == ORA_NULL && sz == 0) ? 0 : ((uint32_t)tid | ((uint32_t)r << 20) | ((uint32_t)op << 31));
}

int ora_run_trace(const ora_layout* lay, uint64_t heap_bytes, const uint32_t* sizes,
                  uint64_t R, uint64_t T, uint64_t D, ora_rec* log, uint8_t* ok,
                  ora_trace_stats* st, int check_each_round) {
    if ((log && T >= (1u << 20)) || R >= 2047 || D > 1) return -1;
    ora_heap* h = ora_heap_create(lay, heap_bytes);
    if (!h) return -2;
    memset(st, 0, sizeof *st);
    uint64_t* blk = (uint64_t*)malloc(8 * T);                  /* block held per thread */
    uint32_t* bsz = (uint32_t*)malloc(4 * T);
    for (uint64_t i = 0; i < T; i++) { blk[i] = ORA_NULL; bsz[i] = 0; }
    uint64_t live = 0;
    char msg[256];
    uint64_t rounds = D ? R + 1 : R;                           /* D == 1: + free-all round */
    for (uint64_t r = 0; r < rounds; r++) {
        for (uint64_t t = 0; t < T; t++) {
            if (D == 1) {                                      /* free the round r-1 block */
                if (blk[t] != ORA_NULL) {
                    if (ora_free(h, blk[t]) != 0) { st->invariant_error = -100; goto out; }
                    live -= bsz[t]; st->n_free++;
                    logrec(log, T, r, t, 1, blk[t], bsz[t]);
                    blk[t] = ORA_NULL;
                } else logrec(log, T, r, t, 1, ORA_NULL, 0);
                if (r == R) { logrec(log, T, r, t, 0, ORA_NULL, 0); continue; }
            }
            uint32_t n = sizes[r * T + t];
            if (n) {
                uint64_t off = ora_malloc(h, n);
                st->n_malloc++;
                if (off == ORA_NULL) st->n_malloc_fail++;
                else { live += n; blk[t] = off; bsz[t] = n; }
                if (ok) ok[r * T + t] = off != ORA_NULL;
                logrec(log, T, r, t, 0, off, n);
            } else logrec(log, T, r, t, 0, ORA_NULL, 0);
        }
        /* phase boundary */
        if (live > st->peak_live_bytes) st->peak_live_bytes = live;
        uint64_t rb = h->reserved_pages * h->lay.page;
        if (rb > st->peak_reserved_bytes) st->peak_reserved_bytes = rb;
        if (D == 0) {
            for (uint64_t t = 0; t < T; t++) {
                if (blk[t] != ORA_NULL) {
                    if (ora_free(h, blk[t]) != 0) { st->invariant_error = -100; goto out; }
                    live -= bsz[t]; st->n_free++;
                    logrec(log, T, r, t, 1, blk[t], bsz[t]);
                    blk[t] = ORA_NULL;
                } else logrec(log, T, r, t, 1, ORA_NULL, 0);
            }
        }
        if (check_each_round) {
            int e = ora_check_invariants(h, msg, sizeof msg);
            if (e) { st->invariant_error = e; fprintf(stderr, "oracle invariant (round %llu): %s\n", (unsigned long long)r, msg); goto out; }
        }
    }
    st->invariant_error = ora_check_invariants(h, msg, sizeof msg);
    if (st->invariant_error) fprintf(stderr, "oracle invariant (end): %s\n", msg);
out:
    st->calls = st->n_malloc + st->n_free;
    st->peak_reserved_any_bytes = h->peak_reserved_pages * h->lay.page;
    st->final_reserved_bytes = h->reserved_pages * h->lay.page;
    st->n_bin_grow = h->n_bin_grow; st->n_chunk_grow = h->n_chunk_grow;
    st->n_bin_reclaim = h->n_bin_reclaim; st->n_chunk_reclaim = h->n_chunk_reclaim;
    free(blk); free(bsz);
    ora_heap_destroy(h);
    return 0;
}

/* ------------------------------------------------------------------------- */
/* Allocation-log checker, build layout, same trace        */
/* semantics as ora_run_trace.  Checks every successful block: inside the     */
/* heap, 16 B aligned, aligned to its block length relative to the heap base  */
/* (bins: the class; tree: the block size, R-31); every free record names the */
/* block the thread holds; after each round's mallocs the held set (survivors */
/* + new blocks; blocks freed in the round excluded) is pairwise disjoint;    */
/* meta words name their own (tid, round, op).  Returns 0 or an error code.   */
/* ------------------------------------------------------------------------- */
typedef struct {
    uint64_t n_malloc, n_ok, n_fail, n_free;
    uint64_t peak_live_bytes;
    uint64_t bad_index;   /* record index (or round) of the first error */
} ora_check_stats;

typedef struct { uint64_t lo, hi; } ivl;
static int ivl_cmp(const void* a, const void* b) {
    const ivl* x = (const ivl*)a; const ivl* y = (const ivl*)b;
    return x->lo < y->lo ? -1 : x->lo > y->lo ? 1 : 0;
}

/* Bytes a successful request of n occupies: its class, a whole page
   at least on the tree path. */
static uint64_t block_len(const ora_layout* lay, uint64_t n) {
    uint64_t c = ceil_pow2(n < lay->min_class ? lay->min_class : n);
    if (c <= lay->bin_max) return c;
    return c < lay->page ? lay->page : c;
}

int ora_check_log(const ora_layout* lay, uint64_t heap_bytes, const ora_rec* log,
                  uint64_t R, uint64_t T, uint64_t D, ora_check_stats* cs) {
    memset(cs, 0, sizeof *cs);
    if (lay->paper_layout || D > 1) return 90;
    uint64_t* held = (uint64_t*)malloc(8 * T);
    uint32_t* hsz = (uint32_t*)malloc(4 * T);
    for (uint64_t i = 0; i < T; i++) { held[i] = ORA_NULL; hsz[i] = 0; }
    ivl* iv = (ivl*)malloc(sizeof(ivl) * T + 16);
    uint64_t live = 0;
    int err = 0;
    uint64_t rounds = D ? R + 1 : R;
#define BAD(code, idx) do { err = (code); cs->bad_index = (idx); goto done; } while (0)
    for (uint64_t r = 0; r < rounds; r++) {
        for (uint64_t t = 0; t < T; t++) {
            uint64_t im = 2 * (r * T + t), ifr = im + 1;
            const ora_rec* m = &log[im];
            const ora_rec* f = &log[ifr];
            if (D == 1) {
                if (f->off != held[t]) BAD(11, ifr);
                if (held[t] != ORA_NULL) {
                    if (f->size != hsz[t]) BAD(13, ifr);
                    live -= hsz[t]; cs->n_free++; held[t] = ORA_NULL;
                }
                if (r == R) { if (m->off != ORA_NULL || m->size) BAD(5, im); continue; }
            }
            if (m->size) {
                cs->n_malloc++;
                if (m->off == ORA_NULL) cs->n_fail++;
                else {
                    cs->n_ok++;
                    uint64_t len = block_len(lay, m->size);
                    if (m->off + len > heap_bytes || m->off + len < m->off) BAD(1, im);
                    if (m->off % 16) BAD(2, im);
                    if (m->off % len) BAD(3, im);
                    held[t] = m->off; hsz[t] = m->size; live += m->size;
                }
            } else if (m->off != ORA_NULL) BAD(4, im);
        }
        uint64_t nv = 0;
        for (uint64_t i = 0; i < T; i++)
            if (held[i] != ORA_NULL) { iv[nv].lo = held[i]; iv[nv].hi = held[i] + block_len(lay, hsz[i]); nv++; }
        qsort(iv, nv, sizeof(ivl), ivl_cmp);
        for (uint64_t i = 1; i < nv; i++) if (iv[i].lo < iv[i - 1].hi) BAD(20, r);
        if (live > cs->peak_live_bytes) cs->peak_live_bytes = live;
        if (D == 0) {
            for (uint64_t t = 0; t < T; t++) {
                const ora_rec* f = &log[2 * (r * T + t) + 1];
                if (f->off != held[t]) BAD(12, 2 * (r * T + t) + 1);
                if (held[t] != ORA_NULL) { live -= hsz[t]; cs->n_free++; held[t] = ORA_NULL; }
            }
        }
    }
    for (uint64_t r = 0; r < rounds; r++)
        for (uint64_t t = 0; t < T; t++)
            for (int op = 0; op < 2; op++) {
                uint64_t i = 2 * (r * T + t) + (uint64_t)op;
                const ora_rec* e = &log[i];
                uint32_t want = (e->off == ORA_NULL && e->size == 0) ? 0
                              : ((uint32_t)t | ((uint32_t)r << 20) | ((uint32_t)op << 31));
                if (e->meta != want) BAD(30, i);
            }
done:
    free(held); free(hsz); free(iv);
    return err;
#undef BAD
}
