// ga_host.cu -- host side of the C ABI in include/ga.h.
//
// The host reserves the pool once (the cudaMalloc role of P:L352-356) and a
// separate metadata allocation (reading R-29: heap_bytes is pure payload).
// Initialisation, reset and quiesce are kernels on the caller's stream; stats,
// snapshot and reserved-page queries copy metadata back and compute on the host.
#include <cuda_runtime.h>

#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <new>
#include <vector>

#include "ga.h"
#include "ga_device_impl.cuh"
#include "ga_internal.h"

using namespace ga;

namespace {

constexpr uint64_t kAlign = 256;
constexpr uint64_t kBaseAlign = 2ull << 20;     // R-31: 2 MiB aligned base
constexpr int kSnapSpanSlots = 5;               // snapshot format: class entries 4 .. 64 KiB (include/ga.h)

inline uint64_t up(uint64_t x, uint64_t a) { return (x + a - 1) / a * a; }
inline uint64_t sem_word(int32_t C, int32_t D) { return ((uint64_t)(uint32_t)C << 32) | (uint32_t)(D + 0x80000000u); }

struct Carve {
    uint64_t off = 0;
    template <class T> uint64_t take(uint64_t count) { uint64_t o = off; off = up(off + count * sizeof(T), kAlign); return o; }
};

// quiesce step 1: every empty bin back to its chunk (and empty chunks to the tree)
__global__ void k_quiesce_bins(const ga_desc* h) {
    for (uint64_t p = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; p < h->pages; p += (uint64_t)gridDim.x * blockDim.x) {
        uint32_t k = h->kind[p];
        if ((k & 0xC0000000u) == kKindBin) bin_reclaim(h, p, 0);
    }
}
// quiesce step 2: chunks whose pages are all free go back to TBuddy
__global__ void k_quiesce_chunks(const ga_desc* h) {
    for (uint64_t ch = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; ch < h->nchunks; ch += (uint64_t)gridDim.x * blockDim.x) {
        if (h->chunk_owner[ch] != 0 && ld_rlx(&h->chunk_used[ch]) == 0) chunk_release(h, ch);
    }
}
// quiesce step 3: no candidate can remain (every empty bin was reclaimed)
__global__ void k_quiesce_clear(const ga_desc* h) {
    uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i < h->nchunks) h->chunk_cand[i] = 0;
    if (i < (uint64_t)h->n_arenas * h->ahb_words) h->ahb[(i / h->ahb_words) * kAhbPerArena * h->ahb_words + kAhbCnd * h->ahb_words + i % h->ahb_words] = 0;
}

inline int grid_for(uint64_t n) { uint64_t b = (n + 255) / 256; return (int)(b > 4096 ? 4096 : (b ? b : 1)); }

// One fused kernel resets every metadata array (a fill or a copy of the
// empty-heap image per segment, blockIdx.y = segment): ga_heap_reset is a
// single launch on the caller's stream.
struct FillSeg { void* p; const uint64_t* src; uint64_t n; uint64_t v; uint32_t bytes; };
constexpr int kMaxSegs = 16;
struct FillPlan { FillSeg s[kMaxSegs]; };
__global__ void __launch_bounds__(256) k_reset(FillPlan plan) {
    const FillSeg g = plan.s[blockIdx.y];
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < g.n; i += (uint64_t)gridDim.x * blockDim.x) {
        if (g.bytes == 8) ((uint64_t*)g.p)[i] = g.src ? g.src[i] : g.v;
        else ((uint32_t*)g.p)[i] = (uint32_t)g.v;
    }
}

ga_status init_heap(ga_heap_t h, cudaStream_t s) {
    const ga_desc& d = h->dev;
    FillPlan plan{};
    int n = 0;
    auto seg = [&](void* p, uint64_t cnt, uint64_t v, uint32_t bytes, const uint64_t* src = nullptr) {
        plan.s[n++] = FillSeg{p, src, cnt, v, bytes};
    };
    seg(d.bits, d.pages * kBinWords, ~0ull, 8);                  // all ones: no live bin
    seg(d.kind, d.pages, 0, 4);
    seg(d.chunk_used, d.nchunks, ~0ull, 8);                      // all ones: not owned
    seg(d.chunk_owner, d.nchunks, 0, 4);
    seg(d.chunk_nonfull, d.nchunks * kNcls, 0, 8);
    seg(d.chunk_cand, d.nchunks, 0, 8);
    seg(d.sem, (uint64_t)d.n_arenas * kNcls * kSemStride, sem_word(0, 0), 8);
    seg(d.psem, (uint64_t)d.n_arenas * kSemStride, sem_word(0, 0), 8);
    seg(d.hint, (uint64_t)d.n_arenas * kNcls, 0xFFFFFFFFu, 4);
    seg(d.ahb, h->ahb_total_words, 0, 8);
    seg(d.stats, kStatWords, 0, 8);
    seg(d.actr, (uint64_t)d.n_arenas * kActrStride, 0, 8);
    seg(d.lvl_hint, 48, 0, 4);
    seg(d.avail, h->avail_words, 0, 8, h->init_img);             // the empty tree (R-30)
    seg(d.tsem, (uint64_t)(d.L + 1) * kSemStride, 0, 8, h->init_img + h->avail_words);
    uint64_t most = 0;
    for (int i = 0; i < n; i++) most = plan.s[i].n > most ? plan.s[i].n : most;
    const uint64_t bx = (most + 255) / 256;
    k_reset<<<dim3((unsigned)(bx > 1184 ? 1184 : bx), n), 256, 0, s>>>(plan);
    return cudaGetLastError() == cudaSuccess ? GA_OK : GA_ECUDA;
}

// set bit i of a 3-level bitset image [w0 | w1 | w2] (section 3 of ga_device_impl.cuh)
void hb_host_set(std::vector<uint64_t>& img, uint64_t base, uint32_t n0, uint64_t i) {
    img[base + (i >> 6)] |= 1ull << (i & 63);
    uint64_t j = i >> 6;
    img[base + n0 + (j >> 6)] |= 1ull << (j & 63);
    uint64_t j1 = j >> 6;
    img[base + n0 + hb3_n1(n0) + (j1 >> 6)] |= 1ull << (j1 & 63);
}

}  // namespace

extern "C" {

const char* ga_status_str(ga_status s) {
    switch (s) {
        case GA_OK: return "ok";
        case GA_EINVAL: return "invalid argument";
        case GA_ENOMEM: return "out of device memory";
        case GA_ECUDA: return "CUDA error";
        case GA_EBUSY: return "busy";
    }
    return "unknown";
}

ga_status ga_layout(ga_layout_t* out) {
    if (!out) return GA_EINVAL;
    out->page = (uint32_t)kPage;
    out->chunk_pages = kChunkPages;
    out->min_class = 1u << kMinShift;
    out->bin_max = 1u << (kMinShift + kNbin - 1);
    out->n_classes = kNbin;
    out->bitmap_bits = 64 * kBinWords;
    out->n_span_classes = kNspan;
    out->span_max = kNspan ? (uint32_t)kPage << (kNspan - 1) : 0;
    return GA_OK;
}

ga_status ga_heap_create(int device, ga_stream_t stream, void* buf, size_t bytes, uint32_t flags, ga_heap_t* out) {
    if (!out) return GA_EINVAL;
    *out = nullptr;
    uint64_t cbytes = kPage * kChunkPages;
    uint64_t nchunks = bytes / cbytes;
    if (nchunks == 0) return GA_EINVAL;
    if (buf && ((uintptr_t)buf % kBaseAlign)) return GA_EINVAL;
    int prev = 0;
    if (cudaGetDevice(&prev) != cudaSuccess) return GA_ECUDA;
    if (cudaSetDevice(device) != cudaSuccess) return GA_EINVAL;
    cudaStream_t s = (cudaStream_t)stream;
    ga_heap_t h = new (std::nothrow) ga_heap_s();
    if (!h) return GA_ENOMEM;
    h->device = device;
    ga_desc& d = h->dev;
    d.pages = nchunks * kChunkPages;
    d.nchunks = nchunks;
    uint32_t L = 0;
    while ((1ull << L) < d.pages) L++;
    d.L = L;
    int nsm = 0;
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, device);
    d.n_arenas = nsm > 0 ? (uint32_t)nsm : 1;             // one arena per SM
    d.chunk_words = (uint32_t)((nchunks + 63) / 64);
    d.flags = flags;
    // tree levels
    uint64_t aw = 0;
    for (uint32_t n = 0; n <= L; n++) {
        uint64_t bits = 1ull << (L - n);
        d.lvl_words[n] = (uint32_t)((bits + 63) / 64);
        d.lvl_off[n] = aw;
        aw += hb3_words(d.lvl_words[n]);
    }
    h->avail_words = aw;
    d.ahb_words = hb3_words(d.chunk_words);
    h->ahb_total_words = (uint64_t)d.n_arenas * kAhbPerArena * d.ahb_words;
    Carve cv;
    uint64_t o_desc = cv.take<ga_desc>(1);
    uint64_t o_bits = cv.take<uint64_t>(d.pages * kBinWords);
    uint64_t o_kind = cv.take<uint32_t>(d.pages);
    uint64_t o_used = cv.take<uint64_t>(nchunks);
    uint64_t o_owner = cv.take<uint32_t>(nchunks);
    uint64_t o_nonfull = cv.take<uint64_t>(nchunks * kNcls);
    uint64_t o_cand = cv.take<uint64_t>(nchunks);
    uint64_t o_sem = cv.take<uint64_t>((uint64_t)d.n_arenas * kNcls * kSemStride);
    uint64_t o_psem = cv.take<uint64_t>((uint64_t)d.n_arenas * kSemStride);
    uint64_t o_hint = cv.take<uint32_t>((uint64_t)d.n_arenas * kNcls);
    uint64_t o_owned = cv.take<uint64_t>(h->ahb_total_words);
    uint64_t o_avail = cv.take<uint64_t>(aw);
    uint64_t o_tsem = cv.take<uint64_t>((uint64_t)(L + 1) * kSemStride);
    uint64_t o_stats = cv.take<uint64_t>(kStatWords);
    uint64_t o_actr = cv.take<uint64_t>((uint64_t)d.n_arenas * kActrStride);
    uint64_t o_lhint = cv.take<uint32_t>(48);
    uint64_t o_img = cv.take<uint64_t>(aw + (uint64_t)(L + 1) * kSemStride);
    h->meta_bytes = cv.off;
    if (cudaMalloc(&h->meta, h->meta_bytes) != cudaSuccess) { delete h; cudaSetDevice(prev); return GA_ENOMEM; }
    if (buf) d.base = (char*)buf;
    else {
        if (cudaMalloc(&h->pool_raw, d.pages * kPage + kBaseAlign) != cudaSuccess) {
            cudaFree(h->meta); delete h; cudaSetDevice(prev); return GA_ENOMEM;
        }
        d.base = (char*)up((uint64_t)(uintptr_t)h->pool_raw, kBaseAlign);
    }
    char* m = h->meta;
    h->ddesc = (ga_desc*)(m + o_desc);
    d.bits = (uint64_t*)(m + o_bits);
    d.kind = (uint32_t*)(m + o_kind);
    d.chunk_used = (uint64_t*)(m + o_used);
    d.chunk_owner = (uint32_t*)(m + o_owner);
    d.chunk_nonfull = (uint64_t*)(m + o_nonfull);
    d.chunk_cand = (uint64_t*)(m + o_cand);
    d.sem = (uint64_t*)(m + o_sem);
    d.psem = (uint64_t*)(m + o_psem);
    d.hint = (uint32_t*)(m + o_hint);
    d.ahb = (uint64_t*)(m + o_owned);
    d.avail = (uint64_t*)(m + o_avail);
    d.tsem = (uint64_t*)(m + o_tsem);
    d.stats = (uint64_t*)(m + o_stats);
    d.actr = (uint64_t*)(m + o_actr);
    h->init_img = (uint64_t*)(m + o_img);
    d.lvl_hint = (uint32_t*)(m + o_lhint);
    // empty heap: the binary decomposition of the pages into maximal aligned roots (R-30)
    h->avail_init.assign(aw, 0ull);
    h->tsem_init.assign((uint64_t)(L + 1) * kSemStride, 0ull);
    std::vector<int32_t> roots(L + 1, 0);
    uint64_t off = 0;
    for (int n = (int)L; n >= 0; n--) {
        if (d.pages - off >= (1ull << n)) {
            hb_host_set(h->avail_init, d.lvl_off[n], d.lvl_words[n], off >> n);
            roots[n]++;
            off += 1ull << n;
        }
    }
    for (uint32_t n = 0; n <= L; n++) h->tsem_init[(uint64_t)n * kSemStride] = sem_word(roots[n], 0);
    // the empty-tree image lives on the device (reset copies it from there);
    // the descriptor changes only with ga_debug_attach
    ga_status st = GA_OK;
    if (cudaMemcpyAsync(h->init_img, h->avail_init.data(), aw * 8, cudaMemcpyHostToDevice, s) != cudaSuccess ||
        cudaMemcpyAsync(h->init_img + aw, h->tsem_init.data(), h->tsem_init.size() * 8, cudaMemcpyHostToDevice, s) != cudaSuccess ||
        cudaMemcpyAsync(h->ddesc, &h->dev, sizeof(ga_desc), cudaMemcpyHostToDevice, s) != cudaSuccess)
        st = GA_ECUDA;
    if (st == GA_OK) st = init_heap(h, s);
    // the host images are read by the async copies above: keep them until done
    if (st == GA_OK && cudaStreamSynchronize(s) != cudaSuccess) st = GA_ECUDA;
    if (st != GA_OK) { ga_heap_destroy(h); cudaSetDevice(prev); return st; }
    cudaSetDevice(prev);
    *out = h;
    return GA_OK;
}

ga_status ga_heap_destroy(ga_heap_t h) {
    if (!h) return GA_EINVAL;
    int prev = 0;
    cudaGetDevice(&prev);
    cudaSetDevice(h->device);
    cudaDeviceSynchronize();
    if (h->pool_raw) cudaFree(h->pool_raw);
    if (h->meta) cudaFree(h->meta);
    if (h->scratch) cudaFree(h->scratch);
    cudaSetDevice(prev);
    delete h;
    return GA_OK;
}

ga_status ga_heap_reset(ga_heap_t h, ga_stream_t stream) {
    if (!h) return GA_EINVAL;
    DeviceGuard g(h->device);
    return init_heap(h, (cudaStream_t)stream);
}

ga_status ga_heap_device(ga_heap_t h, ga_dev_heap* out) {
    if (!h || !out) return GA_EINVAL;
    out->desc = h->ddesc;
    out->base = h->dev.base;
    return GA_OK;
}

ga_status ga_heap_info(ga_heap_t h, uint64_t* heap_bytes, void** base, uint64_t* metadata_bytes) {
    if (!h) return GA_EINVAL;
    if (heap_bytes) *heap_bytes = h->dev.pages * kPage;
    if (base) *base = h->dev.base;
    if (metadata_bytes) *metadata_bytes = h->meta_bytes;
    return GA_OK;
}

ga_status ga_heap_quiesce(ga_heap_t h, ga_stream_t stream) {
    if (!h) return GA_EINVAL;
    DeviceGuard g(h->device);
    cudaStream_t s = (cudaStream_t)stream;
    k_quiesce_bins<<<grid_for(h->dev.pages), 256, 0, s>>>(h->ddesc);
    k_quiesce_chunks<<<grid_for(h->dev.nchunks), 256, 0, s>>>(h->ddesc);
    uint64_t n = h->dev.nchunks > (uint64_t)h->dev.n_arenas * h->dev.ahb_words ? h->dev.nchunks : (uint64_t)h->dev.n_arenas * h->dev.ahb_words;
    k_quiesce_clear<<<(int)((n + 255) / 256), 256, 0, s>>>(h->ddesc);
    return cudaGetLastError() == cudaSuccess ? GA_OK : GA_ECUDA;
}

ga_status ga_reserved_pages(ga_heap_t h, ga_stream_t stream, uint64_t* out) {
    if (!h || !out) return GA_EINVAL;
    DeviceGuard g(h->device);
    const ga_desc& d = h->dev;
    std::vector<uint64_t> av(h->avail_words);
    if (cudaMemcpyAsync(av.data(), d.avail, h->avail_words * 8, cudaMemcpyDeviceToHost, (cudaStream_t)stream) != cudaSuccess) return GA_ECUDA;
    if (cudaStreamSynchronize((cudaStream_t)stream) != cudaSuccess) return GA_ECUDA;
    uint64_t avail_pages = 0;
    for (uint32_t n = 0; n <= d.L; n++) {
        uint64_t cnt = 0;
        for (uint32_t j = 0; j < d.lvl_words[n]; j++) cnt += (uint64_t)__builtin_popcountll(av[d.lvl_off[n] + j]);
        avail_pages += cnt << n;
    }
    *out = d.pages - avail_pages;
    return GA_OK;
}

ga_status ga_stats(ga_heap_t h, ga_stream_t stream, ga_stats_t* out) {
    if (!h || !out) return GA_EINVAL;
    DeviceGuard g(h->device);
    memset(out, 0, sizeof *out);
    const ga_desc& d = h->dev;
    cudaStream_t s = (cudaStream_t)stream;
    uint64_t st[kStatWords];
    std::vector<uint64_t> ctr((uint64_t)d.n_arenas * kActrStride), cand(d.nchunks);
    bool ok = cudaMemcpyAsync(st, d.stats, sizeof st, cudaMemcpyDeviceToHost, s) == cudaSuccess &&
              cudaMemcpyAsync(ctr.data(), d.actr, ctr.size() * 8, cudaMemcpyDeviceToHost, s) == cudaSuccess &&
              cudaMemcpyAsync(cand.data(), d.chunk_cand, cand.size() * 8, cudaMemcpyDeviceToHost, s) == cudaSuccess &&
              cudaStreamSynchronize(s) == cudaSuccess;
    if (!ok) return GA_ECUDA;
    uint64_t pend = 0;
    for (uint64_t c : cand) pend += (uint64_t)__builtin_popcountll(c);
    for (uint32_t A = 0; A < d.n_arenas; A++) {
        out->n_malloc += ctr[(uint64_t)A * kActrStride + 0];
        out->n_free += ctr[(uint64_t)A * kActrStride + 1];
    }
    out->heap_bytes = d.pages * kPage;
    out->metadata_bytes = h->meta_bytes;
    out->reserved_bytes = st[kStatReserved] * kPage;
    out->peak_reserved_bytes = st[kStatPeakReserved] * kPage;
    out->n_bin_grow = st[kStatBinGrow];
    out->n_chunk_grow = st[kStatChunkGrow];
    out->n_bin_reclaim = st[kStatBinReclaim];
    out->n_chunk_reclaim = st[kStatChunkReclaim];
    out->n_fallback = st[kStatFallback];
    out->n_fail = st[kStatFail];
    out->n_pending_reclaim = pend;
    out->n_repair_nonfull = st[kStatRepairNonfull];
    out->n_repair_summary = st[kStatRepairSummary];
    out->n_waiter_reclaim = st[kStatWaiterReclaim];
    out->n_arenas = d.n_arenas;
    return GA_OK;
}

ga_status ga_heap_snapshot(ga_heap_t h, ga_stream_t stream, void* host, size_t cap, size_t* used) {
    if (!h || !used) return GA_EINVAL;
    DeviceGuard g(h->device);
    const ga_desc& d = h->dev;
    cudaStream_t s = (cudaStream_t)stream;
    std::vector<uint64_t> bits(d.pages * kBinWords), used_(d.nchunks), nonfull(1), cand(d.nchunks);
    std::vector<uint32_t> kind(d.pages), owner(d.nchunks);
    std::vector<uint64_t> sem((uint64_t)d.n_arenas * kNcls * kSemStride), psem((uint64_t)d.n_arenas * kSemStride);
    std::vector<uint64_t> av(h->avail_words), ts((uint64_t)(d.L + 1) * kSemStride);
    bool ok = cudaMemcpyAsync(bits.data(), d.bits, bits.size() * 8, cudaMemcpyDeviceToHost, s) == cudaSuccess &&
              cudaMemcpyAsync(kind.data(), d.kind, kind.size() * 4, cudaMemcpyDeviceToHost, s) == cudaSuccess &&
              cudaMemcpyAsync(used_.data(), d.chunk_used, used_.size() * 8, cudaMemcpyDeviceToHost, s) == cudaSuccess &&
              cudaMemcpyAsync(owner.data(), d.chunk_owner, owner.size() * 4, cudaMemcpyDeviceToHost, s) == cudaSuccess &&
              cudaMemcpyAsync(cand.data(), d.chunk_cand, cand.size() * 8, cudaMemcpyDeviceToHost, s) == cudaSuccess &&
              cudaMemcpyAsync(sem.data(), d.sem, sem.size() * 8, cudaMemcpyDeviceToHost, s) == cudaSuccess &&
              cudaMemcpyAsync(psem.data(), d.psem, psem.size() * 8, cudaMemcpyDeviceToHost, s) == cudaSuccess &&
              cudaMemcpyAsync(av.data(), d.avail, av.size() * 8, cudaMemcpyDeviceToHost, s) == cudaSuccess &&
              cudaMemcpyAsync(ts.data(), d.tsem, ts.size() * 8, cudaMemcpyDeviceToHost, s) == cudaSuccess &&
              cudaStreamSynchronize(s) == cudaSuccess;
    if (!ok) return GA_ECUDA;
    std::vector<uint8_t> out;
    auto put = [&](const void* p, size_t n) { const uint8_t* b = (const uint8_t*)p; out.insert(out.end(), b, b + n); };
    auto put64 = [&](uint64_t v) { put(&v, 8); };
    put64(0x31304E5341534147ull);
    put64(d.pages * kPage);
    put64(d.pages);
    put64(kPage | ((uint64_t)(d.L + 1) << 32));
    // the format's class section covers 16 B .. 64 KiB whatever this build
    // routes to spans (kSnapSpanSlots entries above the bins; zeros past kNspan)
    put64((1ull << kMinShift) | ((uint64_t)kNbin << 32) | ((uint64_t)kSnapSpanSlots << 40) | ((uint64_t)kChunkPages << 48));
    std::vector<uint8_t> kb(d.pages, 0x00);
    for (uint32_t n = 0; n <= d.L; n++) {
        uint64_t cnt = 1ull << (d.L - n);
        for (uint64_t i = 0; i < cnt; i++)
            if ((av[d.lvl_off[n] + (i >> 6)] >> (i & 63)) & 1) kb[i << n] = (uint8_t)(0x40 | n);
    }
    for (uint64_t p = 0; p < d.pages; p++) {
        if (kind[p] & kKindTree) {
            uint32_t o = kind[p] & 0xFF;
            kb[p] = (uint8_t)(0x80 | o);
            for (uint64_t q = p + 1; q < p + (1ull << o) && q < d.pages; q++) kb[q] = 0x01;
        }
    }
    for (uint64_t ch = 0; ch < d.nchunks; ch++) {
        if (!owner[ch]) continue;
        for (uint32_t j = 0; j < kChunkPages; j++) {
            uint64_t p = ch * kChunkPages + j;
            const uint32_t c = kind[p] & 0xFF;
            if (!((used_[ch] >> j) & 1)) kb[p] = 0x02;
            else if ((kind[p] & 0xC0000000u) == kKindBin && c < (uint32_t)kNbin) kb[p] = (uint8_t)(0x10 | c);
            else if ((kind[p] & 0xC0000000u) == kKindBin) kb[p] = (uint8_t)(j == 0 ? 0x20 | (c - kNbin) : 0x04);
            else kb[p] = 0xFF;                              // claimed page that is not a bin: not quiescent
        }
    }
    put(kb.data(), kb.size());
    for (uint64_t p = 0; p < d.pages; p++) {
        if (((kb[p] & 0xF0) != 0x10 && (kb[p] & 0xF0) != 0x20) || kb[p] == 0xFF) continue;
        int c = (kb[p] & 0x0F) + ((kb[p] & 0xF0) == 0x20 ? kNbin : 0);
        uint32_t slots = c < kNbin ? 256u >> c : kChunkPages >> (c - kNbin);
        uint8_t tmp[32] = {0};
        for (uint32_t sl = 0; sl < slots; sl++)
            if ((bits[p * kBinWords + sl / 64] >> (sl % 64)) & 1) tmp[sl / 8] |= (uint8_t)(1u << (sl % 8));
        put(tmp, (slots + 7) / 8);
    }
    for (uint32_t n = 0; n <= d.L; n++) {
        uint64_t cnt = 1ull << (d.L - n), nb = (cnt + 7) / 8;
        put(&av[d.lvl_off[n]], nb);                         // little endian words == LSB-first bytes
    }
    for (int c = 0; c < kNbin + kSnapSpanSlots; c++) {
        int64_t sc = 0, md = 0;
        if (c >= kNcls) { put64(0); put64(0); continue; }
        for (uint32_t A = 0; A < d.n_arenas; A++) {
            uint64_t w = sem[((uint64_t)A * kNcls + c) * kSemStride];
            int32_t C = (int32_t)(uint32_t)(w >> 32), D = (int32_t)((uint32_t)w - 0x80000000u);
            sc += C;
            if ((D < 0 ? -D : D) > md) md = D < 0 ? -D : D;
        }
        put64((uint64_t)sc); put64((uint64_t)md);
    }
    {
        int64_t sc = 0, md = 0;
        for (uint32_t A = 0; A < d.n_arenas; A++) {
            uint64_t w = psem[(uint64_t)A * kSemStride];
            int32_t C = (int32_t)(uint32_t)(w >> 32), D = (int32_t)((uint32_t)w - 0x80000000u);
            sc += C;
            if ((D < 0 ? -D : D) > md) md = D < 0 ? -D : D;
        }
        put64((uint64_t)sc); put64((uint64_t)md);
    }
    for (uint32_t n = 0; n <= d.L; n++) {
        uint64_t w = ts[(uint64_t)n * kSemStride];
        int64_t C = (int32_t)(uint32_t)(w >> 32), D = (int32_t)((uint32_t)w - 0x80000000u);
        put64((uint64_t)C); put64((uint64_t)D);
    }
    uint64_t pend = 0;
    for (uint64_t c : cand) pend += (uint64_t)__builtin_popcountll(c);
    put64(pend);
    *used = out.size();
    if (!host || cap < out.size()) return host ? GA_EINVAL : GA_OK;
    memcpy(host, out.data(), out.size());
    return GA_OK;
}

}  // extern "C"
