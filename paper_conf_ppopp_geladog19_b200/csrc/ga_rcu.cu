// ga_rcu.cu -- SRCU with RCU delegation and the Fig. 6 list-removal benchmark
// (include/ga_rcu.h).
//
// B200 shape: one control block of 32-byte-separated words in L2 (epoch,
// the two reader counters, the RCU mutex, the delegation flag, the callback
// queue tail and head, the writer mutex); the list nodes are 16-byte records
// read with one 128-bit load per hop.  Every spin loop backs off with
// __nanosleep.  The model these kernels implement, and its pins, are in
// oracle/rcu.py (readings R-39 and R-40).
#include <cuda_runtime.h>

#include <cstdint>

#include "ga.h"
#include "ga_rcu.h"

namespace {

constexpr uint32_t kNil = 0;                  // node 0 is the head sentinel
constexpr uint32_t kLinked = 0, kUnlinked = 1, kFreed = 2;
constexpr uint32_t kEmptySlot = 0xFFFFFFFFu;
// control words (u64 index; 32 B apart)
enum { kEpoch = 0, kCnt0 = 4, kCnt1 = 8, kRcuMutex = 12, kPending = 16, kQTail = 20, kQDone = 24, kWMutex = 28,
       kCtlWords = 32 };

struct Node { uint32_t tag, prev, next, state; };

struct Ws {
    uint64_t* ctl;
    Node* nodes;          // [n_nodes + 1]
    uint32_t* queue;      // [n_nodes] release callbacks (node ids)
    uint32_t* freed;      // [n_nodes + 1] releases per node
};

__host__ __device__ inline size_t align256(size_t x) { return (x + 255) & ~(size_t)255; }
__host__ __device__ inline size_t ws_bytes(uint32_t n) {
    return align256(kCtlWords * 8) + align256((size_t)(n + 1) * sizeof(Node)) + align256((size_t)n * 4) +
           align256((size_t)(n + 1) * 4);
}
__host__ __device__ inline Ws ws_of(void* base, uint32_t n) {
    char* p = (char*)base;
    Ws w;
    w.ctl = (uint64_t*)p; p += align256(kCtlWords * 8);
    w.nodes = (Node*)p; p += align256((size_t)(n + 1) * sizeof(Node));
    w.queue = (uint32_t*)p; p += align256((size_t)n * 4);
    w.freed = (uint32_t*)p;
    return w;
}

__device__ __forceinline__ uint64_t ld_acq(const uint64_t* p) {
    uint64_t v; asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory"); return v;
}
__device__ __forceinline__ uint32_t ld_acq32(const uint32_t* p) {
    uint32_t v; asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory"); return v;
}
__device__ __forceinline__ void st_rel(uint64_t* p, uint64_t v) {
    asm volatile("st.release.gpu.global.u64 [%0], %1;" :: "l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void st_rel32(uint32_t* p, uint32_t v) {
    asm volatile("st.release.gpu.global.u32 [%0], %1;" :: "l"(p), "r"(v) : "memory");
}
// one 16-byte node read (coherent at L2: other SMs unlink concurrently)
__device__ __forceinline__ Node ld_node(const Node* n) {
    Node x;
    asm volatile("ld.relaxed.gpu.global.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(x.tag), "=r"(x.prev), "=r"(x.next), "=r"(x.state) : "l"(n) : "memory");
    return x;
}
__device__ __forceinline__ unsigned long long* U(uint64_t* p) { return (unsigned long long*)p; }

__device__ void spin_lock(uint64_t* m) {
    uint32_t ns = 32;
    while (atomicCAS(U(m), 0ull, 1ull) != 0ull) { __nanosleep(ns); if (ns < 1024) ns <<= 1; }
    __threadfence();
}
__device__ void spin_unlock(uint64_t* m) { st_rel(m, 0ull); }

// read-side critical section, R-39: re-check the epoch after
// counting in, retreat and retry if a barrier flipped it meanwhile
__device__ uint32_t rcu_read_lock(uint64_t* ctl) {
    for (;;) {
        const uint32_t idx = (uint32_t)(ld_acq(&ctl[kEpoch]) & 1);
        atomicAdd(U(&ctl[idx ? kCnt1 : kCnt0]), 1ull);
        __threadfence();                                   // SC: count in before re-reading the epoch
        if ((uint32_t)(ld_acq(&ctl[kEpoch]) & 1) == idx) return idx;
        atomicAdd(U(&ctl[idx ? kCnt1 : kCnt0]), ~0ull);     // -1
    }
}
__device__ void rcu_read_unlock(uint64_t* ctl, uint32_t idx) {
    __threadfence();                                       // our reads complete before we count out
    atomicAdd(U(&ctl[idx ? kCnt1 : kCnt0]), ~0ull);
}

// release callback: the element goes back (poisoned; its links stay, so a
// buggy reader would not crash, only be counted)
__device__ void release_node(Ws w, uint32_t n, uint64_t* out) {
    w.nodes[n].tag = 0xFFFFFFFFu;
    st_rel32(&w.nodes[n].state, kFreed);
    atomicAdd(&w.freed[n], 1u);
    atomicAdd(U(&out[1]), 1ull);
}

// queued callbacks [q_done, end): wait for each slot's publication, release
__device__ void run_callbacks(Ws w, uint64_t end, uint64_t* out) {
    uint64_t i = ld_acq(&w.ctl[kQDone]);
    for (; i < end; i++) {
        uint32_t n;
        uint32_t ns = 32;
        while ((n = ld_acq32(&w.queue[i])) == kEmptySlot) { __nanosleep(ns); if (ns < 256) ns <<= 1; }
        release_node(w, n, out);
    }
    st_rel(&w.ctl[kQDone], i);                             // == max(q_done, end): only the mutex holder writes it
}

// the barrier proper, called with the RCU mutex held: take the queue, flip
// the epoch, wait for the previous epoch's readers, run the callbacks
__device__ void barrier_locked(Ws w, uint64_t* out) {
    const uint64_t end = ld_acq(&w.ctl[kQTail]);
    const uint32_t old = (uint32_t)(atomicAdd(U(&w.ctl[kEpoch]), 1ull) & 1);
    __threadfence();                                       // SC: flip before reading the old counter
    uint64_t* c = &w.ctl[old ? kCnt1 : kCnt0];
    uint32_t ns = 32;
    while (ld_acq(c) != 0) { __nanosleep(ns); if (ns < 1024) ns <<= 1; }
    run_callbacks(w, end, out);
    atomicAdd(U(&out[3]), 1ull);
}

__device__ void full_barrier(Ws w, uint64_t* out) {
    spin_lock(&w.ctl[kRcuMutex]);
    barrier_locked(w, out);
    spin_unlock(&w.ctl[kRcuMutex]);
}

// RCU delegation, R-40: the caller has queued its callback;
// if a barrier is already pending it will take that callback, so return
__device__ void conditional_barrier(Ws w, uint64_t* out) {
    __threadfence();                                       // SC: queue before testing the flag
    if (atomicCAS(U(&w.ctl[kPending]), 0ull, 1ull) != 0ull) { atomicAdd(U(&out[4]), 1ull); return; }
    spin_lock(&w.ctl[kRcuMutex]);
    atomicExch(U(&w.ctl[kPending]), 0ull);                 // clear the flag, then take the queue
    __threadfence();
    barrier_locked(w, out);
    spin_unlock(&w.ctl[kRcuMutex]);
}

__global__ void k_rcu_init(Ws w, uint32_t n) {
    const uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i < kCtlWords) w.ctl[i] = 0;
    if (i <= n) {
        Node x;
        x.tag = i == 0 ? 0xFFFFFFFEu : (uint32_t)(i - 1);
        x.prev = i == 0 ? n : (uint32_t)(i - 1);
        x.next = i == n ? kNil : (uint32_t)(i + 1);
        x.state = kLinked;
        w.nodes[i] = x;
        w.freed[i] = 0;
    }
    if (i < n) w.queue[i] = kEmptySlot;
}

__global__ void __launch_bounds__(256) k_rcu_bench(Ws w, const uint32_t* __restrict__ tags, uint32_t T, uint32_t delegate,
                                                   uint64_t* out) {
    const uint32_t t = blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= T) return;
    const uint32_t tag = __ldg(&tags[t]);
    uint32_t viol = 0, found = kNil;
    // reader: traverse under RCU
    const uint32_t idx = rcu_read_lock(w.ctl);
    uint32_t n = ld_node(&w.nodes[0]).next;
    while (n != kNil) {
        const Node x = ld_node(&w.nodes[n]);
        if (x.state == kFreed) viol++;
        if (x.tag == tag) { found = n; break; }
        n = x.next;
    }
    rcu_read_unlock(w.ctl, idx);
    if (viol) atomicAdd(U(&out[2]), (unsigned long long)viol);
    if (found == kNil) { atomicAdd(U(&out[7]), 1ull); return; }
    // writer: unlink under the writer mutex
    bool mine = false;
    spin_lock(&w.ctl[kWMutex]);
    Node x = ld_node(&w.nodes[found]);
    if (x.state == kLinked) {
        w.nodes[x.prev].next = x.next;
        if (x.next != kNil) w.nodes[x.next].prev = x.prev; else w.nodes[0].prev = x.prev;
        w.nodes[found].state = kUnlinked;
        mine = true;
    }
    __threadfence();
    spin_unlock(&w.ctl[kWMutex]);
    if (!mine) return;
    atomicAdd(U(&out[0]), 1ull);
    // queue the release, then the barrier
    const uint64_t slot = atomicAdd(U(&w.ctl[kQTail]), 1ull);
    st_rel32(&w.queue[slot], found);
    if (delegate) conditional_barrier(w, out); else full_barrier(w, out);
}

// end of the run: release what no barrier took (no readers remain), then audit
__global__ void k_rcu_flush(Ws w, uint32_t n, uint64_t* out) {
    if (threadIdx.x == 0 && blockIdx.x == 0) {
        run_callbacks(w, w.ctl[kQTail], out);
        uint64_t len = 0;
        for (uint32_t x = w.nodes[0].next; x != kNil && len <= n; x = w.nodes[x].next) len++;
        out[6] = len;
    }
}
__global__ void k_rcu_audit(Ws w, uint32_t n, uint64_t* out) {
    const uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i >= 1 && i <= n && w.freed[i] > 1) atomicAdd(U(&out[5]), 1ull);
}

}  // namespace

extern "C" {

ga_status ga_rcu_workspace_bytes(uint32_t n_nodes, size_t* out) {
    if (!out || n_nodes == 0 || n_nodes >= (1u << 31)) return GA_EINVAL;
    *out = ws_bytes(n_nodes);
    return GA_OK;
}

ga_status ga_rcu_list_removal(ga_stream_t stream, uint32_t n_threads, uint32_t n_nodes, const uint32_t* d_tags,
                              void* d_ws, size_t ws_size, uint32_t delegate, uint32_t block, uint64_t* d_out) {
    if (!d_tags || !d_ws || !d_out || n_threads == 0 || n_nodes == 0 || n_nodes >= (1u << 31) ||
        ws_size < ws_bytes(n_nodes))
        return GA_EINVAL;
    if (block == 0) block = 256;
    if (block > 256) return GA_EINVAL;
    cudaStream_t s = (cudaStream_t)stream;
    Ws w = ws_of(d_ws, n_nodes);
    const uint64_t nin = (uint64_t)n_nodes + 1 > kCtlWords ? (uint64_t)n_nodes + 1 : kCtlWords;
    if (cudaMemsetAsync(d_out, 0, 64, s) != cudaSuccess) return GA_ECUDA;
    k_rcu_init<<<(unsigned)((nin + 255) / 256), 256, 0, s>>>(w, n_nodes);
    k_rcu_bench<<<(n_threads + block - 1) / block, block, 0, s>>>(w, d_tags, n_threads, delegate, d_out);
    k_rcu_flush<<<1, 32, 0, s>>>(w, n_nodes, d_out);
    k_rcu_audit<<<(unsigned)((n_nodes + 256) / 256), 256, 0, s>>>(w, n_nodes, d_out);
    return cudaGetLastError() == cudaSuccess ? GA_OK : GA_ECUDA;
}

}  // extern "C"
