// ga_internal.h -- the heap handle, shared by the library's host files only.
#pragma once
#include <cstddef>
#include <cstdint>
#include <vector>

#include <cuda_runtime.h>

#include "ga.h"

struct ga_heap_s {
    int device = 0;
    char* pool_raw = nullptr;      // owned pool allocation (nullptr if borrowed)
    char* meta = nullptr;          // metadata allocation (R-29)
    size_t meta_bytes = 0;
    ga_desc dev{};                 // host copy of the descriptor
    ga_desc* ddesc = nullptr;      // device copy (start of the metadata allocation)
    std::vector<uint64_t> avail_init;   // host image of the tree bitmaps (empty heap)
    uint64_t* init_img = nullptr;       // device copy: avail image, then tsem image
    std::vector<uint64_t> tsem_init;
    uint64_t avail_words = 0;
    uint64_t ahb_total_words = 0;
    void* scratch = nullptr;       // device scratch for ga_trace_timed_host
    size_t scratch_bytes = 0;
};

// Handle-taking host calls run on the heap's device and restore the caller's
// current device on return.
struct DeviceGuard {
    int prev = -1;
    explicit DeviceGuard(int dev) {
        if (cudaGetDevice(&prev) != cudaSuccess) prev = -1;
        else if (prev != dev) cudaSetDevice(dev);
    }
    ~DeviceGuard() { if (prev >= 0) cudaSetDevice(prev); }
    DeviceGuard(const DeviceGuard&) = delete;
    DeviceGuard& operator=(const DeviceGuard&) = delete;
};
