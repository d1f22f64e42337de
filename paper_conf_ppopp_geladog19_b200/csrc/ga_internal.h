// ga_internal.h -- the heap handle, shared by the library's host files only.
#pragma once
#include <cstddef>
#include <cstdint>
#include <vector>

#include "ga.h"

struct ga_heap_s {
    int device = 0;
    char* pool_raw = nullptr;      // owned pool allocation (nullptr if borrowed)
    char* meta = nullptr;          // metadata allocation (R-29)
    size_t meta_bytes = 0;
    ga_desc dev{};                 // host copy of the descriptor
    ga_desc* ddesc = nullptr;      // device copy (start of the metadata allocation)
    std::vector<uint64_t> avail_init;   // host image of the tree bitmaps (empty heap)
    std::vector<uint64_t> tsem_init;
    uint64_t avail_words = 0;
    uint64_t ahb_total_words = 0;
    uint64_t peak_reserved_pages = 0;
    void* scratch = nullptr;       // device scratch for ga_trace_timed_host
    size_t scratch_bytes = 0;
};
