/*
 * ga_rcu.h -- SRCU with RCU delegation on the GPU, and the paper's Fig. 6
 * benchmark.  C ABI, host side.
 *
 * Gelado & Garland, PPoPP'19, Sec. 4.2.1 and Sec. 5.2
 * (P:L1404-1478):
 *   SRCU keeps an epoch counter and two reader counters; readers count
 *   themselves into the current epoch, a barrier (under the RCU mutex) flips
 *   the epoch and waits for the previous epoch's counter to drain, then runs
 *   the queued release callbacks.  A CONDITIONAL barrier
 *   returns at once when another barrier is waiting to increment the epoch;
 *   that barrier runs its callbacks (RCU delegation, Fig. 4b).
 *   Readings R-39 (readers re-check the epoch after counting in) and R-40
 *   ("waiting to increment" = a pending flag cleared before the queue is
 *   taken) are in DESIGN.md and oracle/rcu.py, which pins them.
 *
 * Benchmark (Fig. 6): a doubly linked list of n_nodes elements
 * with tags 0..n_nodes-1; n_threads threads each search the list for the tag
 * d_tags[t] inside an RCU read-side critical section; a thread that finds its
 * tag unlinks the element under a writer mutex, queues its release and issues
 * an RCU barrier (classical: full; delegate != 0: conditional).  The input
 * holds every list tag once (writers) and tags >= n_nodes (readers), so the
 * writer:reader ratio is n_nodes : n_threads - n_nodes.
 */
#ifndef GA_RCU_H_
#define GA_RCU_H_

#include <stddef.h>
#include <stdint.h>

#include "ga.h"

#ifdef __cplusplus
extern "C" {
#endif

/* Device workspace bytes ga_rcu_list_removal needs for n_nodes list elements
 * (control words, nodes, callback queue, per-node release counters).
 * Errors: GA_EINVAL if out == NULL or n_nodes == 0 or n_nodes >= 2^31. */
ga_status ga_rcu_workspace_bytes(uint32_t n_nodes, size_t* out);

/* Run the Fig. 6 benchmark once on `stream`: init kernel (builds the list in
 * d_ws), the benchmark kernel (n_threads threads, `block` per block, 0 = 256),
 * and a flush kernel (releases what no barrier took, then audits).
 *   d_tags: DEVICE u32[n_threads], borrowed.  d_ws: DEVICE workspace of at
 *   least ga_rcu_workspace_bytes(n_nodes) bytes, borrowed, overwritten.
 *   d_out: DEVICE u64[8], overwritten: [0] elements unlinked, [1] release
 *   callbacks run, [2] read-side violations (a reader reached a released
 *   element: must be 0), [3] full barriers run, [4] conditional barriers that
 *   delegated, [5] elements released more than once (must be 0), [6] list
 *   length after the run, [7] threads that found nothing (readers).
 * Asynchronous; errors: GA_EINVAL on bad arguments or a small workspace,
 * GA_ECUDA if a launch fails. */
ga_status ga_rcu_list_removal(ga_stream_t stream, uint32_t n_threads, uint32_t n_nodes, const uint32_t* d_tags,
                              void* d_ws, size_t ws_bytes, uint32_t delegate, uint32_t block, uint64_t* d_out);

#ifdef __cplusplus
}
#endif

#endif /* GA_RCU_H_ */
