/*
 * tdfs_test.h -- test-only entry points of libtdfs.so.  They drive the same device
 * functions the matching kernel uses (queue, paged stack writer, task tracing) in
 * isolation, so the tests can check the paper's worked mechanisms exactly.
 * Same conventions as tdfs.h (status return, tdfs_last_error()).
 */
#ifndef TDFS_TEST_H_
#define TDFS_TEST_H_

#include <stdint.h>
#include "tdfs.h"

#ifdef __cplusplus
extern "C" {
#endif

/*
 * Q_task (Alg. 3) exercised on the device.
 *  mode 0: ONE warp enqueues the n_in tasks in order until enqueue returns false
 *          (queue full), then dequeues until dequeue returns false (queue empty).
 *          *n_enq = successful enqueues, *n_out = successful dequeues, h_out = the
 *          dequeued tasks in dequeue order (FIFO expected).
 *  mode 1: n_warps warps; warp w enqueues tasks w, w+n_warps, ... and after each
 *          enqueue dequeues one task when it can; finally all warps drain the queue.
 *          h_out = every dequeued task (a permutation of h_in expected).
 *  cap_tasks: capacity in tasks (N = 3 * cap_tasks ints).  ticket_base: initial value
 *          of the 64-bit head/tail tickets (wrap-around tests).
 *  Tasks are 3 ints <v1, v2, v3>; v3 = -2 marks a 2-vertex task.
 */
int tdfs_test_queue(int device, int mode, int n_warps, int64_t cap_tasks, uint64_t ticket_base,
                    int64_t n_in, const int32_t* h_in, int32_t* h_out, int64_t* n_out, int64_t* n_enq);

/*
 * Paged stack-level writer (Alg. 5, Fig. 6) on the device: one warp
 * writes the lanes set in valid_mask, ballot-compacted, at positions start_pos, ...
 * of a fresh stack level whose pages [0, start_pos / ints_per_page] are already
 * allocated.  Outputs per lane (-1 for invalid lanes): the page-table index and the
 * in-page offset the element landed at, plus the number of pages newly taken from the
 * pool and the first lane whose element lies on a newly allocated page (-1 if none).
 * Read back through the paged reader, every written element must equal its value.
 */
int tdfs_test_paged_write(int device, int page_bytes, int64_t start_pos, uint32_t valid_mask,
                          int32_t* h_page_of_lane, int32_t* h_offset_of_lane, int32_t* n_new_pages,
                          int32_t* first_lane_on_new_page, int32_t* readback_ok);

/*
 * tdfs_count with task tracing: every task pushed into Q_task is appended (3 ints) to
 * h_trace in the order the pushing warp created them (single-warp runs give the exact
 * Fig. 5 order).  *n_trace = number of tasks traced (may exceed cap;
 * only cap are stored).
 */
int tdfs_test_count_trace(const tdfs_graph* g, const tdfs_plan* p, const tdfs_run_opts* o, void* workspace,
                          size_t ws_bytes, void* stream, int32_t* h_trace, int64_t cap, int64_t* n_trace,
                          uint64_t* h_count);

#ifdef __cplusplus
}
#endif
#endif /* TDFS_TEST_H_ */
