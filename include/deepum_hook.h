/* DeepUM-B200 PyTorch allocator hook.
 *
 * PAPER.md L283-L285 (Section 5.2, "Invalidating inactive PT blocks"):
 * "we add a few lines of code to the PyTorch memory allocator to tell the
 * DeepUM driver when a PT block is marked inactive.  If a victim page belongs
 * to an inactive PT block, the DeepUM driver simply invalidates the
 * corresponding UM block in the GPU memory."
 *
 * Instead of patching the allocator, libdeepum_hook.so attaches a trace
 * tracker to PyTorch's CUDA caching allocator
 * (c10::cuda::CUDACachingAllocator::attachAllocatorTraceTracker) and keeps,
 * per 2 MiB UM block, the bytes of live PT blocks (allocations) that overlap
 * it.  The allocator's segments are laid out in a block-id space in the order
 * they are created (segment s covers blocks [base_s, base_s + ceil(size/2MiB)),
 * block = base_s + (addr - segment start) >> 21 -- the "all GPU memory in UM
 * space" view of P:L134).  A UM block is inactive iff no live PT block
 * overlaps it (reading D20: "the caller resolves overlap"); a block whose
 * state changed is queued, and dum_hook_flush hands the queued blocks to
 * dum_mark_inactive (active ones with inactive = 0, the rest with 1).
 *
 * Events (torch's TraceEntry actions, DUM_HOOK_*):
 *   SEGMENT_ALLOC / SEGMENT_MAP   a new range: its blocks start inactive
 *   ALLOC                         + overlap bytes; 0 -> > 0 makes a block active
 *   FREE_COMPLETED                - overlap bytes; > 0 -> 0 makes it inactive
 *                                 (FREE_REQUESTED is ignored: the block may
 *                                 still be in use on another stream)
 *   SEGMENT_FREE / SEGMENT_UNMAP  the range's blocks become inactive; a freed
 *                                 segment's block ids are not reused
 * Addresses outside every known segment, and blocks at or beyond max_blocks,
 * are counted in `dropped` and otherwise ignored.
 *
 * Threading: the tracker runs with the allocator's lock held (it never calls
 * back into the allocator); the hook's own mutex guards its state.  Torch has
 * no detach: dum_hook_destroy only disables the tracker (its state is kept
 * alive, a few bytes, until process exit).
 * Errors: DUM_EINVAL for null / bad arguments; DUM_ECUDA for CUDA failures in
 * dum_hook_flush; other codes are returned from dum_mark_inactive. */
#ifndef DEEPUM_HOOK_H
#define DEEPUM_HOOK_H

#include <stdint.h>

#include "deepum_b200.h"

#ifdef __cplusplus
extern "C" {
#endif

enum {
  DUM_HOOK_ALLOC = 0,
  DUM_HOOK_FREE_REQUESTED = 1,
  DUM_HOOK_FREE_COMPLETED = 2,
  DUM_HOOK_SEGMENT_ALLOC = 3,
  DUM_HOOK_SEGMENT_FREE = 4,
  DUM_HOOK_SEGMENT_MAP = 5,
  DUM_HOOK_SEGMENT_UNMAP = 6,
};

typedef struct dum_hook dum_hook;

/* A hook over a block-id space of max_blocks UM blocks, for allocator events
 * of CUDA device `device`.  Returns NULL on bad arguments. */
dum_hook *dum_hook_create(uint32_t max_blocks, int device);
void dum_hook_destroy(dum_hook *h);

/* Attach to PyTorch's CUDA caching allocator (once per hook). */
int dum_hook_attach(dum_hook *h);

/* Feed one event by hand (the tracker calls the same handler): replays and
 * host-side tests. */
int dum_hook_feed(dum_hook *h, int action, uint64_t addr, uint64_t size);

/* The UM block of a device address (DUM_NONE if outside every segment). */
uint32_t dum_hook_block_of(dum_hook *h, uint64_t addr);

/* Drain the queued blocks into host arrays (each of capacity cap, ascending
 * block ids): the blocks now inactive and the blocks now active.  Returns the
 * number drained, or -1 if cap is too small (nothing drained). */
int dum_hook_drain(dum_hook *h, uint32_t *inactive, uint32_t *n_inactive, uint32_t *active, uint32_t *n_active,
                   uint32_t cap);

/* Drain and apply: dum_mark_inactive(eng, ...) for both lists on `stream`
 * (the lists are uploaded from the hook's pinned staging buffer; the call is
 * asynchronous -- the staging buffer is reused only after an event of the
 * previous flush completed). */
int dum_hook_flush(dum_hook *h, dum_engine *eng, dum_stream_t stream);

/* Counters: events seen, dropped events (outside the block space), blocks
 * in the space so far, live PT bytes. */
int dum_hook_stats(dum_hook *h, uint64_t out[4]);

#ifdef __cplusplus
}
#endif

#endif /* DEEPUM_HOOK_H */
