// f4: PyTorch allocator hook for inactive-block
// tracking, feeding dum_mark_inactive (include/deepum_hook.h).
//
// Host code only: a trace tracker on PyTorch's CUDA caching allocator keeps,
// per 2 MiB UM block of the allocator's segments, the bytes of live PT blocks
// overlapping it, and queues the blocks whose active / inactive state changed.
#include <c10/cuda/CUDACachingAllocator.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <map>
#include <memory>
#include <mutex>
#include <vector>

#include "deepum_hook.h"

namespace {

constexpr uint64_t BLK = 2ull << 20;  // UM block

struct Segment {
  uint64_t size;
  uint32_t base;  // first UM block of the segment
};

struct HookState {
  uint32_t W;
  int device;
  bool enabled = true;
  std::mutex mu;
  std::map<uint64_t, Segment> seg;  // start address -> segment
  uint32_t next_block = 0;
  std::vector<uint64_t> live;       // live PT bytes per UM block
  std::vector<uint8_t> queued;      // block in `pending`
  std::vector<uint32_t> pending;
  uint64_t events = 0, dropped = 0, live_bytes = 0;

  // the segment holding addr, or seg.end()
  std::map<uint64_t, Segment>::iterator find(uint64_t addr) {
    auto it = seg.upper_bound(addr);
    if (it == seg.begin()) return seg.end();
    --it;
    return addr < it->first + it->second.size ? it : seg.end();
  }
  void touch(uint32_t b) {
    if (!queued[b]) {
      queued[b] = 1;
      pending.push_back(b);
    }
  }
  // add (sign > 0) or remove the bytes of [addr, addr + size) inside segment it
  void account(std::map<uint64_t, Segment>::iterator it, uint64_t addr, uint64_t size, int sign) {
    const uint64_t s0 = it->first, end = std::min(addr + size, s0 + it->second.size);
    for (uint64_t a = addr; a < end;) {
      const uint64_t off = a - s0, b64 = it->second.base + off / BLK;
      const uint64_t stop = std::min(end, s0 + (off / BLK + 1) * BLK);
      if (b64 >= W) {
        ++dropped;
        return;
      }
      const uint32_t b = (uint32_t)b64;
      const uint64_t n = stop - a;
      const bool was = live[b] != 0;
      if (sign > 0) {
        live[b] += n;
        live_bytes += n;
      } else {
        const uint64_t d = std::min(live[b], n);
        live[b] -= d;
        live_bytes -= d;
      }
      if (was != (live[b] != 0)) touch(b);
      a = stop;
    }
  }
  void range_inactive(std::map<uint64_t, Segment>::iterator it, uint64_t addr, uint64_t size) {
    const uint64_t s0 = it->first, end = std::min(addr + size, s0 + it->second.size);
    for (uint64_t a = addr; a < end;) {
      const uint64_t off = a - s0, b64 = it->second.base + off / BLK;
      if (b64 >= W) {
        ++dropped;
        return;
      }
      const uint32_t b = (uint32_t)b64;
      live_bytes -= live[b];
      live[b] = 0;
      touch(b);
      a = s0 + (off / BLK + 1) * BLK;
    }
  }
  int feed(int action, uint64_t addr, uint64_t size) {
    std::lock_guard<std::mutex> g(mu);
    if (!enabled) return DUM_OK;
    ++events;
    switch (action) {
      case DUM_HOOK_SEGMENT_ALLOC:
      case DUM_HOOK_SEGMENT_MAP: {
        if (find(addr) != seg.end()) return DUM_OK;  // (a re-mapped part of a known range)
        const uint32_t nb = (uint32_t)((size + BLK - 1) / BLK);
        auto it = seg.emplace(addr, Segment{size, next_block}).first;
        next_block += nb;
        range_inactive(it, addr, size);  // free cached memory: inactive PT blocks
        return DUM_OK;
      }
      case DUM_HOOK_SEGMENT_FREE:
      case DUM_HOOK_SEGMENT_UNMAP: {
        auto it = find(addr);
        if (it == seg.end()) {
          ++dropped;
          return DUM_OK;
        }
        range_inactive(it, addr, size);
        if (action == DUM_HOOK_SEGMENT_FREE && it->first == addr) seg.erase(it);
        return DUM_OK;
      }
      case DUM_HOOK_ALLOC:
      case DUM_HOOK_FREE_COMPLETED: {
        auto it = find(addr);
        if (it == seg.end()) {
          ++dropped;
          return DUM_OK;
        }
        account(it, addr, size, action == DUM_HOOK_ALLOC ? 1 : -1);
        return DUM_OK;
      }
      case DUM_HOOK_FREE_REQUESTED:
        return DUM_OK;
      default:
        return DUM_EINVAL;
    }
  }
};

}  // namespace

struct dum_hook {
  std::shared_ptr<HookState> st;
  bool attached = false;
  // flush staging: pinned host + device lists, reused after ev completes
  uint32_t *h_buf = nullptr, *d_buf = nullptr;
  uint32_t buf_cap = 0;
  cudaEvent_t ev = nullptr;
};

extern "C" {

dum_hook *dum_hook_create(uint32_t max_blocks, int device) {
  if (max_blocks == 0 || device < 0) return nullptr;
  auto *h = new dum_hook;
  h->st = std::make_shared<HookState>();
  h->st->W = max_blocks;
  h->st->device = device;
  h->st->live.assign(max_blocks, 0);
  h->st->queued.assign(max_blocks, 0);
  return h;
}

void dum_hook_destroy(dum_hook *h) {
  if (!h) return;
  {
    std::lock_guard<std::mutex> g(h->st->mu);
    h->st->enabled = false;  // the attached tracker keeps the state alive but ignores events
  }
  if (h->ev) cudaEventDestroy(h->ev);
  if (h->h_buf) cudaFreeHost(h->h_buf);
  if (h->d_buf) cudaFree(h->d_buf);
  delete h;
}

int dum_hook_attach(dum_hook *h) {
  if (!h || h->attached) return DUM_EINVAL;
  std::shared_ptr<HookState> st = h->st;
  c10::cuda::CUDACachingAllocator::attachAllocatorTraceTracker(
      [st](const c10::CachingDeviceAllocator::TraceEntry &te) {
        if (te.device_ != st->device) return;
        st->feed((int)te.action_, (uint64_t)te.addr_, (uint64_t)te.size_);
      });
  h->attached = true;
  return DUM_OK;
}

int dum_hook_feed(dum_hook *h, int action, uint64_t addr, uint64_t size) {
  if (!h) return DUM_EINVAL;
  return h->st->feed(action, addr, size);
}

uint32_t dum_hook_block_of(dum_hook *h, uint64_t addr) {
  if (!h) return DUM_NONE;
  std::lock_guard<std::mutex> g(h->st->mu);
  auto it = h->st->find(addr);
  if (it == h->st->seg.end()) return DUM_NONE;
  const uint64_t b = it->second.base + (addr - it->first) / BLK;
  return b < h->st->W ? (uint32_t)b : DUM_NONE;
}

int dum_hook_drain(dum_hook *h, uint32_t *inactive, uint32_t *n_inactive, uint32_t *active, uint32_t *n_active,
                   uint32_t cap) {
  if (!h || !n_inactive || !n_active || (cap && (!inactive || !active))) return DUM_EINVAL;
  HookState &s = *h->st;
  std::lock_guard<std::mutex> g(s.mu);
  if (s.pending.size() > cap) return -1;
  std::sort(s.pending.begin(), s.pending.end());
  uint32_t ni = 0, na = 0;
  for (uint32_t b : s.pending) {
    s.queued[b] = 0;
    if (s.live[b]) active[na++] = b;
    else inactive[ni++] = b;
  }
  s.pending.clear();
  *n_inactive = ni;
  *n_active = na;
  return (int)(ni + na);
}

int dum_hook_flush(dum_hook *h, dum_engine *eng, dum_stream_t stream) {
  if (!h || !eng) return DUM_EINVAL;
  cudaStream_t s = (cudaStream_t)stream;
  uint32_t n = 0;
  {
    std::lock_guard<std::mutex> g(h->st->mu);
    n = (uint32_t)h->st->pending.size();
  }
  if (n == 0) return DUM_OK;
  if (h->ev && cudaEventSynchronize(h->ev) != cudaSuccess) return DUM_ECUDA;  // the last flush's upload is done
  if (n > h->buf_cap) {
    const uint32_t cap = std::max<uint32_t>(n, 4096);
    if (h->h_buf) cudaFreeHost(h->h_buf);
    if (h->d_buf) cudaFree(h->d_buf);
    h->h_buf = nullptr;
    h->d_buf = nullptr;
    if (cudaMallocHost((void **)&h->h_buf, 2ull * 4 * cap) != cudaSuccess ||
        cudaMalloc((void **)&h->d_buf, 2ull * 4 * cap) != cudaSuccess)
      return DUM_ECUDA;
    h->buf_cap = cap;
  }
  if (!h->ev && cudaEventCreateWithFlags(&h->ev, cudaEventDisableTiming) != cudaSuccess) return DUM_ECUDA;
  uint32_t ni = 0, na = 0;
  // (events arriving between the size read and the drain: drained next time if they overflow)
  int rc = dum_hook_drain(h, h->h_buf, &ni, h->h_buf + h->buf_cap, &na, h->buf_cap);
  if (rc < 0) return DUM_OK;  // grew meanwhile: the next flush takes them
  if (ni && cudaMemcpyAsync(h->d_buf, h->h_buf, 4ull * ni, cudaMemcpyHostToDevice, s) != cudaSuccess)
    return DUM_ECUDA;
  if (na && cudaMemcpyAsync(h->d_buf + h->buf_cap, h->h_buf + h->buf_cap, 4ull * na, cudaMemcpyHostToDevice, s) !=
                cudaSuccess)
    return DUM_ECUDA;
  if (ni && (rc = dum_mark_inactive(eng, h->d_buf, ni, 1, stream)) != DUM_OK) return rc;
  if (na && (rc = dum_mark_inactive(eng, h->d_buf + h->buf_cap, na, 0, stream)) != DUM_OK) return rc;
  // the staging buffers are free again once the uploads and both marks ran
  return cudaEventRecord(h->ev, s) == cudaSuccess ? DUM_OK : DUM_ECUDA;
}

int dum_hook_stats(dum_hook *h, uint64_t out[4]) {
  if (!h || !out) return DUM_EINVAL;
  std::lock_guard<std::mutex> g(h->st->mu);
  out[0] = h->st->events;
  out[1] = h->st->dropped;
  out[2] = h->st->next_block;
  out[3] = h->st->live_bytes;
  return DUM_OK;
}

}  // extern "C"
