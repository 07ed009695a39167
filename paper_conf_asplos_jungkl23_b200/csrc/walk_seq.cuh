// Sequential one-warp walker shared by k_build.cu (fallback) and
// k_predict.cu (fault-anchored walks).
#pragma once
#include "device_util.cuh"
#include "kernels.cuh"

namespace dum {

// ---------------------------------------------------------------------------
// sequential walker (one warp): WALK(e, anchor) exactly as PAPER.md L218-L224 /
// D13-D14, probing rows in global memory.  Returns the walk length, or NONE if
// out_cap / scratch overflowed.
// ---------------------------------------------------------------------------
static __device__ __noinline__ uint32_t walk_seq(const Geo &g, const uint32_t *tbl_e, uint32_t start, uint32_t end, uint32_t anchor,
                             uint32_t *out, uint32_t out_cap, const WalkScratch &ws, uint32_t slot) {
  const uint32_t lane = lane_id();
  uint32_t *seen = ws.seen + (uint64_t)slot * ws.cap;
  uint32_t *chain = ws.chain + (uint64_t)slot * ws.cap;
  uint32_t *tmp = ws.tmp + (uint64_t)slot * ws.tmp_cap;
  if (anchor == NONE && start == NONE) return 0;
  uint32_t x = anchor != NONE ? anchor : start;
  uint32_t ntmp = 0, n = 0;
  bool overflow = false;
  if (lane == 0) {
    bool added;
    uint32_t s1 = hset_insert(seen, ws.cap, x, &added);
    uint32_t s2 = hset_insert(chain, ws.cap, x, &added);
    tmp[0] = s1;
    tmp[1] = s2 | 0x80000000u;
    if (anchor == NONE) out[0] = x;
  }
  ntmp = 2;
  if (anchor == NONE) n = 1;
  __syncwarp();
  if (x != end && tbl_e != nullptr) {
    for (;;) {
      const uint32_t *set = tbl_e + (uint64_t)row_of(g, x) * g.stride;
      uint32_t tg = lane < g.A ? __ldcg(set + lane * (1 + g.S)) : NONE;
      uint32_t m = __ballot_sync(0xffffffffu, lane < g.A && tg == x);
      if (!m) break;
      const uint32_t w = __ffs(m) - 1;
      uint32_t s = lane < g.S ? __ldcg(set + w * (1 + g.S) + 1 + lane) : NONE;
      const bool valid = s != NONE;
      const bool inseen = valid && hset_contains(seen, ws.cap, s);
      const bool inch = valid && hset_contains(chain, ws.cap, s);
      const uint32_t emit = __ballot_sync(0xffffffffu, valid && !inseen);
      const bool hit = __ballot_sync(0xffffffffu, valid && s == end) != 0;
      const uint32_t cand = __ballot_sync(0xffffffffu, valid && !inch);
      const uint32_t lt = (1u << lane) - 1;
      bool added = false;
      uint32_t sl = NONE;
      if (valid && !inseen) {
        const uint32_t pos = n + __popc(emit & lt);
        if (pos < out_cap) out[pos] = s;
        sl = hset_insert(seen, ws.cap, s, &added);
      }
      const uint32_t am = __ballot_sync(0xffffffffu, added);
      if (added) {
        const uint32_t tp = ntmp + __popc(am & lt);
        if (tp < ws.tmp_cap) tmp[tp] = sl;
      }
      ntmp += __popc(am);
      n += __popc(emit);
      if (n > out_cap || ntmp + 1 > ws.tmp_cap) {
        overflow = true;
        break;
      }
      if (hit || cand == 0) break;
      const uint32_t nxt = __shfl_sync(0xffffffffu, s, __ffs(cand) - 1);
      if (lane == 0) {
        bool a2;
        uint32_t s2 = hset_insert(chain, ws.cap, nxt, &a2);
        if (a2) tmp[ntmp] = s2 | 0x80000000u;
      }
      ++ntmp;
      x = nxt;
      __syncwarp();
    }
  }
  __syncwarp();
  const uint32_t nclr = ntmp < ws.tmp_cap ? ntmp : ws.tmp_cap;
  for (uint32_t p = lane; p < nclr; p += 32) {
    uint32_t v = tmp[p];
    if (v == NONE) continue;
    if (v & 0x80000000u) chain[v & 0x7FFFFFFFu] = NONE;
    else seen[v] = NONE;
    tmp[p] = NONE;
  }
  __syncwarp();
  return overflow ? NONE : n;
}

}  // namespace dum
