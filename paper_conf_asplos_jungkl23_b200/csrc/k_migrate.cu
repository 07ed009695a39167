// a9: block migration and residency bookkeeping.
//
// "it evicts some pages from the GPU to the CPU (4). Then, it populates faulted
// pages in the GPU (5) ... and it transfers the pages to the GPU (6) ... mapped
// to the GPU (7)"; "the migration thread migrates the UM
// blocks between the CPU and the GPU" (L158); invalidation drops a block
// without a copy (L285).  Readings: frames are the lowest free ones in list
// order (D21); the LRM order is the migration-in stamp order (D19).
//
//  k_mig_plan     one CTA: validates the list (no duplicates, residency),
//                 assigns frames (i-th block -> i-th lowest free frame, a scan
//                 over the free-frame bitmap), updates frame_of /
//                 block_of / stamps / the LRM log, or leaves everything
//                 untouched and raises a sticky error.
//  k_copy_blocks  persistent SM copy: 16 B vector loads/stores, 64 KiB work
//                 items, 8 loads in flight per thread; host memory is read or
//                 written through its mapped device address (PCIe).
//  k_checksums    position-weighted 64-bit sums of 2 MiB blocks (verification).
#include <algorithm>
#include <vector>

#include "device_util.cuh"
#include "kernels.cuh"

namespace dum {

constexpr int PLAN_NT = 1024;
constexpr uint64_t BLK = 2ull << 20;

__global__ void k_res_reset(uint32_t W, uint32_t C, uint32_t *frame_of, uint32_t *stamp_of, uint32_t *block_of,
                            uint32_t *free_bits, uint32_t *inactive, uint32_t *res_bits, bool clear_inactive,
                            DevState *st) {
  const uint32_t t = blockIdx.x * blockDim.x + threadIdx.x, nt = gridDim.x * blockDim.x;
  for (uint32_t i = t; i < W; i += nt) {
    frame_of[i] = NONE;
    stamp_of[i] = 0;
  }
  for (uint32_t i = t; i < C; i += nt) block_of[i] = NONE;
  for (uint32_t w = t; w < (C + 31) / 32; w += nt) {
    const uint32_t lo = w * 32;
    free_bits[w] = C - lo >= 32 ? 0xFFFFFFFFu : ((1u << (C - lo)) - 1u);
  }
  for (uint32_t w = t; w < (W + 31) / 32; w += nt) {
    res_bits[w] = 0;
    if (clear_inactive) inactive[w] = 0;
  }
  if (t == 0) {
    st->lrm_head = st->lrm_tail = 0;
    st->log_dirty = 0;
    st->free_count = C;
    st->mig_counter = 0;
    st->n_resident = 0;
  }
}

__global__ void k_load_res(const uint32_t *__restrict__ lrm, uint32_t n, uint32_t W, uint32_t *frame_of,
                           uint32_t *stamp_of, uint32_t *block_of, uint32_t *free_bits, uint32_t *lrm_blk,
                           uint32_t *lrm_stamp, uint32_t *res_bits, const uint32_t *inactive, uint32_t *logpos,
                           DevState *st) {
  const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i == 0) {
    st->lrm_head = 0;
    st->lrm_tail = n;
    st->free_count -= n;
    st->mig_counter = n;
    st->n_resident = n;
  }
  if (i >= n) return;
  const uint32_t b = lrm[i];
  if (b >= W || atomicCAS(&frame_of[b], NONE, i) != NONE) {
    set_err(st, ERR_EINVAL);
    return;
  }
  block_of[i] = b;
  stamp_of[b] = i;
  lrm_blk[i] = b | (((inactive[b >> 5] >> (b & 31)) & 1u) << 31);  // inactive flag packed in bit 31
  logpos[b] = i;
  lrm_stamp[i] = i;
  atomicAnd(&free_bits[i >> 5], ~(1u << (i & 31)));
  atomicOr(&res_bits[b >> 5], 1u << (b & 31));
}

__global__ void k_mark_inactive(const uint32_t *__restrict__ blocks, uint32_t n, int flag, uint32_t W,
                                uint32_t *inactive, const uint32_t *frame_of, const uint32_t *logpos,
                                uint32_t *lrm_blk, DevState *st) {
  const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  const uint32_t b = blocks[i];
  if (b >= W) {
    set_err(st, ERR_EINVAL);
    return;
  }
  if (flag) atomicOr(&inactive[b >> 5], 1u << (b & 31));
  else atomicAnd(&inactive[b >> 5], ~(1u << (b & 31)));
  // resident blocks carry the flag in their LRM-log entry (bit 31)
  if (frame_of[b] != NONE) lrm_blk[logpos[b]] = b | ((flag ? 1u : 0u) << 31);
}

struct MigArgs {
  int dir;
  const uint32_t *blocks, *dst;
  uint32_t n;
  const uint64_t *rng;  // device (begin, end) into blocks: the list is blocks[begin, end), n caps it (closed loop)
  uint32_t W, C;
  uint32_t *frame_of, *stamp_of, *block_of, *free_bits, *lrm_blk, *lrm_stamp, *res_bits, *logpos;
  const uint32_t *inactive;
  uint32_t lrm_cap;
  uint32_t *mig_frames, *mig_src, *mig_blocks;
  DevState *st;
};

// k-th (0-based) set bit positions of a bitmap, for ranks [0, want): writes
// out[rank] = bit index.  Bits >= nbits are ignored.  invert: scan zero bits.
__device__ void select_bits(const uint32_t *bits, uint32_t nbits, bool invert, uint32_t lo_bit, uint32_t want,
                            uint32_t *out, uint32_t *ws) {
  uint32_t run = 0;
  const uint32_t w0 = lo_bit / 32, nw = (nbits + 31) / 32;
  for (uint32_t c = w0; c < nw && run < want; c += PLAN_NT) {
    const uint32_t w = c + threadIdx.x;
    uint32_t m = 0;
    if (w < nw) {
      m = bits[w];
      if (invert) m = ~m;
      if (w * 32 < lo_bit) m &= ~((1u << (lo_bit - w * 32)) - 1u);
      if (w * 32 + 32 > nbits) m &= (nbits - w * 32 >= 32) ? 0xFFFFFFFFu : ((1u << (nbits - w * 32)) - 1u);
    }
    uint32_t tot;
    uint32_t r = run + block_excl_scan(__popc(m), ws, &tot);
    while (m && r < want) {
      const uint32_t bit = __ffs(m) - 1;
      out[r++] = w * 32 + bit;
      m &= m - 1;
    }
    run += tot;
  }
}

__global__ void __launch_bounds__(PLAN_NT) k_mig_plan(MigArgs a) {
  __shared__ uint32_t ws[PLAN_NT / 32];
  __shared__ uint32_t s_bad;
  DevState *st = a.st;
  const uint32_t tid = threadIdx.x;
  if (tid == 0) {
    s_bad = 0;
    st->mig_ok = 0;
  }
  __syncthreads();
  uint32_t n = a.n;
  const uint32_t *blocks_in = a.blocks;
  if (a.rng) {  // a device-sized list (dum_simulate): blocks[rng[0], rng[1])
    const uint64_t b0 = a.rng[0], b1 = a.rng[1];
    const uint64_t len = b1 > b0 ? b1 - b0 : 0;
    if (len < n) n = (uint32_t)len;
    blocks_in += b0;
  }
  a.blocks = blocks_in;
  if (a.dir == DUM_H2D) {
    if (n > st->free_count) {
      if (tid == 0) set_err(st, ERR_ECAPACITY, n);
      return;
    }
    for (uint32_t i = tid; i < n; i += PLAN_NT) {
      const uint32_t b = a.blocks[i];
      bool ok = b < a.W && atomicCAS(&a.frame_of[b], NONE, CLAIM) == NONE;
      a.mig_blocks[i] = ok ? b : NONE;  // remember successful claims
      if (!ok) s_bad = 1;
    }
    __syncthreads();
    if (s_bad) {
      for (uint32_t i = tid; i < n; i += PLAN_NT)
        if (a.mig_blocks[i] != NONE) a.frame_of[a.mig_blocks[i]] = NONE;
      if (tid == 0) set_err(st, ERR_EINVAL);
      return;
    }
    // make room in the LRM log: stable compaction of still-valid entries
    uint32_t head = st->lrm_head, tail = st->lrm_tail;
    if (tail + n > a.lrm_cap) {
      uint32_t outp = 0;
      for (uint32_t c = head; c < tail; c += PLAN_NT) {
        const uint32_t i = c + tid;
        uint32_t b = NONE, s = 0, keep = 0;
        if (i < tail) {
          b = a.lrm_blk[i];
          s = a.lrm_stamp[i];
          const uint32_t f = a.frame_of[b & 0x7FFFFFFFu];
          keep = f != NONE && f != CLAIM && a.stamp_of[b & 0x7FFFFFFFu] == s;
        }
        uint32_t tot;
        const uint32_t pre = block_excl_scan(keep, ws, &tot);  // syncs: reads done before writes
        if (keep) {
          a.lrm_blk[outp + pre] = b;
          a.lrm_stamp[outp + pre] = s;
          a.logpos[b & 0x7FFFFFFFu] = outp + pre;
        }
        outp += tot;
        __syncthreads();
      }
      head = 0;
      tail = outp;
      if (tid == 0) st->log_dirty = 0;
      if (tail + n > a.lrm_cap) {
        if (tid == 0) set_err(st, ERR_ECAPACITY, tail + n);
        for (uint32_t i = tid; i < n; i += PLAN_NT) a.frame_of[a.blocks[i]] = NONE;
        return;
      }
    }
    select_bits(a.free_bits, a.C, false, 0, n, a.mig_frames, ws);
    __syncthreads();
    const uint32_t mc = st->mig_counter;
    for (uint32_t i = tid; i < n; i += PLAN_NT) {
      const uint32_t b = a.blocks[i], f = a.mig_frames[i];
      a.frame_of[b] = f;
      a.block_of[f] = b;
      a.stamp_of[b] = mc + i;
      a.lrm_blk[tail + i] = b | (((a.inactive[b >> 5] >> (b & 31)) & 1u) << 31);
      a.logpos[b] = tail + i;
      a.lrm_stamp[tail + i] = mc + i;
      atomicAnd(&a.free_bits[f >> 5], ~(1u << (f & 31)));
      atomicOr(&a.res_bits[b >> 5], 1u << (b & 31));
    }
    if (tid == 0) {
      st->free_count -= n;
      st->mig_counter = mc + n;
      st->lrm_head = head;
      st->lrm_tail = tail + n;
      st->n_resident += n;
    }
  } else if (a.dir == DUM_D2H || a.dir == DUM_INVALIDATE) {
    for (uint32_t i = tid; i < n; i += PLAN_NT) {
      const uint32_t b = a.blocks[i];
      uint32_t f = b < a.W ? a.frame_of[b] : NONE;
      bool ok = f != NONE && f < a.C && atomicCAS(&a.block_of[f], b, CLAIM) == b;
      a.mig_frames[i] = ok ? f : NONE;
      if (!ok) s_bad = 1;
    }
    __syncthreads();
    if (s_bad) {
      for (uint32_t i = tid; i < n; i += PLAN_NT)
        if (a.mig_frames[i] != NONE) a.block_of[a.mig_frames[i]] = a.blocks[i];
      if (tid == 0) set_err(st, ERR_EINVAL);
      return;
    }
    for (uint32_t i = tid; i < n; i += PLAN_NT) {
      const uint32_t b = a.blocks[i], f = a.mig_frames[i];
      a.frame_of[b] = NONE;
      a.block_of[f] = NONE;
      a.mig_blocks[i] = b;
      atomicOr(&a.free_bits[f >> 5], 1u << (f & 31));
      atomicAnd(&a.res_bits[b >> 5], ~(1u << (b & 31)));
    }
    if (tid == 0) {
      st->free_count += n;
      st->n_resident -= n;
      st->log_dirty = 1;
    }
  } else if (a.dir == DUM_D2D && a.blocks != nullptr) {
    for (uint32_t i = tid; i < n; i += PLAN_NT) {
      const uint32_t b = a.blocks[i], d = a.dst[i];
      uint32_t f = b < a.W ? a.frame_of[b] : NONE;
      bool ok = f != NONE && f < a.C && d < a.C && atomicCAS(&a.block_of[f], b, CLAIM) == b;
      bool okd = ok && atomicCAS(&a.block_of[d], NONE, CLAIM_DST) == NONE;
      if (ok && !okd) a.block_of[f] = b;
      a.mig_src[i] = okd ? f : NONE;
      if (!okd) s_bad = 1;
    }
    __syncthreads();
    if (s_bad) {
      for (uint32_t i = tid; i < n; i += PLAN_NT)
        if (a.mig_src[i] != NONE) {
          a.block_of[a.mig_src[i]] = a.blocks[i];
          a.block_of[a.dst[i]] = NONE;
        }
      if (tid == 0) set_err(st, ERR_EINVAL);
      return;
    }
    for (uint32_t i = tid; i < n; i += PLAN_NT) {
      const uint32_t f = a.mig_src[i];
      a.block_of[f] = NONE;
      atomicOr(&a.free_bits[f >> 5], 1u << (f & 31));
    }
    __syncthreads();
    for (uint32_t i = tid; i < n; i += PLAN_NT) {
      const uint32_t b = a.blocks[i], d = a.dst[i];
      a.frame_of[b] = d;
      a.block_of[d] = b;
      a.mig_frames[i] = d;
      a.mig_blocks[i] = b;
      atomicAnd(&a.free_bits[d >> 5], ~(1u << (d & 31)));
    }
  } else {  // D2D compaction
    const uint32_t nres = a.C - st->free_count;
    // holes: free frames in [0, nres) ascending; movers: occupied frames in
    // [nres, C), taken from the top
    uint32_t *holes = a.mig_frames, *occ = a.mig_blocks;
    select_bits(a.free_bits, nres, false, 0, a.C, holes, ws);
    __syncthreads();
    select_bits(a.free_bits, a.C, true, nres, a.C, occ, ws);
    __syncthreads();
    // number of holes = number of occupied frames at or above nres
    uint32_t h = 0;
    for (uint32_t w = 0; w < (nres + 31) / 32; ++w) {
      uint32_t m = a.free_bits[w];
      if (w * 32 + 32 > nres) m &= (nres - w * 32 >= 32) ? 0xFFFFFFFFu : ((1u << (nres - w * 32)) - 1u);
      h += __popc(m);
    }
    for (uint32_t i = tid; i < h; i += PLAN_NT) a.mig_src[i] = occ[h - 1 - i];
    __syncthreads();
    for (uint32_t i = tid; i < h; i += PLAN_NT) {
      const uint32_t src = a.mig_src[i], d = holes[i], b = a.block_of[src];
      a.frame_of[b] = d;
      a.block_of[d] = b;
      a.block_of[src] = NONE;
      a.mig_blocks[i] = b;
      atomicAnd(&a.free_bits[d >> 5], ~(1u << (d & 31)));
      atomicOr(&a.free_bits[src >> 5], 1u << (src & 31));
    }
    if (tid == 0) st->mig_n = h;
  }
  if (tid == 0) {
    if (!(a.dir == DUM_D2D && a.blocks == nullptr)) st->mig_n = n;
    st->mig_ok = 1;
  }
}

// copy kernel: work item = (block i, 64 KiB chunk c)
constexpr int COPY_NT = 256;
constexpr uint32_t CHUNK = 64u << 10;
constexpr uint32_t CHUNKS = (uint32_t)(BLK / CHUNK);

__global__ void __launch_bounds__(COPY_NT) k_copy_blocks(int dir, const uint32_t *__restrict__ blocks,
                                                         const uint32_t *__restrict__ src_frames,
                                                         const uint32_t *__restrict__ frames, char *host,
                                                         char *pool, const DevState *st) {
  if (!st->mig_ok || dir == DUM_INVALIDATE) return;
  const uint32_t n = st->mig_n;
  const uint64_t items = (uint64_t)n * CHUNKS;
  if (blockIdx.x == 0 && threadIdx.x == 0) ctr_add(const_cast<DevState *>(st), DUM_CTR_MIG_BLOCKS, n);
  for (uint64_t it = blockIdx.x; it < items; it += gridDim.x) {
    const uint32_t i = (uint32_t)(it / CHUNKS), c = (uint32_t)(it % CHUNKS);
    const char *src;
    char *dst;
    if (dir == DUM_H2D) {
      src = host + (uint64_t)blocks[i] * BLK;
      dst = pool + (uint64_t)frames[i] * BLK;
    } else if (dir == DUM_D2H) {
      src = pool + (uint64_t)frames[i] * BLK;
      dst = host + (uint64_t)blocks[i] * BLK;
    } else {
      src = pool + (uint64_t)src_frames[i] * BLK;
      dst = pool + (uint64_t)frames[i] * BLK;
    }
    const uint4 *s4 = reinterpret_cast<const uint4 *>(src + (uint64_t)c * CHUNK);
    uint4 *d4 = reinterpret_cast<uint4 *>(dst + (uint64_t)c * CHUNK);
    constexpr int PER = CHUNK / 16 / COPY_NT;  // 16 vectors per thread
#pragma unroll
    for (int u = 0; u < PER; u += 8) {
      uint4 v[8];
#pragma unroll
      for (int k = 0; k < 8; ++k) v[k] = __ldcs(s4 + (u + k) * COPY_NT + threadIdx.x);
#pragma unroll
      for (int k = 0; k < 8; ++k) __stcs(d4 + (u + k) * COPY_NT + threadIdx.x, v[k]);
    }
  }
}

// TMA bulk path (method 3): one elected thread per CTA moves 32 KiB tiles
// with the bulk-copy engine -- cp.async.bulk global -> shared (completion on an
// mbarrier), then cp.async.bulk shared -> global -- NBULK tiles in flight per
// CTA, one CTA per SM; the same (block i, tile) work split as k_copy_blocks.
constexpr uint32_t BULK_TILE = 32u << 10;
constexpr uint32_t NBULK = 4;
constexpr uint32_t BULK_TILES = (uint32_t)(BLK / BULK_TILE);

__device__ __forceinline__ uint32_t smem_u32(const void *p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}

__global__ void __launch_bounds__(32) k_copy_bulk(int dir, const uint32_t *__restrict__ blocks,
                                                  const uint32_t *__restrict__ src_frames,
                                                  const uint32_t *__restrict__ frames, char *host, char *pool,
                                                  const DevState *st) {
  extern __shared__ __align__(128) unsigned char tiles[];  // NBULK x BULK_TILE
  __shared__ __align__(8) unsigned long long bar[NBULK];
  if (!st->mig_ok || dir == DUM_INVALIDATE) return;
  if (threadIdx.x != 0) return;
  const uint32_t n = st->mig_n;
  const uint64_t items = (uint64_t)n * BULK_TILES;
  if (blockIdx.x == 0) ctr_add(const_cast<DevState *>(st), DUM_CTR_MIG_BLOCKS, n);
  for (uint32_t s = 0; s < NBULK; ++s)
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&bar[s])));
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  auto addr = [&](uint64_t it, const char *&src, char *&dst) {
    const uint32_t i = (uint32_t)(it / BULK_TILES), c = (uint32_t)(it % BULK_TILES);
    if (dir == DUM_H2D) {
      src = host + (uint64_t)blocks[i] * BLK;
      dst = pool + (uint64_t)frames[i] * BLK;
    } else if (dir == DUM_D2H) {
      src = pool + (uint64_t)frames[i] * BLK;
      dst = host + (uint64_t)blocks[i] * BLK;
    } else {
      src = pool + (uint64_t)src_frames[i] * BLK;
      dst = pool + (uint64_t)frames[i] * BLK;
    }
    src += (uint64_t)c * BULK_TILE;
    dst += (uint64_t)c * BULK_TILE;
  };
  auto load = [&](uint64_t it, uint32_t s) {
    const char *src;
    char *dst;
    addr(it, src, dst);
    const uint32_t b = smem_u32(&bar[s]), t = smem_u32(tiles + (uint64_t)s * BULK_TILE);
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(b), "r"(BULK_TILE) : "memory");
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 ::"r"(t), "l"(src), "r"(BULK_TILE), "r"(b) : "memory");
  };
  // tiles of this CTA: it = blockIdx.x + j * gridDim.x; ring of NBULK stages
  uint32_t phase[NBULK] = {0, 0, 0, 0};
  uint64_t j = 0;
  for (uint32_t s = 0; s < NBULK; ++s) {
    const uint64_t it = blockIdx.x + (uint64_t)s * gridDim.x;
    if (it < items) load(it, s);
  }
  for (uint64_t it = blockIdx.x; it < items; it += gridDim.x, ++j) {
    const uint32_t s = (uint32_t)(j % NBULK);
    const uint32_t b = smem_u32(&bar[s]), t = smem_u32(tiles + (uint64_t)s * BULK_TILE);
    // the tile has landed
    asm volatile(
        "{\n\t.reg .pred p;\n\tWAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
        "@!p bra WAIT_%=;\n\t}" ::"r"(b), "r"(phase[s]) : "memory");
    phase[s] ^= 1u;
    const char *src;
    char *dst;
    addr(it, src, dst);
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst), "r"(t), "r"(BULK_TILE)
                 : "memory");
    asm volatile("cp.async.bulk.commit_group;" ::: "memory");
    // refill this stage once its store has read the tile
    const uint64_t nxt = it + (uint64_t)NBULK * gridDim.x;
    if (nxt < items) {
      asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
      load(nxt, s);
    }
  }
  asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}

constexpr int SUM_NT = 512;
__global__ void __launch_bounds__(SUM_NT) k_checksums(const uint32_t *__restrict__ ids, const char *base,
                                                      unsigned long long *out) {
  __shared__ unsigned long long red[SUM_NT / 32];
  const uint64_t *p = reinterpret_cast<const uint64_t *>(base + (uint64_t)ids[blockIdx.x] * BLK);
  unsigned long long acc = 0;
  for (uint32_t w = threadIdx.x; w < BLK / 8; w += SUM_NT) acc += p[w] * (2ull * w + 1ull);
#pragma unroll
  for (int o = 16; o; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
  if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = acc;
  __syncthreads();
  if (threadIdx.x == 0) {
    unsigned long long t = 0;
    for (int k = 0; k < SUM_NT / 32; ++k) t += red[k];
    out[blockIdx.x] = t;
  }
}

// ---------------------------------------------------------------------------
cudaError_t launch_reset_residency(dum_engine *e, cudaStream_t s) {
  k_res_reset<<<256, 256, 0, s>>>(e->g.W, e->g.C, e->d_frame_of, e->d_stamp_of, e->d_block_of, e->d_free_bits,
                                  e->d_inactive_bits, e->d_res_bits, true, e->d_state);
  e->kernel_launches += 1;
  return cudaGetLastError();
}

cudaError_t launch_load_residency(dum_engine *e, const uint32_t *lrm, uint32_t n, cudaStream_t s) {
  TimerScope t(e, DUM_T_RESIDENCY, s);
  k_res_reset<<<256, 256, 0, s>>>(e->g.W, e->g.C, e->d_frame_of, e->d_stamp_of, e->d_block_of, e->d_free_bits,
                                  e->d_inactive_bits, e->d_res_bits, false, e->d_state);
  k_load_res<<<(n + 255) / 256 + 1, 256, 0, s>>>(lrm, n, e->g.W, e->d_frame_of, e->d_stamp_of, e->d_block_of,
                                                  e->d_free_bits, e->d_lrm_blk, e->d_lrm_stamp, e->d_res_bits,
                                                  e->d_inactive_bits, e->d_logpos, e->d_state);
  e->kernel_launches += 2;
  return cudaGetLastError();
}

cudaError_t launch_mark_inactive(dum_engine *e, const uint32_t *blocks, uint32_t n, int flag, cudaStream_t s) {
  if (n == 0) return cudaSuccess;
  k_mark_inactive<<<(n + 255) / 256, 256, 0, s>>>(blocks, n, flag, e->g.W, e->d_inactive_bits, e->d_frame_of,
                                                  e->d_logpos, e->d_lrm_blk, e->d_state);
  e->kernel_launches += 1;
  return cudaGetLastError();
}

static int copy_sms(const dum_engine *e) {
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  return e->copy_sms && (int)e->copy_sms < sms ? (int)e->copy_sms : sms;
}

static int copy_grid(const dum_engine *e, uint32_t n) {
  const int sms = copy_sms(e);
  const uint64_t items = (uint64_t)(n ? n : 1) * CHUNKS;
  const uint64_t g = std::min<uint64_t>(items, (uint64_t)sms * 8);
  return (int)g;
}

cudaError_t launch_migrate(dum_engine *e, int dir, const uint32_t *blocks, const uint32_t *dst, uint32_t n,
                           uint32_t method, cudaStream_t s, const uint64_t *rng) {
  MigArgs a;
  a.dir = dir;
  a.blocks = blocks;
  a.dst = dst;
  a.n = n;
  a.rng = rng;
  a.W = e->g.W;
  a.C = e->g.C;
  a.frame_of = e->d_frame_of;
  a.stamp_of = e->d_stamp_of;
  a.block_of = e->d_block_of;
  a.free_bits = e->d_free_bits;
  a.lrm_blk = e->d_lrm_blk;
  a.lrm_stamp = e->d_lrm_stamp;
  a.res_bits = e->d_res_bits;
  a.logpos = e->d_logpos;
  a.inactive = e->d_inactive_bits;
  a.lrm_cap = e->lrm_cap;
  a.mig_frames = e->d_mig_frames;
  a.mig_src = e->d_mig_src;
  a.mig_blocks = e->d_mig_blocks;
  a.st = e->d_state;
  {
    TimerScope t(e, DUM_T_MIG_PLAN, s);
    k_mig_plan<<<1, PLAN_NT, 0, s>>>(a);
  }
  e->kernel_launches += 1;
  if (dir == DUM_INVALIDATE) return cudaGetLastError();
  // metadata-only engines (dum_simulate at B/G scale): the residency moves, no bytes
  if (!e->frame_pool || (dir != DUM_D2D && !e->host_arena)) return cudaGetLastError();
  const bool compaction = dir == DUM_D2D && blocks == nullptr;
  if (method == 2) {
    // copy-engine baseline: needs the plan on the host
    cudaError_t err = cudaStreamSynchronize(s);
    if (err != cudaSuccess) return err;
    DevState hs;
    if ((err = cudaMemcpy(&hs, e->d_state, sizeof(hs), cudaMemcpyDeviceToHost)) != cudaSuccess) return err;
    if (!hs.mig_ok) return cudaSuccess;
    const uint32_t m = hs.mig_n;
    std::vector<uint32_t> fr(m), bl(m), sr(m);
    if (m) {
      if ((err = cudaMemcpy(fr.data(), e->d_mig_frames, 4ull * m, cudaMemcpyDeviceToHost)) != cudaSuccess) return err;
      if ((err = cudaMemcpy(bl.data(), e->d_mig_blocks, 4ull * m, cudaMemcpyDeviceToHost)) != cudaSuccess) return err;
      if (dir == DUM_D2D &&
          (err = cudaMemcpy(sr.data(), e->d_mig_src, 4ull * m, cudaMemcpyDeviceToHost)) != cudaSuccess)
        return err;
    }
    uint32_t i = 0;
    while (i < m) {
      // coalesce runs contiguous on both sides
      uint32_t j = i + 1;
      auto sidx = [&](uint32_t k) { return dir == DUM_H2D ? bl[k] : (dir == DUM_D2H ? fr[k] : sr[k]); };
      auto didx = [&](uint32_t k) { return dir == DUM_H2D ? fr[k] : (dir == DUM_D2H ? bl[k] : fr[k]); };
      while (j < m && sidx(j) == sidx(j - 1) + 1 && didx(j) == didx(j - 1) + 1) ++j;
      const char *src = (dir == DUM_H2D ? e->host_arena : e->frame_pool) + (uint64_t)sidx(i) * BLK;
      char *dstp = (dir == DUM_D2H ? e->host_arena : e->frame_pool) + (uint64_t)didx(i) * BLK;
      cudaMemcpyKind kind = dir == DUM_H2D ? cudaMemcpyHostToDevice
                                           : (dir == DUM_D2H ? cudaMemcpyDeviceToHost : cudaMemcpyDeviceToDevice);
      err = cudaMemcpyAsync(dstp, src, (uint64_t)(j - i) * BLK, kind, s);
      if (err != cudaSuccess) return err;
      i = j;
    }
    return cudaSuccess;
  }
  if (method == 3) {  // TMA bulk copies: one CTA per SM, NBULK tiles in flight
    const size_t bsm = (size_t)NBULK * BULK_TILE;
    if (!e->bulk_smem) {
      cudaFuncSetAttribute(k_copy_bulk, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bsm);
      e->bulk_smem = 1;
    }
    const int sms = copy_sms(e);
    TimerScope t(e, DUM_T_COPY, s);
    k_copy_bulk<<<sms, 32, bsm, s>>>(dir, e->d_mig_blocks, e->d_mig_src, e->d_mig_frames, e->host_arena_dev,
                                     e->frame_pool, e->d_state);
    e->kernel_launches += 1;
    return cudaGetLastError();
  }
  const int grid = copy_grid(e, compaction ? e->g.C : n);
  TimerScope t(e, DUM_T_COPY, s);
  k_copy_blocks<<<grid, COPY_NT, 0, s>>>(dir, e->d_mig_blocks, e->d_mig_src, e->d_mig_frames, e->host_arena_dev,
                                         e->frame_pool, e->d_state);
  e->kernel_launches += 1;
  return cudaGetLastError();
}

cudaError_t launch_checksums(dum_engine *e, int where, const uint32_t *ids, uint32_t n, uint64_t *out,
                             cudaStream_t s) {
  if (n == 0) return cudaSuccess;
  const char *base = where == 0 ? e->frame_pool : e->host_arena_dev;
  k_checksums<<<n, SUM_NT, 0, s>>>(ids, base, reinterpret_cast<unsigned long long *>(out));
  e->kernel_launches += 1;
  return cudaGetLastError();
}

}  // namespace dum
