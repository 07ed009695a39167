// f3: the DeepUM runtime over real CUDA Unified
// Memory on B200 -- managed arena, launch interposition (exec-ID hashes of
// kernel name + arguments), CUPTI UM fault records where the
// driver provides them, and cudaMemPrefetchAsync driven by the engine's
// lists.  See include/deepum_um.h.  Built with the shared CUDA
// runtime (the interposed launches are PyTorch's and ours alike).
#include <cuda.h>
#include <cuda_runtime.h>
#include <cupti.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <string>
#include <unordered_map>
#include <vector>

#include "deepum_um.h"

namespace {

constexpr uint64_t BLK = 2ull << 20;   // UM block
constexpr uint64_t PAGE = 64ull << 10;  // one touched word per 64 KiB

__global__ void k_um_touch(const char *base, const uint32_t *blocks, uint32_t n, int *sink) {
  const uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
  if (i >= (uint64_t)n * (BLK / PAGE)) return;
  const uint32_t b = blocks[i / (BLK / PAGE)];
  const int v = *(const volatile int *)(base + (uint64_t)b * BLK + (i % (BLK / PAGE)) * PAGE);
  if (v == 0x7fffffff) *sink = v;
}

struct Launch {
  uint64_t hash;
  uint32_t corr;
  uint64_t t0 = 0, t1 = 0;
  std::vector<uint32_t> faults;
};

struct Fault {
  uint64_t t, addr;
};

uint64_t fnv(uint64_t h, const void *p, size_t n) {
  const unsigned char *c = static_cast<const unsigned char *>(p);
  for (size_t i = 0; i < n; ++i) {
    h ^= c[i];
    h *= 0x100000001b3ull;
  }
  return h;
}

}  // namespace

struct dum_um {
  int device = 0;
  uint32_t n_blocks = 0;
  char *base = nullptr;
  int *sink = nullptr;
  std::string err, fault_why = "fault records not requested";
  std::mutex mu;
  std::vector<Launch> launches;                  // since the last take
  std::unordered_map<uint32_t, size_t> by_corr;  // correlation id -> launch
  std::vector<Fault> faults;                     // CUPTI fault records not yet assigned
  bool intercepting = false, fault_on = false;
  CUpti_SubscriberHandle sub = nullptr;
};

namespace {

dum_um *g_um = nullptr;  // the intercepting runtime (one per process)
std::mutex g_mu;

void CUPTIAPI buf_req(uint8_t **buf, size_t *size, size_t *maxrec) {
  *size = 8 << 20;
  *buf = static_cast<uint8_t *>(aligned_alloc(8, *size));
  *maxrec = 0;
}

void CUPTIAPI buf_done(CUcontext, uint32_t, uint8_t *buf, size_t, size_t valid) {
  std::lock_guard<std::mutex> g(g_mu);
  dum_um *u = g_um;
  CUpti_Activity *rec = nullptr;
  while (u && cuptiActivityGetNextRecord(buf, valid, &rec) == CUPTI_SUCCESS) {
    std::lock_guard<std::mutex> l(u->mu);
    if (rec->kind == CUPTI_ACTIVITY_KIND_CONCURRENT_KERNEL || rec->kind == CUPTI_ACTIVITY_KIND_KERNEL) {
      const auto *k = reinterpret_cast<const CUpti_ActivityKernel9 *>(rec);
      auto it = u->by_corr.find(k->correlationId);
      if (it != u->by_corr.end()) {
        u->launches[it->second].t0 = k->start;
        u->launches[it->second].t1 = k->end;
      }
    } else if (rec->kind == CUPTI_ACTIVITY_KIND_UNIFIED_MEMORY_COUNTER) {
      const auto *m = reinterpret_cast<const CUpti_ActivityUnifiedMemoryCounter3 *>(rec);
      if (m->counterKind == CUPTI_ACTIVITY_UNIFIED_MEMORY_COUNTER_KIND_GPU_PAGE_FAULT)
        u->faults.push_back(Fault{m->start, m->address});
    }
  }
  free(buf);
}

// the execution ID of a launch is found by the hash of the kernel's
// name and arguments
void CUPTIAPI on_callback(void *ud, CUpti_CallbackDomain dom, CUpti_CallbackId cbid, const void *cbdata) {
  auto *u = static_cast<dum_um *>(ud);
  const auto *d = static_cast<const CUpti_CallbackData *>(cbdata);
  if (dom != CUPTI_CB_DOMAIN_RUNTIME_API || d->callbackSite != CUPTI_API_ENTER) return;
  if (cbid != CUPTI_RUNTIME_TRACE_CBID_cudaLaunchKernel_v7000 &&
      cbid != CUPTI_RUNTIME_TRACE_CBID_cudaLaunchKernel_ptsz_v7000)
    return;
  const auto *p = static_cast<const cudaLaunchKernel_v7000_params *>(d->functionParams);
  uint64_t h = 0xcbf29ce484222325ull;
  const char *name = d->symbolName ? d->symbolName : "";
  h = fnv(h, name, strlen(name));
  cudaFunction_t f = nullptr;
  if (cudaGetFuncBySymbol(&f, p->func) == cudaSuccess && p->args) {
    size_t off = 0, sz = 0;
    for (size_t i = 0; cuFuncGetParamInfo(reinterpret_cast<CUfunction>(f), i, &off, &sz) == CUDA_SUCCESS; ++i)
      if (p->args[i]) h = fnv(h, p->args[i], sz);
  }
  std::lock_guard<std::mutex> l(u->mu);
  u->by_corr[d->correlationId] = u->launches.size();
  Launch L;
  L.hash = h;
  L.corr = d->correlationId;
  u->launches.push_back(std::move(L));
}

const char *cupti_msg(CUptiResult r) {
  const char *m = "?";
  cuptiGetResultString(r, &m);
  return m;
}

}  // namespace

extern "C" {

dum_um *dum_um_create(uint32_t n_blocks, int device) {
  if (n_blocks == 0 || device < 0) return nullptr;
  auto *u = new dum_um;
  u->device = device;
  u->n_blocks = n_blocks;
  if (cudaSetDevice(device) != cudaSuccess ||
      cudaMallocManaged(reinterpret_cast<void **>(&u->base), (size_t)n_blocks * BLK) != cudaSuccess ||
      cudaMalloc(reinterpret_cast<void **>(&u->sink), 4) != cudaSuccess) {
    cudaGetLastError();
    delete u;
    return nullptr;
  }
  return u;
}

void dum_um_destroy(dum_um *u) {
  if (!u) return;
  if (u->intercepting) dum_um_intercept(u, 0, 0);
  cudaFree(u->base);
  cudaFree(u->sink);
  delete u;
}

void *dum_um_base(dum_um *u) { return u ? u->base : nullptr; }

const char *dum_um_last_error(dum_um *u) { return u ? u->err.c_str() : "null runtime"; }

int dum_um_intercept(dum_um *u, int enable, int faults) {
  if (!u) return DUM_EINVAL;
  std::lock_guard<std::mutex> g(g_mu);
  if (enable) {
    if (u->intercepting) return DUM_OK;
    if (g_um) {
      u->err = "another runtime intercepts launches";
      return DUM_EINVAL;
    }
    CUptiResult r;
    if ((r = cuptiActivityRegisterCallbacks(buf_req, buf_done)) != CUPTI_SUCCESS ||
        (r = cuptiActivityEnable(CUPTI_ACTIVITY_KIND_CONCURRENT_KERNEL)) != CUPTI_SUCCESS ||
        (r = cuptiSubscribe(&u->sub, on_callback, u)) != CUPTI_SUCCESS ||
        (r = cuptiEnableCallback(1, u->sub, CUPTI_CB_DOMAIN_RUNTIME_API,
                                 CUPTI_RUNTIME_TRACE_CBID_cudaLaunchKernel_v7000)) != CUPTI_SUCCESS ||
        (r = cuptiEnableCallback(1, u->sub, CUPTI_CB_DOMAIN_RUNTIME_API,
                                 CUPTI_RUNTIME_TRACE_CBID_cudaLaunchKernel_ptsz_v7000)) != CUPTI_SUCCESS) {
      u->err = std::string("CUPTI: ") + cupti_msg(r);
      return DUM_ECUDA;
    }
    u->fault_on = false;
    if (faults) {
      CUpti_ActivityUnifiedMemoryCounterConfig c;
      memset(&c, 0, sizeof(c));
      c.scope = CUPTI_ACTIVITY_UNIFIED_MEMORY_COUNTER_SCOPE_PROCESS_SINGLE_DEVICE;
      c.kind = CUPTI_ACTIVITY_UNIFIED_MEMORY_COUNTER_KIND_GPU_PAGE_FAULT;
      c.deviceId = (uint32_t)u->device;
      c.enable = 1;
      if ((r = cuptiActivityConfigureUnifiedMemoryCounter(&c, 1)) == CUPTI_SUCCESS &&
          (r = cuptiActivityEnable(CUPTI_ACTIVITY_KIND_UNIFIED_MEMORY_COUNTER)) == CUPTI_SUCCESS) {
        u->fault_on = true;
        u->fault_why = "CUPTI unified-memory GPU page-fault records";
      } else {
        u->fault_why = std::string("CUPTI unified-memory counters unavailable: ") + cupti_msg(r);
      }
    }
    g_um = u;
    u->intercepting = true;
    return DUM_OK;
  }
  if (!u->intercepting) return DUM_OK;
  cuptiActivityFlushAll(1);
  cuptiUnsubscribe(u->sub);
  cuptiActivityDisable(CUPTI_ACTIVITY_KIND_CONCURRENT_KERNEL);
  if (u->fault_on) cuptiActivityDisable(CUPTI_ACTIVITY_KIND_UNIFIED_MEMORY_COUNTER);
  u->sub = nullptr;
  u->intercepting = false;
  g_um = nullptr;
  return DUM_OK;
}

int dum_um_fault_source(dum_um *u, char *why, uint32_t cap) {
  if (!u) return DUM_EINVAL;
  if (why && cap) {
    strncpy(why, u->fault_why.c_str(), cap - 1);
    why[cap - 1] = 0;
  }
  return u->fault_on ? 1 : 0;
}

int dum_um_add_faults(dum_um *u, const uint32_t *blocks, uint32_t n) {
  if (!u || (n && !blocks)) return DUM_EINVAL;
  std::lock_guard<std::mutex> l(u->mu);
  if (u->launches.empty()) return DUM_EINVAL;
  auto &f = u->launches.back().faults;
  f.insert(f.end(), blocks, blocks + n);
  return DUM_OK;
}

int dum_um_take(dum_um *u, uint64_t *hashes, uint64_t *offsets, uint32_t *faults, uint32_t launch_cap,
                uint64_t fault_cap, uint32_t *n_launch, uint64_t *n_fault, uint64_t needed[2]) {
  if (!u || !n_launch || !n_fault) return DUM_EINVAL;
  if (u->intercepting) cuptiActivityFlushAll(1);  // kernel intervals and fault records delivered
  std::lock_guard<std::mutex> l(u->mu);
  // CUPTI faults -> the launch whose kernel interval holds them, in time order
  std::sort(u->faults.begin(), u->faults.end(), [](const Fault &a, const Fault &b) { return a.t < b.t; });
  for (const Fault &f : u->faults) {
    if (f.addr < (uint64_t)u->base || f.addr >= (uint64_t)u->base + (uint64_t)u->n_blocks * BLK) continue;
    for (auto &L : u->launches)
      if (L.t0 && f.t >= L.t0 && f.t <= L.t1) {
        L.faults.push_back((uint32_t)((f.addr - (uint64_t)u->base) / BLK));
        break;
      }
  }
  u->faults.clear();
  // first occurrence per launch (D2), CSR layout of dum_record_faults
  uint64_t nf = 0;
  std::vector<std::vector<uint32_t>> lists(u->launches.size());
  for (size_t i = 0; i < u->launches.size(); ++i) {
    std::vector<uint32_t> seen;
    for (uint32_t b : u->launches[i].faults)
      if (b < u->n_blocks && std::find(seen.begin(), seen.end(), b) == seen.end()) seen.push_back(b);
    nf += seen.size();
    lists[i] = std::move(seen);
  }
  if (u->launches.size() > launch_cap || nf > fault_cap) {
    if (needed) {
      needed[0] = u->launches.size();
      needed[1] = nf;
    }
    return DUM_ECAPACITY;
  }
  uint64_t o = 0;
  for (size_t i = 0; i < u->launches.size(); ++i) {
    hashes[i] = u->launches[i].hash;
    offsets[i] = o;
    for (uint32_t b : lists[i]) faults[o++] = b;
  }
  if (offsets) offsets[u->launches.size()] = o;
  *n_launch = (uint32_t)u->launches.size();
  *n_fault = o;
  u->launches.clear();
  u->by_corr.clear();
  return DUM_OK;
}

int dum_um_prefetch(dum_um *u, const uint32_t *blocks, uint32_t n, int to_device, dum_stream_t stream) {
  if (!u || (n && !blocks)) return DUM_EINVAL;
  cudaMemLocation loc{};
  loc.type = to_device ? cudaMemLocationTypeDevice : cudaMemLocationTypeHost;
  loc.id = to_device ? u->device : 0;
  for (uint32_t i = 0; i < n;) {
    uint32_t j = i + 1;
    while (j < n && blocks[j] == blocks[j - 1] + 1) ++j;  // a run of consecutive blocks: one call
    if (blocks[i] + (uint64_t)(j - i) > u->n_blocks) return DUM_EINVAL;
    const cudaError_t e = cudaMemPrefetchAsync(u->base + (uint64_t)blocks[i] * BLK, (size_t)(j - i) * BLK, loc, 0,
                                               (cudaStream_t)stream);
    if (e != cudaSuccess) {
      u->err = std::string("cudaMemPrefetchAsync: ") + cudaGetErrorString(e);
      return DUM_ECUDA;
    }
    i = j;
  }
  return DUM_OK;
}

int dum_um_touch(dum_um *u, const uint32_t *blocks_dev, uint32_t n, dum_stream_t stream) {
  if (!u || (n && !blocks_dev)) return DUM_EINVAL;
  if (!n) return DUM_OK;
  const uint64_t threads = (uint64_t)n * (BLK / PAGE);
  k_um_touch<<<(unsigned)((threads + 255) / 256), 256, 0, (cudaStream_t)stream>>>(u->base, blocks_dev, n, u->sink);
  const cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) {
    u->err = std::string("k_um_touch: ") + cudaGetErrorString(e);
    return DUM_ECUDA;
  }
  return DUM_OK;
}

}  // extern "C"
