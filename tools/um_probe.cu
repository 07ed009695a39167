// Probe (run under gpurun): does this box deliver CUPTI unified-memory GPU
// page-fault records, kernel activity records and launch callbacks with the
// kernel arguments?  Prints counts and the first records.
//   nvcc -gencode arch=compute_100a,code=sm_100a -I/usr/local/cuda/include tools/um_probe.cu \
//        -L/usr/local/cuda/lib64 -lcupti -lcuda -o /tmp/um_probe && /tmp/um_probe
#include <cuda.h>
#include <cuda_runtime.h>
#include <cupti.h>

#include <cstdio>
#include <cstdlib>
#include <cstring>

#define CK(x)                                                                          \
  do {                                                                                 \
    CUptiResult r_ = (x);                                                              \
    if (r_ != CUPTI_SUCCESS) {                                                         \
      const char *m_;                                                                  \
      cuptiGetResultString(r_, &m_);                                                   \
      printf("CUPTI error %s at %s:%d: %s\n", #x, __FILE__, __LINE__, m_);            \
    }                                                                                  \
  } while (0)

static int n_fault = 0, n_kernel = 0, n_htod = 0, n_other = 0, n_cb = 0;

static void CUPTIAPI buf_req(uint8_t **buf, size_t *size, size_t *maxrec) {
  *size = 16 << 20;
  *buf = (uint8_t *)aligned_alloc(8, *size);
  *maxrec = 0;
}

static void CUPTIAPI buf_done(CUcontext, uint32_t, uint8_t *buf, size_t, size_t valid) {
  CUpti_Activity *rec = nullptr;
  while (cuptiActivityGetNextRecord(buf, valid, &rec) == CUPTI_SUCCESS) {
    if (rec->kind == CUPTI_ACTIVITY_KIND_UNIFIED_MEMORY_COUNTER) {
      auto *u = (CUpti_ActivityUnifiedMemoryCounter3 *)rec;
      if (u->counterKind == CUPTI_ACTIVITY_UNIFIED_MEMORY_COUNTER_KIND_GPU_PAGE_FAULT) {
        if (n_fault < 12)
          printf("fault addr=%llx value=%llu start=%llu end=%llu src=%u flags=%u\n",
                 (unsigned long long)u->address, (unsigned long long)u->value, (unsigned long long)u->start,
                 (unsigned long long)u->end, u->srcId, u->flags);
        ++n_fault;
      } else if (u->counterKind == CUPTI_ACTIVITY_UNIFIED_MEMORY_COUNTER_KIND_BYTES_TRANSFER_HTOD) {
        if (n_htod < 4)
          printf("htod addr=%llx bytes=%llu start=%llu\n", (unsigned long long)u->address,
                 (unsigned long long)u->value, (unsigned long long)u->start);
        ++n_htod;
      } else {
        ++n_other;
      }
    } else if (rec->kind == CUPTI_ACTIVITY_KIND_CONCURRENT_KERNEL || rec->kind == CUPTI_ACTIVITY_KIND_KERNEL) {
      auto *k = (CUpti_ActivityKernel9 *)rec;
      printf("kernel %s corr=%u start=%llu end=%llu\n", k->name, k->correlationId, (unsigned long long)k->start,
             (unsigned long long)k->end);
      ++n_kernel;
    } else {
      ++n_other;
    }
  }
  free(buf);
}

static void CUPTIAPI on_cb(void *, CUpti_CallbackDomain dom, CUpti_CallbackId cbid, const void *cbdata) {
  auto *d = (const CUpti_CallbackData *)cbdata;
  if (d->callbackSite != CUPTI_API_ENTER) return;
  if (dom == CUPTI_CB_DOMAIN_RUNTIME_API && cbid == CUPTI_RUNTIME_TRACE_CBID_cudaLaunchKernel_v7000) {
    auto *p = (const cudaLaunchKernel_v7000_params *)d->functionParams;
    cudaFunction_t f = nullptr;
    cudaGetFuncBySymbol(&f, p->func);
    size_t off = 0, sz = 0, np = 0, tot = 0;
    while (cuFuncGetParamInfo((CUfunction)f, np, &off, &sz) == CUDA_SUCCESS) {
      tot += sz;
      ++np;
    }
    printf("launch cb %s corr=%u params=%zu bytes=%zu\n", d->symbolName ? d->symbolName : "?", d->correlationId,
           np, tot);
    ++n_cb;
  }
}

__global__ void touch(const int *p, size_t n_pages, size_t stride, int *out) {
  size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x;
  int s = 0;
  if (i < n_pages) s = p[i * stride];
  if (s == 12345) out[0] = s;
}

int main(int argc, char **argv) {
  // mode: bit4 = cuInit first; bit5 = enable before configure; bit0 = configure before the CUDA context; bit1 = all-devices scope;
  //       bit2 = page faults only; bit3 = transfers only
  const int mode = argc > 1 ? atoi(argv[1]) : 0;
  if (mode & 16) printf("cuInit: %d\n", (int)cuInit(0));
  if (!(mode & 1)) cudaFree(0);
  CUpti_ActivityUnifiedMemoryCounterConfig cfg[2];
  memset(cfg, 0, sizeof(cfg));
  cfg[0].scope = CUPTI_ACTIVITY_UNIFIED_MEMORY_COUNTER_SCOPE_PROCESS_SINGLE_DEVICE;
  cfg[0].kind = CUPTI_ACTIVITY_UNIFIED_MEMORY_COUNTER_KIND_GPU_PAGE_FAULT;
  cfg[0].deviceId = 0;
  cfg[0].enable = 1;
  cfg[1] = cfg[0];
  cfg[1].kind = CUPTI_ACTIVITY_UNIFIED_MEMORY_COUNTER_KIND_BYTES_TRANSFER_HTOD;
  if (mode & 2) cfg[0].scope = cfg[1].scope = CUPTI_ACTIVITY_UNIFIED_MEMORY_COUNTER_SCOPE_PROCESS_ALL_DEVICES;
  if (mode & 8) cfg[0] = cfg[1];
  printf("mode %d\n", mode);
  CK(cuptiActivityRegisterCallbacks(buf_req, buf_done));
  if (mode & 32) CK(cuptiActivityEnable(CUPTI_ACTIVITY_KIND_UNIFIED_MEMORY_COUNTER));
  CK(cuptiActivityConfigureUnifiedMemoryCounter(cfg, (mode & 12) ? 1 : 2));
  CK(cuptiActivityEnable(CUPTI_ACTIVITY_KIND_UNIFIED_MEMORY_COUNTER));
  CK(cuptiActivityEnable(CUPTI_ACTIVITY_KIND_CONCURRENT_KERNEL));
  CUpti_SubscriberHandle sub;
  CK(cuptiSubscribe(&sub, (CUpti_CallbackFunc)on_cb, nullptr));
  CK(cuptiEnableCallback(1, sub, CUPTI_CB_DOMAIN_RUNTIME_API, CUPTI_RUNTIME_TRACE_CBID_cudaLaunchKernel_v7000));

  const size_t bytes = 64ull << 21;  // 64 UM blocks of 2 MiB
  int *p = nullptr, *out = nullptr;
  printf("cudaMallocManaged: %d\n", (int)cudaMallocManaged(&p, bytes));
  cudaMalloc(&out, 4);
  memset(p, 1, bytes);  // pages on the host
  int dev = 0, cma = 0, pma = 0;
  cudaDeviceGetAttribute(&cma, cudaDevAttrConcurrentManagedAccess, dev);
  cudaDeviceGetAttribute(&pma, cudaDevAttrPageableMemoryAccess, dev);
  printf("concurrentManagedAccess=%d pageableMemoryAccess=%d\n", cma, pma);
  // kernel 1: touch blocks 0..7 (one int per 64 KiB page)
  touch<<<(8 * 32 + 255) / 256, 256>>>(p, 8 * 32, 16384, out);
  // prefetch blocks 8..15 to the GPU, then touch them: no faults expected
  cudaMemLocation loc{};
  loc.type = cudaMemLocationTypeDevice;
  loc.id = 0;
  printf("prefetch: %d\n", (int)cudaMemPrefetchAsync((char *)p + (8ull << 21), 8ull << 21, loc, 0, 0));
  touch<<<(8 * 32 + 255) / 256, 256>>>(p + (8ull << 21) / 4, 8 * 32, 16384, out);
  cudaDeviceSynchronize();
  printf("sync: %s\n", cudaGetErrorString(cudaGetLastError()));
  CK(cuptiActivityFlushAll(1));
  printf("SUMMARY faults=%d kernels=%d htod=%d other=%d launch_cbs=%d\n", n_fault, n_kernel, n_htod, n_other, n_cb);
  return 0;
}
