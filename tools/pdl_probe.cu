// Probe: what a kernel boundary costs inside a CUDA graph on this GPU, with
// and without programmatic dependent launch (PDL).  A chain of K dependent
// small kernels (each reads the previous one's output), captured once and
// replayed; per-boundary cost = (chain time - K x kernel time) / K.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/pdl_probe tools/pdl_probe.cu && /tmp/pdl_probe
#include <cstdio>
#include <cuda_runtime.h>

#define CK(x)                                                                                  \
  do {                                                                                         \
    cudaError_t e_ = (x);                                                                      \
    if (e_ != cudaSuccess) {                                                                   \
      printf("%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e_));                       \
      return 1;                                                                                \
    }                                                                                          \
  } while (0)

template <bool PDL>
__global__ void step_kernel(const unsigned *in, unsigned *out, int n, int iters) {
  if (PDL) {
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    asm volatile("griddepcontrol.wait;" ::: "memory");
  }
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    unsigned v = __ldcg(in + i);
    for (int k = 0; k < iters; ++k) v = v * 1664525u + 1013904223u;
    out[i] = v;
  }
}

template <bool PDL>
static float chain(cudaStream_t s, unsigned *a, unsigned *b, int n, int K, int grid, int iters, int reps) {
  cudaGraph_t g;
  cudaGraphExec_t ge;
  cudaStreamBeginCapture(s, cudaStreamCaptureModeThreadLocal);
  for (int k = 0; k < K; ++k) {
    cudaLaunchConfig_t cfg = {};
    cudaLaunchAttribute at[1];
    cfg.gridDim = dim3(grid);
    cfg.blockDim = dim3(256);
    cfg.stream = s;
    if (PDL) {
      at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
      at[0].val.programmaticStreamSerializationAllowed = 1;
      cfg.attrs = at;
      cfg.numAttrs = 1;
    }
    cudaLaunchKernelEx(&cfg, step_kernel<PDL>, (const unsigned *)(k & 1 ? b : a), k & 1 ? a : b, n, iters);
  }
  cudaStreamEndCapture(s, &g);
  if (cudaGraphInstantiate(&ge, g, 0) != cudaSuccess) return -1.f;
  for (int r = 0; r < 3; ++r) cudaGraphLaunch(ge, s);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  cudaEventRecord(e0, s);
  for (int r = 0; r < reps; ++r) cudaGraphLaunch(ge, s);
  cudaEventRecord(e1, s);
  cudaEventSynchronize(e1);
  float ms = 0;
  cudaEventElapsedTime(&ms, e0, e1);
  cudaGraphExecDestroy(ge);
  cudaGraphDestroy(g);
  return 1000.f * ms / reps;  // us per chain
}

int main() {
  int sms = 0;
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  const int n = 1 << 20;
  unsigned *a, *b;
  CK(cudaMalloc(&a, 4ull * n));
  CK(cudaMalloc(&b, 4ull * n));
  CK(cudaMemset(a, 0, 4ull * n));
  cudaStream_t s;
  CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  printf("{\"sms\": %d, \"points\": [", sms);
  bool first = true;
  for (int grid : {sms, 4 * sms}) {
    for (int iters : {1, 64, 512}) {
      const int K = 20, reps = 50;
      const float one = chain<false>(s, a, b, n, 1, grid, iters, 200);
      const float plain = chain<false>(s, a, b, n, K, grid, iters, reps);
      const float pdl = chain<true>(s, a, b, n, K, grid, iters, reps);
      printf("%s{\"grid\": %d, \"iters\": %d, \"one_kernel_us\": %.2f, \"chain20_us\": %.2f, \"chain20_pdl_us\": %.2f,"
             " \"per_boundary_us\": %.2f, \"per_boundary_pdl_us\": %.2f}",
             first ? "" : ", ", grid, iters, one, plain, pdl, (plain - one) / (K - 1) - 0.f, (pdl - one) / (K - 1));
      first = false;
    }
  }
  printf("]}\n");
  CK(cudaGetLastError());
  return 0;
}
