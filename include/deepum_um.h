/* DeepUM-B200 real-UM runtime.
 *
 * PAPER.md L134 (Section 3.1, DeepUM runtime): "wrapper functions for CUDA
 * memory allocation API functions to switch all GPU memory allocation
 * requests to UM space allocation requests"; L136: the runtime "computes the
 * hash value of the kernel name and arguments" of every launch and passes the
 * execution ID to the driver; L140-L158: the driver's fault-handling,
 * prefetching and migration threads.
 *
 * libdeepum_um.so puts that runtime on a B200 over CUDA Unified Memory:
 *   - a managed arena (cudaMallocManaged) of n_blocks 2 MiB UM blocks; the
 *     engine's block id is (address - base) >> 21 (D1);
 *   - launch interposition through CUPTI runtime-API callbacks on
 *     cudaLaunchKernel: per launch, hash = FNV-1a 64 of the kernel's symbol
 *     name followed by its parameter bytes (sizes from cuFuncGetParamInfo),
 *     i.e. the kernel name and arguments of P:L136;
 *   - GPU page-fault records from CUPTI unified-memory activity
 *     (CUPTI_ACTIVITY_UNIFIED_MEMORY_COUNTER_KIND_GPU_PAGE_FAULT), assigned to
 *     the launch whose kernel-activity interval holds the fault's timestamp.
 *     Where the driver refuses UM counters (measured on this pool:
 *     cuptiActivityEnable returns CUPTI_ERROR_INVALID_PARAMETER;
 *     profiles/r02_um_probe_*.log), dum_um_fault_source says so and the caller
 *     supplies faults itself (dum_um_add_faults);
 *   - migrations driven by the engine's lists: dum_um_prefetch issues
 *     cudaMemPrefetchAsync per run of consecutive blocks, to the GPU (a
 *     window's blocks) or to the host (write-back victims).
 * The launch log comes out in dum_record_faults's layout (hash per launch,
 * CSR offsets, fault blocks), first occurrence per launch kept (D2).
 *
 * Errors: DUM_EINVAL (bad arguments), DUM_ECUDA (a CUDA / CUPTI call failed;
 * dum_um_last_error says which), DUM_ECAPACITY (output too small: *needed
 * set, nothing taken). */
#ifndef DEEPUM_UM_H
#define DEEPUM_UM_H

#include <stdint.h>

#include "deepum_b200.h"

#ifdef __cplusplus
extern "C" {
#endif

typedef struct dum_um dum_um;

/* A managed arena of n_blocks UM blocks on CUDA device `device`; NULL on failure. */
dum_um *dum_um_create(uint32_t n_blocks, int device);
void dum_um_destroy(dum_um *u);
void *dum_um_base(dum_um *u);
const char *dum_um_last_error(dum_um *u);

/* Start / stop launch interposition (CUPTI callbacks; one runtime per process
 * may intercept).  With faults != 0, also CUPTI UM page-fault records. */
int dum_um_intercept(dum_um *u, int enable, int faults);

/* 1 if CUPTI UM fault records are flowing, 0 if not; why[] (if given, cap
 * bytes) gets the reason. */
int dum_um_fault_source(dum_um *u, char *why, uint32_t cap);

/* Faults of the most recent intercepted launch from another source (block
 * ids in the arena, in access order). */
int dum_um_add_faults(dum_um *u, const uint32_t *blocks, uint32_t n);

/* Take the launch log (flushing CUPTI buffers first): n_launch hashes,
 * offsets[n_launch + 1] into faults[]; returns DUM_ECAPACITY with
 * needed[0..1] = {launches, faults} if a capacity is too small. */
int dum_um_take(dum_um *u, uint64_t *hashes, uint64_t *offsets, uint32_t *faults, uint32_t launch_cap,
                uint64_t fault_cap, uint32_t *n_launch, uint64_t *n_fault, uint64_t needed[2]);

/* cudaMemPrefetchAsync of the listed blocks (host array), runs of consecutive
 * ids merged, to the GPU (to_device != 0) or to host memory, on `stream`. */
int dum_um_prefetch(dum_um *u, const uint32_t *blocks, uint32_t n, int to_device, dum_stream_t stream);

/* A kernel reading one word per 64 KiB page of the listed blocks (device
 * array): an access stream for tests and demos.  Launched through the
 * intercepted runtime API. */
int dum_um_touch(dum_um *u, const uint32_t *blocks_dev, uint32_t n, dum_stream_t stream);

#ifdef __cplusplus
}
#endif

#endif /* DEEPUM_UM_H */
