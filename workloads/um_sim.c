/*
 * workloads/um_sim.c -- seeded synthetic INPUT generator (shared by the oracle
 * and the CUDA path as a source of inputs only; holds none of DeepUM's
 * arithmetic).
 *
 * It models the behaviour the paper assumes of the *baseline* NVIDIA UM driver
 * (Sec. 2.2-2.3, Fig. 3): a GPU access to a non-resident
 * 2 MiB UM block faults, the block is migrated in, and when no frame is free
 * the least-recently-migrated block is evicted ("the policy
 * implemented in the NVIDIA driver ... evicts pages that are least recently
 * migrated to the GPU").  No prefetch.  The output is "the fault trace of 2 MB
 * UM blocks grouped by kernel execution" that BASELINE.json's north_star names.
 *
 * Optional duplicate injection models the fault buffer holding several
 * entries of the same UM block ("there can be multiple fault
 * entries for the same page in the fault buffer").
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

static inline uint64_t sm64_next(uint64_t *s) {
    uint64_t z = (*s += 0x9E3779B97F4A7C15ull);
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

/*
 * Simulate n_iter repetitions of one iteration's access stream.
 *   access_off[K+1], access_blk[]: block ids each launch touches, in order.
 *   dup_ppm: per-fault probability (parts per million) of also emitting a
 *            duplicate record of one of the last 4 faulted blocks of the launch.
 * Outputs (may be NULL for a counting pass):
 *   fault_off[n_iter*K+1], fault_blk[fault_cap]
 *   snap_blk[n_iter*C], snap_cnt[n_iter]: resident blocks at the start of each
 *            iteration, oldest migration first.
 * Returns the number of fault records, or -1 on bad input / capacity.
 */
int64_t um_fifo_sim(uint32_t W, uint32_t C, uint32_t K,
                    const uint64_t *access_off, const uint32_t *access_blk,
                    uint32_t n_iter, uint64_t dup_seed, uint32_t dup_ppm,
                    uint64_t *fault_off, uint32_t *fault_blk, uint64_t fault_cap,
                    uint32_t *snap_blk, uint32_t *snap_cnt)
{
    if (C == 0 || W == 0) return -1;
    uint8_t *resident = (uint8_t *)calloc(W, 1);
    uint32_t *ring = (uint32_t *)malloc(sizeof(uint32_t) * (size_t)C);
    if (!resident || !ring) { free(resident); free(ring); return -1; }
    uint64_t head = 0, count = 0; /* FIFO ring of resident blocks */
    uint64_t nf = 0;
    uint64_t rng = dup_seed;
    uint32_t recent[4];
    for (uint32_t it = 0; it < n_iter; ++it) {
        if (snap_blk) {
            for (uint64_t i = 0; i < count; ++i)
                snap_blk[(uint64_t)it * C + i] = ring[(head + i) % C];
        }
        if (snap_cnt) snap_cnt[it] = (uint32_t)count;
        for (uint32_t k = 0; k < K; ++k) {
            uint64_t gk = (uint64_t)it * K + k;
            if (fault_off) fault_off[gk] = nf;
            uint32_t nrecent = 0;
            for (uint64_t a = access_off[k]; a < access_off[k + 1]; ++a) {
                uint32_t b = access_blk[a];
                if (b >= W) { free(resident); free(ring); return -1; }
                if (resident[b]) continue;
                /* fault: evict the least recently migrated block if full */
                if (count == C) {
                    uint32_t v = ring[head];
                    resident[v] = 0;
                    head = (head + 1) % C;
                    --count;
                }
                ring[(head + count) % C] = b;
                ++count;
                resident[b] = 1;
                if (fault_blk) {
                    if (nf >= fault_cap) { free(resident); free(ring); return -1; }
                    fault_blk[nf] = b;
                }
                ++nf;
                if (dup_ppm && nrecent) {
                    uint64_t r = sm64_next(&rng);
                    if ((r % 1000000ull) < dup_ppm) {
                        uint32_t d = recent[(r >> 32) % nrecent];
                        if (fault_blk) {
                            if (nf >= fault_cap) { free(resident); free(ring); return -1; }
                            fault_blk[nf] = d;
                        }
                        ++nf;
                    }
                }
                if (nrecent < 4) recent[nrecent++] = b;
                else { recent[0] = recent[1]; recent[1] = recent[2]; recent[2] = recent[3]; recent[3] = b; }
            }
        }
    }
    if (fault_off) fault_off[(uint64_t)n_iter * K] = nf;
    free(resident);
    free(ring);
    return (int64_t)nf;
}
