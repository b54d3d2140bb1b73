// gather.cuh — NEXT-4a: the tokens-only exchange after verification (
// the request manager and the GPU workers "only communicate tokens") fused into
// the verifiers.  The CTA that finishes request b writes its packed row [n | tokens | nodes] straight
// into EVERY rank's receive table with peer stores (NVLink / NVSwitch peer-mapped memory, CUDA IPC),
// and the last request of a rank publishes an epoch flag on every rank with a system-scope release;
// specinfer_gather_wait acquires the flags of all ranks.  No collective launch, no host round trip.
//
// Per rank: recv [2][world * rows_per_rank][row_len] int32 (double-buffered by epoch parity, so a
// fast rank can write step s+1 while a slow one still reads step s), flags [world] uint32 (flags[r]
// = last epoch rank r published here), state [2] uint32 {epoch, requests done} (local).
#pragma once
#include "common.cuh"

namespace specinfer {

constexpr int kMaxPeers = SPECINFER_MAX_PEERS;

struct GatherDev {
    int32_t *recv[kMaxPeers];
    uint32_t *flags[kMaxPeers];
    uint32_t *state;
    int world, rank, rows_per_rank, row_len, nreq;   // world 0: no fused gather
};

__device__ __forceinline__ void st_release_sys(uint32_t *p, uint32_t v) {
    asm volatile("st.release.sys.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ uint32_t ld_acquire_sys(const uint32_t *p) {
    uint32_t v;
    asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ uint32_t ld_volatile_u32(const uint32_t *p) {
    uint32_t v;
    asm volatile("ld.volatile.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}

// Called by one full warp once request b's outputs (an / at, n) are final in global memory and
// visible to the warp (after __syncwarp / __syncthreads): the
// packed row goes to row (rank * rows_per_rank + b) of every rank's table (buffer epoch & 1); the
// warp of the rank's last request then releases epoch + 1 on every rank's flag `rank`.
__device__ __forceinline__ void gather_publish(const GatherDev &g, int b, int n, const int32_t *an,
                                               const int32_t *at, int Lp) {
    if (g.world <= 0) return;
    const int lane = threadIdx.x & 31;
    const uint32_t e = ld_volatile_u32(g.state);
    const size_t table = (size_t)g.world * g.rows_per_rank * g.row_len;
    const size_t row = ((size_t)g.rank * g.rows_per_rank + b) * g.row_len;
    for (int r = 0; r < g.world; ++r) {
        int32_t *dst = g.recv[r] + (size_t)(e & 1u) * table + row;
        for (int j = lane; j < g.row_len; j += 32)
            dst[j] = j == 0 ? n : (j <= Lp ? at[j - 1] : an[j - 1 - Lp]);
    }
    __threadfence_system();   // every lane's part of this row (all peers) before the count
    __syncwarp();
    if (lane == 0) {
        const unsigned old = atomicAdd(g.state + 1, 1u);
        if (old == (unsigned)(g.nreq - 1)) {
            __threadfence_system();   // every request's rows (fence cumulativity) before the flags
            g.state[1] = 0u;          // ready for the next step
            for (int r = 0; r < g.world; ++r) st_release_sys(g.flags[r] + g.rank, e + 1u);
        }
    }
}

}  // namespace specinfer
