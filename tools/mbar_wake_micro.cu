// mbar_wake_micro.cu — mbarrier wake-up latency probe (development tool): warp 0 lane 0 waits on an
// mbarrier phase, warp 1 lane 0 arrives after a delay; reports (waiter's clock after the wait) -
// (arriver's clock before the arrive), in SM cycles, for three wait loops:
//   0: mbarrier.try_wait.parity (no suspend-time hint; the kernels' mbar_wait)
//   1: mbarrier.try_wait.parity with suspendTimeHint = 32 ns
//   2: mbarrier.test_wait.parity spin (never suspends)
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o tools/mbar_wake_micro tools/mbar_wake_micro.cu
#include <cstdio>
#include <vector>
#include <algorithm>

#include "../paper_conf_asplos_miaoozcwzwzyssc24_b200/csrc/common.cuh"

using namespace specinfer;

template <int kMode>
__device__ __forceinline__ bool try_wait_mode(uint64_t *bar, uint32_t parity) {
    uint32_t ok;
    if (kMode == 0)
        asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}"
                     : "=r"(ok) : "r"(smem_u32(bar)), "r"(parity) : "memory");
    else if (kMode == 1)
        asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, 32;\n\tselp.u32 %0, 1, 0, p;\n\t}"
                     : "=r"(ok) : "r"(smem_u32(bar)), "r"(parity) : "memory");
    else
        asm volatile("{\n\t.reg .pred p;\n\tmbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}"
                     : "=r"(ok) : "r"(smem_u32(bar)), "r"(parity) : "memory");
    return ok != 0;
}

template <int kMode>
__global__ void probe(int delay, int reps, long long *out) {
    __shared__ uint64_t bar;
    __shared__ long long t_arr[64];
    if (threadIdx.x == 0) {
        mbar_init(&bar, 1);
        fence_barrier_init();
    }
    __syncthreads();
    long long acc = 0;
    for (int r = 0; r < reps; ++r) {
        if (threadIdx.x == 0) {
            while (!try_wait_mode<kMode>(&bar, r & 1)) {}
            const long long t = clock64();
            acc += t - t_arr[r & 63];
        } else if (threadIdx.x == 32) {
            const long long t0 = clock64();
            while (clock64() - t0 < delay) {}
            t_arr[r & 63] = clock64();
            __threadfence_block();
            mbar_arrive(&bar);
        }
        __syncthreads();
    }
    if (threadIdx.x == 0) out[blockIdx.x] = acc / reps;
}

int main() {
    long long *d;
    cudaMalloc(&d, 148 * 8);
    std::vector<long long> h(148);
    for (int mode = 0; mode < 3; ++mode)
        for (int delay : {200, 2000, 20000}) {
            if (mode == 0) probe<0><<<148, 64>>>(delay, 200, d);
            if (mode == 1) probe<1><<<148, 64>>>(delay, 200, d);
            if (mode == 2) probe<2><<<148, 64>>>(delay, 200, d);
            if (cudaDeviceSynchronize() != cudaSuccess) { printf("error\n"); return 1; }
            cudaMemcpy(h.data(), d, 148 * 8, cudaMemcpyDeviceToHost);
            std::sort(h.begin(), h.end());
            printf("  mode %d (%s) delay %6d cyc: wake latency median %lld, max %lld cycles\n", mode,
                   mode == 0 ? "try_wait        " : mode == 1 ? "try_wait hint 32" : "test_wait spin  ", delay,
                   h[74], h[147]);
        }
    return 0;
}
