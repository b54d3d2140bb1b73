// mma_issue_micro.cu — tcgen05.mma issue-path probe (development tool): the same stream of
// M = 128 kind::f16 MMAs (K = 16 each, 8 per K = 128 round, two alternating accumulators) issued
//   (a) by one divergent lane (`if (lane == 0)`, descriptors in per-thread registers -> R2UR +
//       ELECT loop per instruction: the rows / swapped kernels' issuer as of round 2), or
//   (b) by a whole warp with warp-uniform descriptors and `elect.sync` in the same asm block.
// Reports cycles per MMA instruction for N = 32, 64, 128, 256 (A and B from smem).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o tools/mma_issue_micro tools/mma_issue_micro.cu
#include <algorithm>
#include <cstdio>
#include <vector>

#include "../paper_conf_asplos_miaoozcwzwzyssc24_b200/csrc/common.cuh"

using namespace specinfer;

__device__ __forceinline__ void umma_ss_elect(uint32_t d_tmem, uint64_t adesc, uint64_t bdesc, uint32_t idesc,
                                              uint32_t accumulate) {
    asm volatile(
        "{\n\t.reg .pred p, e;\n\t"
        "setp.ne.b32 p, %4, 0;\n\t"
        "elect.sync _|e, 0xffffffff;\n\t"
        "@e tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(d_tmem),
        "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate)
        : "memory");
}
__device__ __forceinline__ void umma_commit_elect(uint64_t *bar) {
    asm volatile(
        "{\n\t.reg .pred e;\n\telect.sync _|e, 0xffffffff;\n\t"
        "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n\t}" ::"r"(smem_u32(bar))
        : "memory");
}

template <bool kWarp>
__global__ void __launch_bounds__(128, 1) probe(int N, int reps, long long *out) {
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    uint8_t *smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
    uint8_t *sA = smem;            // 32 KB: 128 rows x 128 K
    uint8_t *sB = smem + 32768;    // 64 KB: N rows x 128 K
    __shared__ uint64_t bar;
    __shared__ uint32_t tbase;
    for (int i = threadIdx.x; i < (32768 + 65536) / 16; i += blockDim.x)
        reinterpret_cast<uint4 *>(smem)[i] = make_uint4(0x3c003c00u, 0x3c003c00u, 0, 0);
    fence_proxy_async_smem();
    if (threadIdx.x == 0) {
        mbar_init(&bar, 1);
        fence_barrier_init();
    }
    if (threadIdx.x < 32) tmem_alloc<512>(&tbase);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tm = tbase;
    const uint32_t idesc = make_idesc_bf16(128, N, false, false);
    const uint32_t a0 = smem_u32(sA), b0 = smem_u32(sB);
    if (kWarp ? threadIdx.x < 32 : threadIdx.x == 0) {
        const long long t0 = clock64();
        for (int it = 0; it < reps; ++it) {
#pragma unroll
            for (int kk = 0; kk < 8; ++kk) {
                const uint64_t ad = make_smem_desc(a0 + (kk >> 2) * 16384 + (kk & 3) * 32, 16, 1024, kSw128);
                const uint64_t bd = make_smem_desc(b0 + (kk >> 2) * (N * 128) + (kk & 3) * 32, 16, 1024, kSw128);
                const uint32_t d = tm + (it & 1) * N;
                if (kWarp) umma_ss_elect(d, ad, bd, idesc, kk > 0 ? 1u : 0u);
                else umma_bf16_ss(d, ad, bd, idesc, kk > 0 ? 1u : 0u);
            }
        }
        if (kWarp) umma_commit_elect(&bar);
        else umma_commit(&bar);
        mbar_wait(&bar, 0);
        if (threadIdx.x == 0) out[blockIdx.x] = clock64() - t0;
    }
    tc_fence_before();
    __syncthreads();
    if (threadIdx.x < 32) {
        tc_fence_after();
        tmem_dealloc<512>(tm);
    }
}

int main() {
    long long *d_out;
    cudaMalloc(&d_out, 148 * sizeof(long long));
    const int smem = 32768 + 65536 + 1024;
    cudaFuncSetAttribute(probe<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    cudaFuncSetAttribute(probe<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    std::vector<long long> h(148);
    const int reps = 400;
    for (int w = 0; w < 2; ++w)
        for (int N : {32, 64, 128, 256}) {
            cudaMemset(d_out, 0, 148 * sizeof(long long));
            if (w) probe<true><<<148, 128, smem>>>(N, reps, d_out);
            else probe<false><<<148, 128, smem>>>(N, reps, d_out);
            cudaError_t e = cudaDeviceSynchronize();
            if (e != cudaSuccess) {
                printf("error %s\n", cudaGetErrorString(e));
                return 1;
            }
            cudaMemcpy(h.data(), d_out, 148 * 8, cudaMemcpyDeviceToHost);
            std::sort(h.begin(), h.end());
            const double cyc = h[74] / (reps * 8.0);
            printf("  %s N=%3d : %6.1f cyc/MMA  %6.0f MAC/cyc/SM (%.0f%% of 4096)\n",
                   w ? "warp + elect.sync" : "one lane         ", N, cyc, 128.0 * N * 16 / cyc,
                   100.0 * 128.0 * N * 16 / cyc / 4096.0);
        }
    return 0;
}
