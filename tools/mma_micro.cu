// mma_micro.cu — tcgen05 throughput probe for the tree-attention MMA shapes (development tool).
// Measures cycles per tcgen05.mma (kind::f16, cta_group::1, M=128) for N in {16,32,64,128,256},
// A K-major (SW128) vs MN-major (SW128), with the 8 K-steps of one head accumulating into 1, 2 or
// 4 independent TMEM accumulators.  One CTA per SM, operands resident in smem (no HBM traffic).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o tools/mma_micro tools/mma_micro.cu
#include <cstdio>
#include <vector>
#include <algorithm>

#include "../paper_conf_asplos_miaoozcwzwzyssc24_b200/csrc/common.cuh"

using namespace specinfer;

__global__ void __launch_bounds__(128, 1) mma_probe(int N, int a_mn, int nacc, int reps, long long *out) {
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    uint8_t *smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
    uint8_t *sA = smem;              // 32 KB: 128 x 128 bf16
    uint8_t *sB = smem + 32768;      // up to 64 KB: 256 x 128 bf16
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
    if (threadIdx.x == 0) {
        const uint32_t idesc = make_idesc_bf16(128, N, a_mn != 0, false);
        const uint32_t a0 = smem_u32(sA), b0 = smem_u32(sB);
        long long t0 = 0;
        for (int it = 0; it < reps + 1; ++it) {
            if (it == 1) t0 = clock64();
            for (int kk = 0; kk < 8; ++kk) {
                uint64_t ad;
                if (a_mn) ad = make_smem_desc(a0 + kk * 16 * 128, 16384, 1024, kSw128);
                else ad = make_smem_desc(a0 + (kk >> 2) * 16384 + (kk & 3) * 32, 16, 1024, kSw128);
                const uint64_t bd = make_smem_desc(b0 + (kk >> 2) * (N * 128) + (kk & 3) * 32, 16, 1024, kSw128);
                const int acc = kk % nacc;
                umma_bf16_ss(tm + acc * N, ad, bd, idesc, kk >= nacc ? 1u : 0u);
            }
            umma_commit(&bar);
            mbar_wait(&bar, it & 1);
        }
        const long long t1 = clock64();
        out[blockIdx.x] = (t1 - t0);
    }
    tc_fence_before();
    __syncthreads();
    if (threadIdx.x < 32) {
        tc_fence_after();
        tmem_dealloc<512>(tm);
    }
}

// Same, but the issue loop never waits: it issues `reps` rounds back to back and waits once
// (throughput of independent rounds into alternating accumulator sets).
__device__ __forceinline__ void umma_ts(uint32_t d_tmem, uint32_t a_tmem, uint64_t bdesc, uint32_t idesc,
                                        uint32_t accumulate) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "setp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n\t}" ::"r"(d_tmem),
        "r"(a_tmem), "l"(bdesc), "r"(idesc), "r"(accumulate)
        : "memory");
}

// a_mn: 0 = A K-major smem, 1 = A MN-major smem, 2 = A from TMEM (cols 256..); b_mn: B MN-major
__global__ void __launch_bounds__(128, 1) mma_probe_stream(int N, int a_mn, int reps, long long *out, int b_mn = 0) {
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    uint8_t *smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
    uint8_t *sA = smem;
    uint8_t *sB = smem + 32768;
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
    if (threadIdx.x == 0) {
        const uint32_t idesc = make_idesc_bf16(128, N, a_mn == 1, b_mn != 0);
        const uint32_t a0 = smem_u32(sA), b0 = smem_u32(sB);
        const long long t0 = clock64();
        for (int it = 0; it < reps; ++it) {
            for (int kk = 0; kk < 8; ++kk) {
                uint64_t ad;
                if (a_mn == 1) ad = make_smem_desc(a0 + kk * 16 * 128, 16384, 1024, kSw128);
                else ad = make_smem_desc(a0 + (kk >> 2) * 16384 + (kk & 3) * 32, 16, 1024, kSw128);
                const uint64_t bd = b_mn ? make_smem_desc(b0 + kk * 16 * 128, N * 128, 1024, kSw128)
                                         : make_smem_desc(b0 + (kk >> 2) * (N * 128) + (kk & 3) * 32, 16, 1024, kSw128);
                if (a_mn == 2) umma_ts(tm + (it & 1) * N, tm + 256 + kk * 8, bd, idesc, kk > 0 ? 1u : 0u);
                else umma_bf16_ss(tm + (it & 1) * N, ad, bd, idesc, kk > 0 ? 1u : 0u);
            }
        }
        umma_commit(&bar);
        mbar_wait(&bar, 0);
        out[blockIdx.x] = clock64() - t0;
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
    cudaFuncSetAttribute(mma_probe, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    cudaFuncSetAttribute(mma_probe_stream, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    std::vector<long long> h(148);
    const int reps = 200;
    printf("PV-like variants, N=128 (a: 0 K-major smem, 1 MN-major smem, 2 TMEM; b: 0 K-major, 1 MN-major):\n");
    for (int a = 0; a < 3; ++a)
        for (int b = 0; b < 2; ++b) {
            mma_probe_stream<<<148, 128, smem>>>(128, a, reps, d_out, b);
            cudaDeviceSynchronize();
            cudaMemcpy(h.data(), d_out, 148 * 8, cudaMemcpyDeviceToHost);
            std::sort(h.begin(), h.end());
            printf("  a=%d b=%d : %7.1f cyc/MMA\n", a, b, h[74] / (reps * 8.0));
        }
    return 0;
    printf("latency-bound rounds (8 MMAs + commit + wait per round), cycles per MMA (median over 148 SMs):\n");
    for (int a_mn = 0; a_mn < 2; ++a_mn)
        for (int N : {16, 32, 64, 128, 256})
            for (int nacc : {1, 2, 4}) {
                if (nacc * N > 512) continue;
                mma_probe<<<148, 128, smem>>>(N, a_mn, nacc, reps, d_out);
                cudaError_t e = cudaDeviceSynchronize();
                if (e != cudaSuccess) {
                    printf("error %s\n", cudaGetErrorString(e));
                    return 1;
                }
                cudaMemcpy(h.data(), d_out, 148 * 8, cudaMemcpyDeviceToHost);
                std::sort(h.begin(), h.end());
                printf("  A %s N=%3d acc=%d : %7.1f cyc/MMA  (round %7.1f)\n", a_mn ? "MN" : "K ", N, nacc,
                       h[74] / (reps * 8.0), h[74] / (double)reps);
            }
    printf("streaming (no waits between rounds, 2 accumulators alternating per round):\n");
    for (int a_mn = 0; a_mn < 2; ++a_mn)
        for (int N : {16, 32, 64, 128, 256}) {
            mma_probe_stream<<<148, 128, smem>>>(N, a_mn, reps, d_out);
            cudaDeviceSynchronize();
            cudaMemcpy(h.data(), d_out, 148 * 8, cudaMemcpyDeviceToHost);
            std::sort(h.begin(), h.end());
            const double cyc = h[74] / (reps * 8.0);
            printf("  A %s N=%3d : %7.1f cyc/MMA = %6.0f MAC/cyc\n", a_mn ? "MN" : "K ", N, cyc,
                   128.0 * N * 16 / cyc);
        }
    return 0;
}
