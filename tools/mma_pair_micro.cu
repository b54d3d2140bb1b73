// mma_pair_micro.cu — tcgen05 throughput probe: cta_group::1 (M = 128) vs cta_group::2 (M = 256 over a
// CTA pair, B split along N between the pair) for the rows kernel's shapes (development tool).
// Streaming: rounds of 8 K-steps (K = 128) issued back to back into two alternating accumulators,
// one wait at the end.  Reports cycles per MMA instruction and MACs per cycle PER SM.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o tools/mma_pair_micro tools/mma_pair_micro.cu
#include <algorithm>
#include <cstdio>
#include <vector>

#include "../paper_conf_asplos_miaoozcwzwzyssc24_b200/csrc/common.cuh"

using namespace specinfer;

__device__ __forceinline__ uint32_t cta_rank() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
}
__device__ __forceinline__ void cluster_sync() {
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}

// pair = 0: cta_group::1, M = 128.  pair = 1: cta_group::2, M = 256 (leader issues; each CTA holds its
// 128 rows of A and N/2 rows of B).  a_tmem: A from TMEM (TS) instead of smem (SS).
// (a kernel containing any cta_group::2 instruction must be launched as clusters: two instantiations)
template <int pair>
__global__ void __launch_bounds__(128, 1) probe(int N, int a_tmem, int reps, long long *out) {
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    uint8_t *smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
    uint8_t *sA = smem;            // 32 KB: 128 rows x 128 K (two 64-wide SW128 halves)
    uint8_t *sB = smem + 32768;    // <= 64 KB: N (or N/2) rows x 128 K
    __shared__ uint64_t bar;
    __shared__ uint32_t tbase;
    for (int i = threadIdx.x; i < (32768 + 65536) / 16; i += blockDim.x)
        reinterpret_cast<uint4 *>(smem)[i] = make_uint4(0x3c003c00u, 0x3c003c00u, 0, 0);
    fence_proxy_async_smem();
    if (threadIdx.x == 0) {
        mbar_init(&bar, 1);
        fence_barrier_init();
    }
    if (threadIdx.x < 32) {
        if constexpr (pair) {
            asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(smem_u32(&tbase)) : "memory");
            asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;" ::: "memory");
        } else {
            tmem_alloc<512>(&tbase);
        }
    }
    tc_fence_before();
    __syncthreads();
    if (pair) cluster_sync();
    tc_fence_after();
    const uint32_t tm = tbase;
    const bool leader = !pair || cta_rank() == 0;
    const int Nl = pair ? N / 2 : N;   // B rows held by this CTA
    if (threadIdx.x == 0 && leader) {
        const uint32_t idesc = make_idesc_bf16(pair ? 256 : 128, N, false, false);
        const uint32_t a0 = smem_u32(sA), b0 = smem_u32(sB);
        const long long t0 = clock64();
        for (int it = 0; it < reps; ++it) {
            for (int kk = 0; kk < 8; ++kk) {
                const uint64_t ad = make_smem_desc(a0 + (kk >> 2) * 16384 + (kk & 3) * 32, 16, 1024, kSw128);
                const uint64_t bd = make_smem_desc(b0 + (kk >> 2) * (Nl * 128) + (kk & 3) * 32, 16, 1024, kSw128);
                const uint32_t d = tm + (it & 1) * N;
                const uint32_t acc = kk > 0 ? 1u : 0u;
                if constexpr (pair) {
                    if (a_tmem)
                        asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                                     "tcgen05.mma.cta_group::2.kind::f16 [%0], [%1], %2, %3, p;\n\t}" ::"r"(d),
                                     "r"(tm + 2 * N + kk * 8), "l"(bd), "r"(idesc), "r"(acc) : "memory");
                    else
                        asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                                     "tcgen05.mma.cta_group::2.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(d),
                                     "l"(ad), "l"(bd), "r"(idesc), "r"(acc) : "memory");
                } else {
                    if (a_tmem)
                        asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                                     "tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n\t}" ::"r"(d),
                                     "r"(tm + 2 * N + kk * 8), "l"(bd), "r"(idesc), "r"(acc) : "memory");
                    else
                        umma_bf16_ss(d, ad, bd, idesc, acc);
                }
            }
        }
        if constexpr (pair)
            asm volatile("tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;"
                         ::"r"(smem_u32(&bar)), "h"((uint16_t)3) : "memory");
        else
            umma_commit(&bar);
        mbar_wait(&bar, 0);
        out[blockIdx.x] = clock64() - t0;
    } else if (threadIdx.x == 0 && pair) {
        mbar_wait(&bar, 0);   // the leader's multicast commit arrives here too
    }
    tc_fence_before();
    __syncthreads();
    if (pair) cluster_sync();
    if (threadIdx.x < 32) {
        tc_fence_after();
        if constexpr (pair)
            asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, 512;" ::"r"(tm) : "memory");
        else
            tmem_dealloc<512>(tm);
    }
}

int main() {
    long long *d_out;
    cudaMalloc(&d_out, 148 * sizeof(long long));
    cudaMemset(d_out, 0, 148 * sizeof(long long));
    const int smem = 32768 + 65536 + 1024;
    cudaFuncSetAttribute(probe<0>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    cudaFuncSetAttribute(probe<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    std::vector<long long> h(148);
    const int reps = 400;
    printf("streaming tcgen05.mma kind::f16, K = 16 per instruction, 8 per round, 2 accumulators:\n");
    for (int pair = 0; pair < 2; ++pair)
        for (int a_tmem = 0; a_tmem < 2; ++a_tmem)
            for (int N : {64, 128, 256}) {
                if (a_tmem && N > 128) continue;   // TMEM: 2 accumulators of N + A (64 cols)
                cudaLaunchConfig_t cfg = {};
                cfg.gridDim = dim3(148);
                cfg.blockDim = dim3(128);
                cfg.dynamicSmemBytes = smem;
                cudaLaunchAttribute attr[1];
                attr[0].id = cudaLaunchAttributeClusterDimension;
                attr[0].val.clusterDim.x = pair ? 2 : 1;
                attr[0].val.clusterDim.y = 1;
                attr[0].val.clusterDim.z = 1;
                cfg.attrs = attr;
                cfg.numAttrs = pair ? 1 : 0;
                cudaMemset(d_out, 0, 148 * sizeof(long long));
                cudaError_t e = pair ? cudaLaunchKernelEx(&cfg, probe<1>, N, a_tmem, reps, d_out)
                                     : cudaLaunchKernelEx(&cfg, probe<0>, N, a_tmem, reps, d_out);
                if (e == cudaSuccess) e = cudaDeviceSynchronize();
                if (e != cudaSuccess) {
                    printf("  pair=%d a_tmem=%d N=%d: error %s\n", pair, a_tmem, N, cudaGetErrorString(e));
                    return 1;
                }
                cudaMemcpy(h.data(), d_out, 148 * 8, cudaMemcpyDeviceToHost);
                std::vector<long long> v;
                for (auto x : h)
                    if (x > 0) v.push_back(x);
                std::sort(v.begin(), v.end());
                const double cyc = v[v.size() / 2] / (reps * 8.0);
                const double macs_per_sm = (pair ? 256.0 : 128.0) * N * 16 / cyc / (pair ? 2 : 1);
                printf("  %s M=%3d N=%3d A=%s : %7.1f cyc/MMA  %7.0f MAC/cyc/SM  (%.0f%% of 4096)\n",
                       pair ? "cta_group::2" : "cta_group::1", pair ? 256 : 128, N, a_tmem ? "TMEM" : "smem", cyc,
                       macs_per_sm, 100.0 * macs_per_sm / 4096.0);
            }
    return 0;
}
