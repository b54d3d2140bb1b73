// tmem_micro.cu — TMEM load/store and MUFU ex2 throughput probe (development tool).
// One CTA per SM with W warps; each warp repeatedly reads (tcgen05.ld 32x32b.x32) or writes
// (tcgen05.st 32x32b.x16) its lane quarter of a 512-column TMEM allocation, or runs ex2.approx on
// 32 independent registers.  Prints bytes (or ex2) per SM clock.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o tools/tmem_micro tools/tmem_micro.cu
#include <algorithm>
#include <cstdio>

#include "../paper_conf_asplos_miaoozcwzwzyssc24_b200/csrc/common.cuh"

using namespace specinfer;

__device__ __forceinline__ void ld32(uint32_t taddr, uint32_t (&r)[32]) {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, "
        "%14, %15, %16, %17, %18, %19, %20, %21, %22, %23, %24, %25, %26, %27, %28, %29, %30, %31}, [%32];"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
          "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]),
          "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]),
          "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
        : "r"(taddr));
}

// mode 0: LDTM x32 (+wait each), mode 1: 4 x LDTM x32 then one wait, mode 2: STTM x16, mode 3: ex2
__global__ void __launch_bounds__(512, 1) probe(int mode, int reps, long long *cyc, uint32_t *sink) {
    __shared__ uint32_t tbase;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (warp == 0) tmem_alloc<512>(&tbase);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tm = tbase + ((uint32_t)((warp & 3) * 32) << 16) + (warp >> 2) * 64;
    uint32_t acc = 0;
    __syncthreads();
    long long t0 = clock64();
    if (mode == 0) {
        for (int i = 0; i < reps; ++i) {
            uint32_t r[32];
            ld32(tm + (i & 1) * 32, r);
            tmem_ld_wait();
#pragma unroll
            for (int k = 0; k < 32; ++k) acc ^= r[k];
        }
    } else if (mode == 1) {
        for (int i = 0; i < reps; i += 4) {
            uint32_t r[4][32];
            ld32(tm, r[0]);
            ld32(tm + 32, r[1]);
            ld32(tm + 256, r[2]);
            ld32(tm + 288, r[3]);
            tmem_ld_wait();
#pragma unroll
            for (int j = 0; j < 4; ++j)
#pragma unroll
                for (int k = 0; k < 32; ++k) acc += r[j][k];
        }
    } else if (mode == 2) {
        uint32_t w[16];
#pragma unroll
        for (int k = 0; k < 16; ++k) w[k] = k + lane;
        for (int i = 0; i < reps; ++i) {
            tmem_st16(tm + (i & 3) * 16, w);
            w[0] += 1;
        }
        tmem_st_wait();
    } else {
        float x[32];
#pragma unroll
        for (int k = 0; k < 32; ++k) x[k] = -0.001f * (k + lane);
        for (int i = 0; i < reps; ++i) {
#pragma unroll
            for (int k = 0; k < 32; ++k) x[k] = ex2(x[k]) - 1.0f;
        }
#pragma unroll
        for (int k = 0; k < 32; ++k) acc += __float_as_uint(x[k]);
    }
    __syncthreads();
    long long t1 = clock64();
    if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
    sink[blockIdx.x * blockDim.x + threadIdx.x] = acc;
    tc_fence_before();
    __syncthreads();
    if (warp == 0) {
        tc_fence_after();
        tmem_dealloc<512>(tbase);
    }
}

__device__ __forceinline__ void umma_ts(uint32_t d_tmem, uint32_t a_tmem, uint64_t bdesc, uint32_t idesc,
                                        uint32_t accumulate) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "setp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n\t}" ::"r"(d_tmem),
        "r"(a_tmem), "l"(bdesc), "r"(idesc), "r"(accumulate)
        : "memory");
}

// M=128 N=128 K=128 rounds (8 MMAs of K=16), streamed (one wait at the end), timed in ns.
// kind: 0 SS (A K-major smem, B K-major smem) = S = Q K^T;  1 TS (A TMEM, B MN-major) = O += P V;
//       2 TS (A TMEM, B K-major);  3 SS (B MN-major);  4 alternate rounds of kind 0 and kind 1
__device__ __forceinline__ uint32_t rnd_bf16x2(uint32_t i) {
    // two pseudo-random bf16 values ~ U(-2, 2)
    uint32_t h = i * 2654435761u;
    h ^= h >> 13;
    h *= 0x5bd1e995u;
    h ^= h >> 15;
    const float a = ((h & 0xFFFF) / 65536.0f) * 4.f - 2.f, b = ((h >> 16) / 65536.0f) * 4.f - 2.f;
    return pack_bf16x2(a, b);
}

__global__ void __launch_bounds__(128, 1) mma_shape(int kind, int acol, int dcol, int reps, long long *out,
                                                    int random = 0) {
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    uint8_t *smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
    __shared__ uint64_t bar;
    __shared__ uint32_t tbase;
    for (int i = threadIdx.x; i < 65536 / 16; i += blockDim.x)
        reinterpret_cast<uint4 *>(smem)[i] =
            random ? make_uint4(rnd_bf16x2(4 * i), rnd_bf16x2(4 * i + 1), rnd_bf16x2(4 * i + 2), rnd_bf16x2(4 * i + 3))
                   : make_uint4(0x3c003c00u, 0x3c003c00u, 0, 0);
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
    {
        // A operand region of the TS variants (cols acol .. acol + 63), every lane quarter
        uint32_t w[16];
        const int wq = threadIdx.x >> 5;
        for (int c = 0; c < 64; c += 16) {
            for (int k = 0; k < 16; ++k) w[k] = random ? rnd_bf16x2(threadIdx.x * 977 + c * 31 + k) : 0x3c003c00u;
            tmem_st16(tm + ((uint32_t)(wq * 32) << 16) + acol + c, w);
        }
        tmem_st_wait();
    }
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    if (threadIdx.x == 0) {
        const uint32_t idesc_k = make_idesc_bf16(128, 128, false, false);
        const uint32_t idesc_mn = make_idesc_bf16(128, 128, false, true);
        const uint32_t a0 = smem_u32(smem), b0 = smem_u32(smem + 32768);
        unsigned long long t0;
        asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t0));
        for (int it = 0; it < reps; ++it) {
            const int k = kind == 4 ? (it & 1) : kind;
            for (int kk = 0; kk < 8; ++kk) {
                const uint64_t ad = make_smem_desc(a0 + (kk >> 2) * 16384 + (kk & 3) * 32, 16, 1024, kSw128);
                const uint64_t bk = make_smem_desc(b0 + (kk >> 2) * 16384 + (kk & 3) * 32, 16, 1024, kSw128);
                const uint64_t bmn = make_smem_desc(b0 + kk * 16 * 128, 16384, 1024, kSw128);
                if (k == 0) umma_bf16_ss(tm + (kind == 4 ? 0 : dcol), ad, bk, idesc_k, kk > 0 ? 1u : 0u);
                else if (k == 1) umma_ts(tm + dcol, tm + acol + kk * 8, bmn, idesc_mn, kk > 0 ? 1u : 0u);
                else if (k == 2) umma_ts(tm + dcol, tm + acol + kk * 8, bk, idesc_k, kk > 0 ? 1u : 0u);
                else umma_bf16_ss(tm + dcol, ad, bmn, idesc_mn, kk > 0 ? 1u : 0u);
            }
        }
        umma_commit(&bar);
        mbar_wait(&bar, 0);
        unsigned long long t1;
        asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t1));
        out[blockIdx.x] = (long long)(t1 - t0);
    }
    tc_fence_before();
    __syncthreads();
    if (threadIdx.x < 32) {
        tc_fence_after();
        tmem_dealloc<512>(tm);
    }
}

int main() {
    long long *cyc;
    uint32_t *sink;
    cudaMalloc(&cyc, 148 * 8);
    cudaMalloc(&sink, 148 * 512 * 4);
    const char *names[4] = {"LDTM x32 + wait", "4 x LDTM x32, 1 wait", "STTM x16", "MUFU ex2"};
    for (int mode = 0; mode < 0; ++mode) {
        for (int warps : {4, 8, 16}) {
            const int reps = 4096;
            probe<<<148, warps * 32>>>(mode, reps, cyc, sink);
            cudaError_t e = cudaDeviceSynchronize();
            if (e != cudaSuccess) {
                printf("error %s\n", cudaGetErrorString(e));
                return 1;
            }
            long long h[148];
            cudaMemcpy(h, cyc, sizeof(h), cudaMemcpyDeviceToHost);
            double c = (double)h[0];
            double per_sm;
            const char *unit;
            if (mode <= 1) {
                per_sm = (double)warps * reps * 32 * 32 * 4 / c;
                unit = "B/clk/SM";
            } else if (mode == 2) {
                per_sm = (double)warps * reps * 32 * 16 * 4 / c;
                unit = "B/clk/SM";
            } else {
                per_sm = (double)warps * reps * 32 * 32 / c;
                unit = "ex2/clk/SM";
            }
            printf("%-22s warps %2d: %8.0f cycles, %7.1f %s\n", names[mode], warps, c, per_sm, unit);
        }
    }
    cudaFuncSetAttribute(mma_shape, cudaFuncAttributeMaxDynamicSharedMemorySize, 160 * 1024);
    struct V { int kind, acol, dcol; const char *name; };
    const V vs[] = {{0, 0, 0, "SS Kmaj D@0        (S=QK^T)"}, {0, 0, 256, "SS Kmaj D@256"},
                    {1, 0, 256, "TS MN A@0 D@256    (our PV)"}, {1, 128, 384, "TS MN A@128 D@384  (our PV)"},
                    {1, 256, 0, "TS MN A@256 D@0"}, {1, 0, 128, "TS MN A@0 D@128"},
                    {2, 0, 256, "TS Kmaj A@0 D@256"}, {2, 256, 0, "TS Kmaj A@256 D@0"},
                    {3, 0, 256, "SS B-MN D@256"}, {4, 0, 256, "alternate S / PV rounds"}};
    for (int warm = 0; warm < 3; ++warm)
        for (const V &v : vs) {
            const int reps = 512;
            mma_shape<<<148, 128, 160 * 1024>>>(v.kind, v.acol, v.dcol, reps, cyc, warm == 2);
            cudaError_t e = cudaDeviceSynchronize();
            if (e != cudaSuccess) {
                printf("error %s\n", cudaGetErrorString(e));
                return 1;
            }
            long long h[148];
            cudaMemcpy(h, cyc, sizeof(h), cudaMemcpyDeviceToHost);
            std::sort(h, h + 148);
            const double ns = (double)h[74] / (reps * 8.0);
            if (warm) printf("%s %-30s: %6.1f ns per 128x128x16 MMA = %6.0f TFLOP/s chip\n", warm == 2 ? "random" : "const ", v.name, ns,
                             128.0 * 128 * 16 * 2 * 148 / ns / 1e3);
        }
    return 0;
}
