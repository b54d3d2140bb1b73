// common.cuh — sm_100a PTX building blocks (mbarrier, TMA, tcgen05/TMEM) and the workspace
// layout shared by the kernels of libspecinfer.so.  B200-only: compiled for sm_100a.
#pragma once

#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>

#include "../../include/specinfer.h"

namespace specinfer {

constexpr int kHeadDim = 128;
constexpr int kKeyTile = 128;        // keys per KV tile (= UMMA M of the swapped S^T = K Q^T)
constexpr int kMaxNodes = 256;       // Nmax limit (8 x 32-bit words of ancestor bitset)
constexpr int kBitWords = kMaxNodes / 32;
constexpr int kMaxCtasPerSm = 2;

// ------------------------------------------------------------------------------------------
// workspace layout (offsets in bytes, each region 256-aligned)
// ------------------------------------------------------------------------------------------
struct WsLayout {
    size_t status;      // int32[64]: [0] sticky status bits, [1] total tiles
    size_t req_ok;      // int32[B]
    size_t anc;         // uint32[B][Nmax][8]   ancestor-or-self bitsets
    size_t desc;        // uint32[B][Nmax][8]   descendant-or-self bitsets
    size_t rowmask;     // uint64[B][chunks][Nmax] query rows of chunk c that see tree key j
    size_t item_start;  // int32[n_items + 1]   tile prefix of the attention schedule
    size_t item_cnt;    // uint32[n_items]       split-combine counters
    size_t item_info;   // int4[n_items]         {first tile, end tile, P_b, n_b}
    size_t cta_info;    // int4[max_ctas][2]     {t0, t1, first item, total tiles}, item_info[first item]
    size_t dyn_ctr;     // uint32                 rows kernel's dynamic item tickets (reset by tree_prepare)
    size_t part_o;      // float[max_ctas][2][NT][128]
    size_t part_ml;     // float[max_ctas][2][2][NT]
    size_t argmax;      // int32[B][Nmax]
    size_t verify_cnt;  // uint32[2][B]          last-CTA counters: greedy, MSS
    size_t mss_p;       // float[B][2][V]        MSS residual distributions (double buffer)
    size_t total;
    int nt;             // query rows per chunk (UMMA N): 16, 32 or 64
    int npc;            // tree nodes per chunk = nt / G
    int chunks;         // chunks per (b, kv-head) item = ceil(Nmax / npc)
    int n_items;        // B * Hkv * chunks
    int lanes;          // CTAs sharing one KV stream in lock-step (rows kernel: chunks; else 1)
    int grid;           // attention CTAs: the largest multiple of `lanes` <= the SM count, or
                        // n_items * splitk in split-KV mode
    int splitk;         // > 1: split-KV mode, each item's tiles split over a cluster of splitk CTAs
    int max_ctas;
};

inline size_t align256(size_t x) { return (x + 255) & ~size_t(255); }

// Query rows per work item.  Up to 64 rows (G * Nmax <= 64): the "swapped" kernel (keys as the
// UMMA M dimension, NT = 16/32/64 rows as N).  Wider trees / GQA groups: the rows-as-M kernel with
// 128-row blocks (kRowsBlock), one TMEM lane per query row.
constexpr int kRowsBlock = 128;
inline int choose_nt(int G, int nmax) {
    const int r = G * nmax;
    if (r <= 16 && G <= 16) return 16;
    if (r <= 32 && G <= 32) return 32;
    if (r <= 64) return 64;
    return kRowsBlock;
}

inline WsLayout ws_layout(const specinfer_shape_t &s, int num_sms, bool allow_split_kv = true) {
    WsLayout w{};
    const int B = s.batch, N = s.max_nodes;
    const int G = s.num_q_heads / s.num_kv_heads;
    w.nt = choose_nt(G, N);
    w.npc = w.nt / G;
    w.chunks = (N + w.npc - 1) / w.npc;
    w.n_items = B * s.num_kv_heads * w.chunks;
    w.lanes = (w.nt == kRowsBlock && w.chunks > 1 && 2 * w.chunks <= num_sms) ? w.chunks : 1;
    // split-KV mode (swapped kernel, few items: batch 1-4 decoding): every item gets a thread-block
    // cluster of splitk CTAs, each streaming a contiguous part of its tiles, merged through DSMEM;
    // otherwise the persistent stream-K / one-unit-per-CTA schedule
    w.splitk = 1;
    // (only when an item can span enough 128-key tiles for the split to pay for the cluster merge:
    // the schedule keeps items shorter than 12 tiles whole on rank 0)
    if (allow_split_kv && w.nt != kRowsBlock && w.lanes == 1 && (s.max_seq + 127) / 128 >= 12) {
        int k = 1;
        // rank 0 gathers the k partials ([nt][128] + 2 [nt] floats each) in its K/V rings (>= 160 KB)
        const int kmax = w.nt == 64 ? 4 : 8;
        while (k < kmax && (long long)w.n_items * k * 2 <= num_sms) k *= 2;
        w.splitk = k;
    }
    w.grid = w.splitk > 1 ? w.n_items * w.splitk : (num_sms / w.lanes) * w.lanes;
    w.max_ctas = num_sms * kMaxCtasPerSm;
    size_t o = 0;
    auto take = [&](size_t bytes) { size_t r = o; o = align256(o + bytes); return r; };
    w.status = take(64 * 4);
    w.req_ok = take(size_t(B) * 4);
    w.anc = take(size_t(B) * N * kBitWords * 4);
    w.desc = take(size_t(B) * N * kBitWords * 4);
    w.rowmask = take(size_t(B) * w.chunks * N * 8);
    w.item_start = take(size_t(w.n_items + 1) * 4);
    w.item_cnt = take(size_t(w.n_items) * 4);
    w.item_info = take(size_t(w.n_items + 1) * 16);  // + sentinel
    w.cta_info = take(size_t(w.max_ctas) * 32);
    w.dyn_ctr = take(4);
    w.part_o = take(size_t(w.max_ctas) * 2 * w.nt * kHeadDim * 4);
    w.part_ml = take(size_t(w.max_ctas) * 2 * 2 * w.nt * 4);
    w.argmax = take(size_t(B) * N * 4);
    w.verify_cnt = take(size_t(B) * 2 * 4);
    w.mss_p = take(size_t(B) * 2 * (size_t)(s.vocab > 0 ? s.vocab : 1) * 4);
    w.total = o;
    return w;
}

enum StatusBits : int32_t {
    kStatusBadTree = 1,
};

// ------------------------------------------------------------------------------------------
// PTX helpers
// ------------------------------------------------------------------------------------------
__device__ __forceinline__ uint32_t smem_u32(const void *p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ void mbar_init(uint64_t *bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}

__device__ __forceinline__ void fence_barrier_init() {
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}

__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t *bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)),
                 "r"(bytes)
                 : "memory");
}

__device__ __forceinline__ void mbar_arrive(uint64_t *bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}

__device__ __forceinline__ bool mbar_try_wait(uint64_t *bar, uint32_t parity) {
    uint32_t ok;
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(ok)
        : "r"(smem_u32(bar)), "r"(parity)
        : "memory");
    return ok != 0;
}

// Blocks until the phase with the given parity of `bar` has completed.  A watchdog turns a
// protocol bug into a trapped launch (cudaErrorLaunchFailure) instead of a hung GPU.
#ifndef SPECINFER_WATCHDOG_CYCLES
#define SPECINFER_WATCHDOG_CYCLES 40000000000ll
#endif
// A wait that never completes is a protocol bug: trap (the launch fails with an error instead of hanging
// the GPU).  Inline on purpose -- no printf: a called subroutine in a kernel that reallocates registers
// per warpgroup (setmaxnreg) makes ptxas compile the whole kernel under the smallest register budget.
__device__ __forceinline__ void mbar_hang_report(uint64_t *, uint32_t) { __trap(); }
__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t parity) {
    if (mbar_try_wait(bar, parity)) return;
    const long long t0 = clock64();
    while (!mbar_try_wait(bar, parity)) {
        if (clock64() - t0 > SPECINFER_WATCHDOG_CYCLES) mbar_hang_report(bar, parity);
    }
}

__device__ __forceinline__ void fence_proxy_async_smem() {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

__device__ __forceinline__ void named_bar_sync(uint32_t id, uint32_t nthreads) {
    asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(nthreads) : "memory");
}

// named barrier + OR-reduction of a predicate over the participating threads (one instruction)
__device__ __forceinline__ bool named_bar_red_or(uint32_t id, uint32_t nthreads, bool pred) {
    uint32_t r;
    asm volatile("{\n\t.reg .pred pi, po;\n\tsetp.ne.u32 pi, %3, 0;\n\t"
                 "bar.red.or.pred po, %1, %2, pi;\n\tselp.u32 %0, 1, 0, po;\n\t}"
                 : "=r"(r) : "r"(id), "r"(nthreads), "r"((uint32_t)pred) : "memory");
    return r != 0;
}

// producer side of a producer/consumer named barrier (does not wait)
__device__ __forceinline__ void named_bar_arrive(uint32_t id, uint32_t nthreads) {
    asm volatile("bar.arrive %0, %1;" ::"r"(id), "r"(nthreads) : "memory");
}

// ---- TMA ---------------------------------------------------------------------------------
__device__ __forceinline__ void tma_prefetch_desc(const CUtensorMap *map) {
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(map)) : "memory");
}

__device__ __forceinline__ uint64_t l2_evict_normal_policy() {
    uint64_t pol;
    asm volatile("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;" : "=l"(pol));
    return pol;
}

__device__ __forceinline__ uint64_t l2_evict_first_policy() {
    uint64_t pol;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
    return pol;
}

__device__ __forceinline__ void tma_load_2d(void *dst, const CUtensorMap *map, uint64_t *bar, int x,
                                            int y, uint64_t policy) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint"
        " [%0], [%1, {%3, %4}], [%2], %5;" ::"r"(smem_u32(dst)),
        "l"(reinterpret_cast<uint64_t>(map)), "r"(smem_u32(bar)), "r"(x), "r"(y), "l"(policy)
        : "memory");
}

__device__ __forceinline__ void tma_load_3d(void *dst, const CUtensorMap *map, uint64_t *bar, int x,
                                            int y, int z) {
    asm volatile(
        "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes"
        " [%0], [%1, {%3, %4, %5}], [%2];" ::"r"(smem_u32(dst)),
        "l"(reinterpret_cast<uint64_t>(map)), "r"(smem_u32(bar)), "r"(x), "r"(y), "r"(z)
        : "memory");
}

// bulk async copy global -> shared (no tensor map), completes `bytes` of transaction on `bar`
__device__ __forceinline__ void bulk_load_g2s(void *sdst, const void *gsrc, uint32_t bytes, uint64_t *bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     smem_u32(sdst)),
                 "l"(gsrc), "r"(bytes), "r"(smem_u32(bar))
                 : "memory");
}

// generic-proxy global writes (made visible by fences + an acquire) -> later async-proxy reads
__device__ __forceinline__ void fence_proxy_async_global() {
    asm volatile("fence.proxy.async.global;" ::: "memory");
}

// bulk async copy shared -> global (no tensor map), tracked by bulk groups of this thread
__device__ __forceinline__ void bulk_store_s2g(void *gdst, const void *ssrc, uint32_t bytes) {
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(gdst), "r"(smem_u32(ssrc)),
                 "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
// waits until all committed bulk copies of this thread have finished READING shared memory
__device__ __forceinline__ void bulk_wait_read_all() {
    asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
}
__device__ __forceinline__ void bulk_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }

// ---- programmatic dependent launch ---------------------------------------------------------
__device__ __forceinline__ void grid_dependency_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void grid_launch_dependents() {
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
}

// ---- tcgen05 / TMEM ------------------------------------------------------------------------
template <int kCols>
__device__ __forceinline__ void tmem_alloc(uint32_t *dst_smem) {  // whole warp
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                     smem_u32(dst_smem)),
                 "n"(kCols)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
}

template <int kCols>
__device__ __forceinline__ void tmem_dealloc(uint32_t taddr) {  // whole warp
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(taddr), "n"(kCols)
                 : "memory");
}

__device__ __forceinline__ void tc_fence_before() {
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
}
__device__ __forceinline__ void tc_fence_after() {
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
}

// D[tmem] (+)= A[smem desc] * B[smem desc], kind::f16 (bf16 inputs, fp32 accumulate).
__device__ __forceinline__ void umma_bf16_ss(uint32_t d_tmem, uint64_t adesc, uint64_t bdesc,
                                             uint32_t idesc, uint32_t accumulate) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "setp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(d_tmem),
        "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate)
        : "memory");
}

// Arrives (once) on `bar` when all previously issued tcgen05.mma of this thread complete.
__device__ __forceinline__ void umma_commit(uint64_t *bar) {
    asm volatile(
        "tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
            smem_u32(bar))
        : "memory");
}

__device__ __forceinline__ void tmem_ld16(uint32_t taddr, uint32_t (&r)[16]) {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, "
        "%11, %12, %13, %14, %15}, [%16];"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]),
          "=r"(r[7]), "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]),
          "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
        : "r"(taddr));
}

__device__ __forceinline__ void tmem_st16(uint32_t taddr, const uint32_t (&r)[16]) {
    asm volatile(
        "tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], {%1, %2, %3, %4, %5, %6, %7, %8, %9, %10, "
        "%11, %12, %13, %14, %15, %16};" ::"r"(taddr),
        "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(r[4]), "r"(r[5]), "r"(r[6]), "r"(r[7]),
        "r"(r[8]), "r"(r[9]), "r"(r[10]), "r"(r[11]), "r"(r[12]), "r"(r[13]), "r"(r[14]),
        "r"(r[15])
        : "memory");
}

__device__ __forceinline__ void tmem_ld_wait() {
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}
__device__ __forceinline__ void tmem_st_wait() {
    asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
}

// ---- UMMA descriptors (PTX ISA "tcgen05 matrix descriptors"; bit layout as in CUTLASS
// cute/arch/mma_sm100_desc.hpp) ------------------------------------------------------------
enum SwizzleMode : uint32_t { kSwNone = 0, kSw128 = 2, kSw64 = 4, kSw32 = 6 };

__device__ __forceinline__ uint64_t make_smem_desc(uint32_t saddr, uint32_t lbo_bytes,
                                                   uint32_t sbo_bytes, uint32_t swizzle) {
    uint64_t d = 0;
    d |= uint64_t((saddr >> 4) & 0x3FFF);
    d |= uint64_t((lbo_bytes >> 4) & 0x3FFF) << 16;
    d |= uint64_t((sbo_bytes >> 4) & 0x3FFF) << 32;
    d |= uint64_t(1) << 46;  // version (sm_100)
    d |= uint64_t(swizzle & 7) << 61;
    return d;
}

// Instruction descriptor for kind::f16 with bf16 A/B and fp32 D.
__host__ __device__ constexpr uint32_t make_idesc_bf16(int M, int N, bool a_mn_major,
                                                       bool b_mn_major) {
    return (1u << 4)                          // D format f32
           | (1u << 7)                        // A bf16
           | (1u << 10)                       // B bf16
           | (uint32_t(a_mn_major) << 15)     // A major
           | (uint32_t(b_mn_major) << 16)     // B major
           | (uint32_t(N >> 3) << 17)         // N / 8
           | (uint32_t(M >> 4) << 24);        // M / 16
}

// ---- misc ---------------------------------------------------------------------------------
// warpgroup register reallocation (all 128 threads of an aligned warpgroup execute it)
template <int N>
__device__ __forceinline__ void setmaxnreg_inc() {
    asm volatile("setmaxnreg.inc.sync.aligned.u32 %0;" ::"n"(N));
}
template <int N>
__device__ __forceinline__ void setmaxnreg_dec() {
    asm volatile("setmaxnreg.dec.sync.aligned.u32 %0;" ::"n"(N));
}

__device__ __forceinline__ float ex2(float x) {
    float y;
    asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
    return y;
}

// Blackwell paired fp32 arithmetic (FFMA2 / FADD2: two lanes of work per instruction); the softmax
// is issue-bound, so halving its FMA and FADD instruction count shortens the per-tile chain
__device__ __forceinline__ uint64_t f2_bits(float a, float b) {
    return (uint64_t)__float_as_uint(a) | ((uint64_t)__float_as_uint(b) << 32);
}
__device__ __forceinline__ uint64_t ffma2(uint64_t a, uint64_t b, uint64_t c) {
    uint64_t d;
    asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(d) : "l"(a), "l"(b), "l"(c));
    return d;
}
__device__ __forceinline__ uint64_t fmul2(uint64_t a, uint64_t b) {
    uint64_t d;
    asm("mul.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(a), "l"(b));
    return d;
}
__device__ __forceinline__ float f2_lo(uint64_t v) { return __uint_as_float((uint32_t)v); }
__device__ __forceinline__ float f2_hi(uint64_t v) { return __uint_as_float((uint32_t)(v >> 32)); }
__device__ __forceinline__ uint64_t fadd2(uint64_t a, uint64_t b) {
    uint64_t d;
    asm("add.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(a), "l"(b));
    return d;
}

__device__ __forceinline__ uint32_t pack_bf16x2(float lo, float hi) {
    __nv_bfloat162 v = __floats2bfloat162_rn(lo, hi);
    return *reinterpret_cast<uint32_t *>(&v);
}

// acc + float(bf16 half of w), one instruction (sm_100 mixed-precision add reads the half in place)
__device__ __forceinline__ float add_bf16lo(uint32_t w, float acc) {
    asm("{\n\t.reg .b16 lo, hi;\n\tmov.b32 {lo, hi}, %1;\n\tadd.rn.f32.bf16 %0, lo, %0;\n\t}" : "+f"(acc) : "r"(w));
    return acc;
}
__device__ __forceinline__ float add_bf16hi(uint32_t w, float acc) {
    asm("{\n\t.reg .b16 lo, hi;\n\tmov.b32 {lo, hi}, %1;\n\tadd.rn.f32.bf16 %0, hi, %0;\n\t}" : "+f"(acc) : "r"(w));
    return acc;
}

__device__ __forceinline__ float ldcg_f32(const float *p) { return __ldcg(p); }

}  // namespace specinfer
