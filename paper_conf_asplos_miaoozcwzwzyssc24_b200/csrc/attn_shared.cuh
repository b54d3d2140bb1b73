// attn_shared.cuh — pieces shared by the two tree-attention kernels (tree_attention.cu:
// swapped keys-as-M kernel for <= 64 query rows per kv-head; tree_attention_rows.cu: rows-as-M
// kernel for wider trees / GQA groups): launch parameters, schedule helpers, TMA helpers,
// tensor-map encoding, debug tracing.
#pragma once
#include <atomic>

#include "common.cuh"

namespace specinfer {

struct AttnParams {
    const int32_t *prefix_len;
    const int32_t *n_nodes;
    const int32_t *item_start;
    const int4 *item_info;
    const int4 *cta_info;
    uint32_t *item_cnt;
    const unsigned long long *rowmask;
    const uint32_t *anc;
    float *part_o;
    float *part_ml;
    __nv_bfloat16 *out;
    int B, Nmax, Hq, Hkv, G, Smax, chunks, npc, n_items, nk_slots, nv_slots;
    int splitk;  // > 1: split-KV mode (cluster of splitk CTAs per item, DSMEM merge)
    int early_prefix;  // SPECINFER_ATTN_EARLY_PREFIX: the producers read the schedule and stage the
                       // first committed-prefix tiles before the programmatic dependency resolves
    int lanes;  // CTAs per lock-step group (schedule_kernel); 1 = plain stream-K over items
    // rows kernel, many short items (dyn = 1): whole items claimed from an atomic ticket counter (reset by
    // tree_prepare) instead of the static stream-K ranges -- CTA c starts with item c, then claims
    uint32_t *dyn_ctr;
    int dyn;
    // paged KV (NEXT-4): page_table[b][t] = page holding keys [128 t, 128 t + 128) of request b;
    // a page is [Hkv][128][128] bf16.  nullptr = contiguous [B][Hkv][Smax][128] caches.
    const int32_t *page_table;
    int max_pages, n_pages;
    float scale_log2;
    unsigned long long *trace;  // optional per-tile timestamps (debug), nullptr in production
    int debug_flags;            // experiments only: 1 = skip K/V TMA, 2 = skip MMAs (results invalid)
};

// Debug hooks (pipeline timestamps, experiment switches) exist only in a library built with
// -DSPECINFER_DEBUG_HOOKS (build_lib.py --debug-hooks -> libspecinfer_debug.so, development tools);
// the production build compiles them out: no trace stores, every experiment branch constant-false.
#ifdef SPECINFER_DEBUG_HOOKS
#define SPI_FLAGS(p) ((p).debug_flags)
#define SPI_TRACING(p) ((p).trace != nullptr)
#else
#define SPI_FLAGS(p) 0
#define SPI_TRACING(p) false
#endif

// debug timestamps: trace[cta][tile][event], CTAs < kTraceCtas, tiles < kTraceTiles
constexpr int kTraceCtas = 8, kTraceTiles = 64, kTraceEv = 16;
__device__ __forceinline__ unsigned long long globaltimer_ns() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}
// kernel-level timestamps of every CTA (ns), 8 slots: 0 entry, 1 exit, 2 first K issue, 3 split-KV
// cluster barrier, 4 prologue done, 5 dependency wait passed, 6 schedule read, 7 first S ready
#define SPI_TRACE_K(slot)                                                                                  \
    do {                                                                                                   \
        if (SPI_TRACING(p))                                                                                \
            p.trace[(size_t)kTraceCtas * kTraceTiles * kTraceEv + blockIdx.x * 8 + (slot)] = globaltimer_ns(); \
    } while (0)
#define SPI_TRACE(ev)                                                                               \
    do {                                                                                            \
        if (SPI_TRACING(p) && blockIdx.x < kTraceCtas && lt < kTraceTiles)                          \
            p.trace[((size_t)blockIdx.x * kTraceTiles + lt) * kTraceEv + (ev)] = clock64();         \
    } while (0)

constexpr int kSlotBytes = kKeyTile * kHeadDim * 2;  // 32 KB: one K or V tile
constexpr int kHalfBytes = kSlotBytes / 2;            // 16 KB: 128 keys x 64 dims
// the last tile of a request is loaded row-exactly (boxes of 16, 4 and 1 rows) so that no cache
// slot at or beyond P_b + n_b is ever read; the rest of the slot keeps stale finite data
constexpr float kRescaleThreshold = 8.0f;              // log2 units: stale max tolerance
constexpr int kCombineBatch = 8;                       // split pieces merged per round
constexpr int kSegRing = 16;                           // segment descriptors in flight
constexpr int kMaxSlots = 8;


struct SegDesc {
    int x, begin, end, ib, ie, b, g, c, P, n;
};

// First cache row (in the 2D [rows][128] view the tensor maps use) of the 128-key tile of request b,
// kv-head g that starts at key0 (a multiple of 128): contiguous or through the page table.
__device__ __forceinline__ int kv_tile_row(const AttnParams &p, int b, int g, int key0) {
    if (p.page_table == nullptr) return (int)((long long)(b * p.Hkv + g) * p.Smax + key0);
    const int page = __ldg(p.page_table + (size_t)b * p.max_pages + (key0 / kKeyTile));
    return (page * p.Hkv + g) * kKeyTile;
}

// 64-bit unsigned division by shift-subtract, inline: the emulated `/` on 64-bit integers is a called
// subroutine, and a call site in a kernel that reallocates registers per warpgroup (setmaxnreg) makes
// ptxas compile the whole kernel under the smallest register budget.  Cold path only.
__device__ __forceinline__ unsigned long long udiv64_inline(unsigned long long n, unsigned long long d) {
    unsigned long long q = 0, r = 0;
#pragma unroll 1
    for (int i = 63; i >= 0; --i) {
        r = (r << 1) | ((n >> i) & 1ull);
        if (r >= d) {
            r -= d;
            q |= 1ull << i;
        }
    }
    return q;
}

__device__ __forceinline__ int cta_start(long long c, long long T, long long NC) {
    // 32-bit division when c * T fits (every practical schedule)
    if (c * T <= 0xFFFFFFFFll) return (int)((uint32_t)(c * T) / (uint32_t)NC);
    return (int)udiv64_inline((unsigned long long)(c * T), (unsigned long long)NC);
}

__device__ __forceinline__ int cta_of_tile(int t, int T, int NC) {
    // the largest c with cta_start(c) <= t: floor(c T / NC) <= t <=> c T < (t + 1) NC
    const long long num = (long long)(t + 1) * NC - 1;
    int c = num <= 0xFFFFFFFFll ? (int)((uint32_t)num / (uint32_t)T)
                                : (int)udiv64_inline((unsigned long long)num, (unsigned long long)T);
    return c < NC ? c : NC - 1;
}

// Cross-lane "transpose reduction": on entry each lane holds N values (one per row); on exit
// lane l holds in v[0] the reduction over the 32 lanes of row (l mod N) (N <= 32).
template <int N, bool kIsMax>
__device__ __forceinline__ void transpose_reduce(float *v) {
    const int lane = threadIdx.x & 31;
#pragma unroll
    for (int off = N / 2; off >= 1; off >>= 1) {
        const bool upper = (lane & off) != 0;
#pragma unroll
        for (int i = 0; i < off; ++i) {
            const float send = upper ? v[i] : v[i + off];
            const float keep = upper ? v[i + off] : v[i];
            const float got = __shfl_xor_sync(0xffffffffu, send, off);
            v[i] = kIsMax ? fmaxf(keep, got) : keep + got;
        }
    }
#pragma unroll
    for (int off = N; off < 32; off <<= 1) {
        const float got = __shfl_xor_sync(0xffffffffu, v[0], off);
        v[0] = kIsMax ? fmaxf(v[0], got) : v[0] + got;
    }
}

// Loads rows [row0, row0 + nv) of a K or V tile (nv < 128) with boxes of 16, 4 and 1 rows.
__device__ __forceinline__ void tma_load_rows(uint8_t *dst, uint64_t *bar, int nv, int row0, uint64_t pol,
                                              const CUtensorMap *m16, const CUtensorMap *m4,
                                              const CUtensorMap *m1) {
    mbar_arrive_expect_tx(bar, (uint32_t)nv * 256u);
    int r = 0;
    for (; r + 16 <= nv; r += 16) {
        tma_load_2d(dst + r * 128, m16, bar, 0, row0 + r, pol);
        tma_load_2d(dst + kHalfBytes + r * 128, m16, bar, 64, row0 + r, pol);
    }
    for (; r + 4 <= nv; r += 4) {
        tma_load_2d(dst + r * 128, m4, bar, 0, row0 + r, pol);
        tma_load_2d(dst + kHalfBytes + r * 128, m4, bar, 64, row0 + r, pol);
    }
    for (; r < nv; ++r) {
        tma_load_2d(dst + r * 128, m1, bar, 0, row0 + r, pol);
        tma_load_2d(dst + kHalfBytes + r * 128, m1, bar, 64, row0 + r, pol);
    }
}

// ------------------------------------------------------------------------------------------
// host side
// ------------------------------------------------------------------------------------------
typedef CUresult (*PFN_encodeTiled_t)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *,
                                      const cuuint64_t *, const cuuint64_t *, const cuuint32_t *,
                                      const cuuint32_t *, CUtensorMapInterleave, CUtensorMapSwizzle,
                                      CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

static PFN_encodeTiled_t get_encode_fn() {
    static PFN_encodeTiled_t fn = nullptr;
    if (!fn) {
        void *ptr = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &ptr, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = reinterpret_cast<PFN_encodeTiled_t>(ptr);
    }
    return fn;
}

// cudaFuncAttributeMaxDynamicSharedMemorySize is per device (context): one bit per attention kernel
// variant and device, set once (part of the per-device capability cache, include/specinfer.h).
// Racing first calls both set the attribute, which is idempotent.
inline cudaError_t ensure_max_smem_attr(const void *func, int variant, size_t max_smem) {
    static std::atomic<uint32_t> done[64];
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return e;
    const uint32_t bit = 1u << variant;
    if (dev >= 0 && dev < 64 && (done[dev].load(std::memory_order_acquire) & bit)) return cudaSuccess;
    e = cudaFuncSetAttribute(func, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)max_smem);
    if (e == cudaSuccess && dev >= 0 && dev < 64) done[dev].fetch_or(bit, std::memory_order_acq_rel);
    return e;
}

static bool encode_2d(CUtensorMap *m, const void *base, uint64_t rows, uint32_t box_rows) {
    PFN_encodeTiled_t enc = get_encode_fn();
    if (!enc) return false;
    const cuuint64_t dims[2] = {128, rows};
    const cuuint64_t strides[1] = {256};
    const cuuint32_t box[2] = {64, box_rows};
    const cuuint32_t estr[2] = {1, 1};
    return enc(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void *>(base), dims, strides, box, estr,
               CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
               CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

static bool encode_q(CUtensorMap *m, const void *base, int Hq, uint64_t nodes, int G, int npc) {
    PFN_encodeTiled_t enc = get_encode_fn();
    if (!enc) return false;
    const cuuint64_t dims[3] = {128, (cuuint64_t)Hq, nodes};
    const cuuint64_t strides[2] = {256, (cuuint64_t)Hq * 256};
    const cuuint32_t box[3] = {64, (cuuint32_t)G, (cuuint32_t)npc};
    const cuuint32_t estr[3] = {1, 1, 1};
    return enc(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 3, const_cast<void *>(base), dims, strides, box, estr,
               CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
               CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}


}  // namespace specinfer
