// tree_attention_rows.cu — K2 tree attention for wide trees / GQA groups (G * Nmax > 64 query rows
// per kv-head), sm_100a.  Same computation and schedule as tree_attention.cu (Def. 4.1
// L594-598, Eq. 1-4, topology-aware mask L645-674), different tiling:
//  * a work item is (request, kv-head, block of 128 query rows); the UMMA M dimension is the query
//    rows (one TMEM lane per row), N = 128 keys for S = Q K^T and N = 128 dims for O += P V, so the
//    MMAs run at full rate (N = 128) instead of the A-read-bound N <= 64 of the swapped kernel;
//  * every row's softmax is thread-local (128 S values per thread per tile): exact tile max, stale
//    running max with a 2^8 tolerance, O row rescaled in TMEM by its own thread when it moves;
//  * P goes to TMEM (bf16 packed, double-buffered) and feeds the PV MMA as the A operand ("TS"
//    form), so smem holds only Q (double-buffered) and the K / V rings;
//  * tree keys are masked with the ancestor-or-self bitset of the row's node (tree_prepare);
//  * the stream-K schedule, producers, segment ring, row-exact tail loads, split combine and PDL
//    are shared with the swapped kernel (attn_shared.cuh).
#include "attn_shared.cuh"

namespace specinfer {

namespace rows {

constexpr int RB = kRowsBlock;              // 128 query rows per item
constexpr int kQBuf = 2 * RB * 128;          // one Q buffer: 2 halves x 128 rows x 128 B
constexpr int kTmemCols = 512;               // S0 S1 | O | P0 P1
constexpr int kColS = 0, kColO = 256, kColP = 384;

struct Misc {
    uint64_t k_full[kMaxSlots], k_empty[kMaxSlots];
    uint64_t v_full[kMaxSlots], v_empty[kMaxSlots];
    uint64_t q_full[2], q_empty[2];
    uint64_t s_full[2], s_empty[2];
    uint64_t p_full[2], p_empty[2];
    uint64_t seg_full[kSegRing];
    SegDesc seg[kSegRing];
    uint32_t tmem_base;
    int32_t bcast;
    float pmax[2][2][RB];  // [tile parity][key half][row] partial tile maxima
    float psum[2][RB];     // [key half][row] partial row sums at a segment's end
};

__device__ __forceinline__ void tmem_ld32(uint32_t taddr, uint32_t (&r)[32]) {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, "
        "%14, %15, %16, %17, %18, %19, %20, %21, %22, %23, %24, %25, %26, %27, %28, %29, %30, %31}, [%32];"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
          "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]),
          "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]),
          "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
        : "r"(taddr));
}

// D[tmem] (+)= A[tmem] * B[smem desc], kind::f16 (A = P, bf16 packed two per column)
__device__ __forceinline__ void umma_bf16_ts(uint32_t d_tmem, uint32_t a_tmem, uint64_t bdesc, uint32_t idesc,
                                             uint32_t accumulate) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "setp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n\t}" ::"r"(d_tmem),
        "r"(a_tmem), "l"(bdesc), "r"(idesc), "r"(accumulate)
        : "memory");
}

}  // namespace rows

__global__ void __launch_bounds__(352, 1)
    tree_attn_rows_kernel(const __grid_constant__ CUtensorMap tm_q, const __grid_constant__ CUtensorMap tm_k,
                          const __grid_constant__ CUtensorMap tm_v, const __grid_constant__ CUtensorMap tm_k16,
                          const __grid_constant__ CUtensorMap tm_v16, const __grid_constant__ CUtensorMap tm_k4,
                          const __grid_constant__ CUtensorMap tm_v4, const __grid_constant__ CUtensorMap tm_k1,
                          const __grid_constant__ CUtensorMap tm_v1, const AttnParams p) {
    using namespace rows;
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    uint8_t *smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
    const int NK = p.nk_slots, NV = p.nv_slots;
    uint8_t *s_k = smem;
    uint8_t *s_v = s_k + (size_t)NK * kSlotBytes;
    uint8_t *s_q = s_v + (size_t)NV * kSlotBytes;
    Misc *misc = reinterpret_cast<Misc *>(s_q + 2 * kQBuf);

    const int warp = threadIdx.x >> 5;
    const int lane = threadIdx.x & 31;
    const int NC = gridDim.x;
    if (threadIdx.x == 0) SPI_TRACE_K(0);

    if (threadIdx.x == 0) {
        for (int i = 0; i < NK; ++i) {
            mbar_init(&misc->k_full[i], 1);
            mbar_init(&misc->k_empty[i], 1);
        }
        for (int i = 0; i < NV; ++i) {
            mbar_init(&misc->v_full[i], 1);
            mbar_init(&misc->v_empty[i], 1);
        }
        for (int i = 0; i < 2; ++i) {
            mbar_init(&misc->q_full[i], 1);
            mbar_init(&misc->q_empty[i], 1);
            mbar_init(&misc->s_full[i], 1);
            mbar_init(&misc->s_empty[i], 8);
            mbar_init(&misc->p_full[i], 8);
            mbar_init(&misc->p_empty[i], 1);
        }
        for (int i = 0; i < kSegRing; ++i) mbar_init(&misc->seg_full[i], 1);
        fence_barrier_init();
    }
    if (warp == 0 && lane == 0) {
        tma_prefetch_desc(&tm_q);
        tma_prefetch_desc(&tm_k);
        tma_prefetch_desc(&tm_v);
    }
    if (warp >= 3) {
        // Q rows beyond an item's G*npc rows are never written by TMA: keep them zero
        for (int i = threadIdx.x - 96; i < 2 * kQBuf / 16; i += 256)
            reinterpret_cast<uint4 *>(s_q)[i] = make_uint4(0, 0, 0, 0);
        // V rows past a request's last key are never loaded: they must hold finite data (0 * NaN)
        for (int i = threadIdx.x - 96; i < NV * kSlotBytes / 16; i += 256)
            reinterpret_cast<uint4 *>(s_v)[i] = make_uint4(0, 0, 0, 0);
        fence_proxy_async_smem();
    }
    if (warp == 1) tmem_alloc<kTmemCols>(&misc->tmem_base);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem = misc->tmem_base;

    grid_dependency_wait();
    const int4 ci = __ldg(p.cta_info + 2 * blockIdx.x);
    const int4 first_info = __ldg(p.cta_info + 2 * blockIdx.x + 1);
    const int t0 = ci.x, t1 = ci.y, x_first = ci.z, T = ci.w;
    const int ntiles = t1 - t0;

    if (ntiles <= 0) {
        // no work for this CTA
    } else if (warp == 0) {
        // ============================ TMA producers ============================
        const uint64_t pol = l2_evict_first_policy();
        if (lane == 0) {
            int lt = 0, ls = 0;
            int4 next_info = first_info;
            for (int x = x_first; lt < ntiles; ++x) {
                const int4 info = next_info;
                next_info = __ldg(p.item_info + x + 1);
                const int begin = max(t0, info.x), end = min(t1, info.y);
                if (end <= begin) continue;
                SegDesc d;
                d.x = x;
                d.begin = begin;
                d.end = end;
                d.ib = info.x;
                d.ie = info.y;
                d.c = x % p.chunks;
                d.g = (x / p.chunks) % p.Hkv;
                d.b = x / (p.chunks * p.Hkv);
                d.P = info.z;
                d.n = info.w;
                misc->seg[ls % kSegRing] = d;
                mbar_arrive(&misc->seg_full[ls % kSegRing]);
                const int Kend = d.P + d.n;
                const int qb = ls & 1;
                if (ls >= 2) mbar_wait(&misc->q_empty[qb], ((ls >> 1) - 1) & 1);
                mbar_arrive_expect_tx(&misc->q_full[qb], 2u * (uint32_t)(p.G * p.npc) * 128u);
                uint8_t *qdst = s_q + qb * kQBuf;
                const int node0 = d.b * p.Nmax + d.c * p.npc;
                tma_load_3d(qdst, &tm_q, &misc->q_full[qb], 0, d.g * p.G, node0);
                tma_load_3d(qdst + RB * 128, &tm_q, &misc->q_full[qb], 64, d.g * p.G, node0);
                const long long rowbase = (long long)(d.b * p.Hkv + d.g) * p.Smax;
                for (int t = d.begin; t < d.end; ++t, ++lt) {
                    const int key0 = (t - d.ib) * kKeyTile;
                    const int nv = min(kKeyTile, Kend - key0);
                    const int row0 = (int)(rowbase + key0);
                    const int slot = lt % NK, f = lt / NK;
                    if (f >= 1) mbar_wait(&misc->k_empty[slot], (f - 1) & 1);
                    SPI_TRACE(0);
                    if (lt == 0) SPI_TRACE_K(2);
                    uint8_t *dst = s_k + (size_t)slot * kSlotBytes;
                    uint64_t *bar = &misc->k_full[slot];
                    if (nv == kKeyTile) {
                        mbar_arrive_expect_tx(bar, kSlotBytes);
                        tma_load_2d(dst, &tm_k, bar, 0, row0, pol);
                        tma_load_2d(dst + kHalfBytes, &tm_k, bar, 64, row0, pol);
                    } else {
                        tma_load_rows(dst, bar, nv, row0, pol, &tm_k16, &tm_k4, &tm_k1);
                    }
                }
                ++ls;
            }
            grid_launch_dependents();
        } else if (lane == 1) {
            int lt = 0, ls = 0;
            while (lt < ntiles) {
                mbar_wait(&misc->seg_full[ls % kSegRing], (ls / kSegRing) & 1);
                const SegDesc d = misc->seg[ls % kSegRing];
                const int Kend = d.P + d.n;
                const long long rowbase = (long long)(d.b * p.Hkv + d.g) * p.Smax;
                for (int t = d.begin; t < d.end; ++t, ++lt) {
                    const int key0 = (t - d.ib) * kKeyTile;
                    const int nv = min(kKeyTile, Kend - key0);
                    const int row0 = (int)(rowbase + key0);
                    const int slot = lt % NV, f = lt / NV;
                    if (f >= 1) mbar_wait(&misc->v_empty[slot], (f - 1) & 1);
                    SPI_TRACE(1);
                    uint8_t *dst = s_v + (size_t)slot * kSlotBytes;
                    uint64_t *bar = &misc->v_full[slot];
                    if (nv == kKeyTile) {
                        mbar_arrive_expect_tx(bar, kSlotBytes);
                        tma_load_2d(dst, &tm_v, bar, 0, row0, pol);
                        tma_load_2d(dst + kHalfBytes, &tm_v, bar, 64, row0, pol);
                    } else {
                        tma_load_rows(dst, bar, nv, row0, pol, &tm_v16, &tm_v4, &tm_v1);
                    }
                }
                ++ls;
            }
        }
    } else if (warp == 1) {
        // ===================== S issuer: S = Q K^T (M = 128 rows, N = 128 keys) =====================
        if (lane == 0) {
            const uint32_t idesc_s = make_idesc_bf16(128, 128, false, false);
            const uint32_t k_addr = smem_u32(s_k), q_addr = smem_u32(s_q);
            int lt = 0, ls = 0;
            while (lt < ntiles) {
                mbar_wait(&misc->seg_full[ls % kSegRing], (ls / kSegRing) & 1);
                const SegDesc d = misc->seg[ls % kSegRing];
                const int qb = ls & 1;
                mbar_wait(&misc->q_full[qb], (ls >> 1) & 1);
                for (int t = d.begin; t < d.end; ++t, ++lt) {
                    const int slot = lt % NK;
                    mbar_wait(&misc->k_full[slot], (lt / NK) & 1);
                    const int sb = lt & 1;
                    if (lt >= 2) mbar_wait(&misc->s_empty[sb], ((lt - 2) >> 1) & 1);
                    tc_fence_after();
                    SPI_TRACE(2);
                    const uint32_t kbase = k_addr + slot * kSlotBytes;
                    const uint32_t qbase = q_addr + qb * kQBuf;
#pragma unroll
                    for (int kk = 0; kk < kHeadDim / 16; ++kk) {
                        const uint32_t off = (kk >> 2) * (RB * 128) + (kk & 3) * 32;
                        const uint64_t adesc = make_smem_desc(qbase + off, 16, 1024, kSw128);
                        const uint64_t bdesc = make_smem_desc(kbase + (kk >> 2) * kHalfBytes + (kk & 3) * 32, 16,
                                                              1024, kSw128);
                        umma_bf16_ss(tmem + kColS + sb * 128, adesc, bdesc, idesc_s, kk > 0 ? 1u : 0u);
                    }
                    umma_commit(&misc->s_full[sb]);
                    umma_commit(&misc->k_empty[slot]);
                    if (t == d.end - 1) umma_commit(&misc->q_empty[qb]);
                }
                ++ls;
            }
        }
    } else if (warp == 2) {
        // ===================== PV issuer: O += P V (A = P in TMEM, N = 128 dims) =====================
        if (lane == 0) {
            const uint32_t idesc_o = make_idesc_bf16(128, 128, false, true);
            const uint32_t v_addr = smem_u32(s_v);
            int lt = 0, ls = 0;
            while (lt < ntiles) {
                mbar_wait(&misc->seg_full[ls % kSegRing], (ls / kSegRing) & 1);
                const SegDesc d = misc->seg[ls % kSegRing];
                for (int t = d.begin; t < d.end; ++t, ++lt) {
                    const int pb = lt & 1;
                    mbar_wait(&misc->p_full[pb], (lt >> 1) & 1);
                    const int slot = lt % NV;
                    mbar_wait(&misc->v_full[slot], (lt / NV) & 1);
                    tc_fence_after();
                    SPI_TRACE(3);
                    const uint32_t vbase = v_addr + slot * kSlotBytes;
                    const bool first = (t == d.begin);
#pragma unroll
                    for (int kk = 0; kk < kKeyTile / 16; ++kk) {
                        const uint64_t bdesc = make_smem_desc(vbase + kk * 16 * 128, kHalfBytes, 1024, kSw128);
                        umma_bf16_ts(tmem + kColO, tmem + kColP + pb * 64 + kk * 8, bdesc, idesc_o,
                                     (first && kk == 0) ? 0u : 1u);
                    }
                    umma_commit(&misc->p_empty[pb]);
                    umma_commit(&misc->v_empty[slot]);
                }
                ++ls;
            }
        }
    } else {
        // ============ softmax / epilogue: 8 warps, two per TMEM lane quarter ============
        // warp pair (w, w+4) owns the 32 query rows of lane quarter qd; half hf of the pair owns
        // keys [64 hf, 64 hf + 64) of every tile and dims [64 hf, 64 hf + 64) of O.  The tile
        // row max is exchanged within the pair through smem (one 64-thread barrier per tile).
        const int sw = warp - 3;               // 0..7
        const int hf = sw >> 2;                // key / dim half
        const int qd = warp & 3;               // TMEM lane quarter
        const int r = qd * 32 + lane;          // query row of the item = TMEM lane
        const uint32_t lane_off = (uint32_t)(qd * 32) << 16;
        const uint32_t pair_bar = 2 + qd;      // named barrier of the warp pair (64 threads)
        int lt = 0, ls = 0;
        while (lt < ntiles) {
            mbar_wait(&misc->seg_full[ls % kSegRing], (ls / kSegRing) & 1);
            const SegDesc sd = misc->seg[ls % kSegRing];
            const int b = sd.b, g = sd.g, c = sd.c, P = sd.P, n = sd.n;
            const int Kend = P + n;
            const int G = p.G;
            const int rc = G * p.npc;
            const int node = c * p.npc + r / G, hl = r % G;
            const bool row_valid = (r < rc) && (node < n);
            // ancestor-or-self bitset of this row's node (rows without a node use node 0's root
            // path, which keeps them finite; they are never written)
            uint32_t anc[kBitWords];
            {
                const uint4 *ap = reinterpret_cast<const uint4 *>(
                    p.anc + ((size_t)b * p.Nmax + (row_valid ? node : 0)) * kBitWords);
                const uint4 a0 = __ldg(ap), a1 = __ldg(ap + 1);
                anc[0] = a0.x; anc[1] = a0.y; anc[2] = a0.z; anc[3] = a0.w;
                anc[4] = a1.x; anc[5] = a1.y; anc[6] = a1.z; anc[7] = a1.w;
            }
            float m = -INFINITY, l = 0.f;  // running row max (log2 units, shared by the pair), partial sum
            for (int t = sd.begin; t < sd.end; ++t, ++lt) {
                const int key0 = (t - sd.ib) * kKeyTile + hf * 64;  // first key of this half
                const int sb = lt & 1;
                mbar_wait(&misc->s_full[sb], (lt >> 1) & 1);
                tc_fence_after();
                if (r == 0 && hf == 0) SPI_TRACE(4);
                float x[64];
                {
                    uint32_t v[2][32];
                    tmem_ld32(tmem + kColS + sb * 128 + hf * 64 + lane_off, v[0]);
                    tmem_ld32(tmem + kColS + sb * 128 + hf * 64 + 32 + lane_off, v[1]);
                    tmem_ld_wait();
#pragma unroll
                    for (int i = 0; i < 32; ++i) {
                        x[i] = __uint_as_float(v[0][i]);
                        x[32 + i] = __uint_as_float(v[1][i]);
                    }
                }
                tc_fence_before();
                __syncwarp();
                if (lane == 0) mbar_arrive(&misc->s_empty[sb]);
                // mask: committed keys visible; tree keys by the ancestor bitset; past the end: none
                if (key0 + 64 > P) {
                    uint32_t vis[2];
#pragma unroll
                    for (int q = 0; q < 2; ++q) {
                        const int j0 = key0 + 32 * q - P;  // tree index of the group's first key
                        uint32_t w;
                        if (j0 + 32 <= 0) {
                            w = 0xFFFFFFFFu;
                        } else {
                            const int jb = max(j0, 0);
                            const int wi = jb >> 5, sh = jb & 31;
                            uint32_t lo = 0, hi = 0;
#pragma unroll
                            for (int k = 0; k < kBitWords; ++k) {
                                lo = (wi == k) ? anc[k] : lo;
                                hi = (wi + 1 == k) ? anc[k] : hi;
                            }
                            uint32_t bits = sh ? ((lo >> sh) | (hi << (32 - sh))) : lo;
                            if (j0 < 0) bits = (bits << (-j0)) | ((1u << (-j0)) - 1u);
                            const int nvalid = Kend - (key0 + 32 * q);
                            if (nvalid < 32) bits &= nvalid <= 0 ? 0u : ((1u << nvalid) - 1u);
                            w = bits;
                        }
                        vis[q] = w;
                    }
#pragma unroll
                    for (int i = 0; i < 64; ++i)
                        if (!((vis[i >> 5] >> (i & 31)) & 1u)) x[i] = -INFINITY;
                }
                float tm4[4] = {x[0], x[1], x[2], x[3]};
#pragma unroll
                for (int i = 4; i < 64; ++i) tm4[i & 3] = fmaxf(tm4[i & 3], x[i]);
                const float tmh = fmaxf(fmaxf(tm4[0], tm4[1]), fmaxf(tm4[2], tm4[3]));
                misc->pmax[sb][hf][r] = tmh;
                named_bar_sync(pair_bar, 64);
                const float tm = fmaxf(tmh, misc->pmax[sb][hf ^ 1][r]) * p.scale_log2;
                // stale running max: move it only when this tile exceeds it by more than 2^8
                float alpha = 1.f;
                if (tm > m + kRescaleThreshold) {
                    alpha = (m == -INFINITY) ? 0.f : ex2(m - tm);
                    m = tm;
                    l *= alpha;
                }
                if (__any_sync(0xffffffffu, alpha != 1.f) && t != sd.begin) {
                    // rescale this warp's half of the O rows: PV of the previous tile must be done
                    mbar_wait(&misc->p_empty[(lt - 1) & 1], ((lt - 1) >> 1) & 1);
                    tc_fence_after();
#pragma unroll
                    for (int q2 = 0; q2 < 2; ++q2) {
                        uint32_t v[32];
                        tmem_ld32(tmem + kColO + hf * 64 + q2 * 32 + lane_off, v);
                        tmem_ld_wait();
                        uint32_t w16[16];
#pragma unroll
                        for (int h = 0; h < 2; ++h) {
#pragma unroll
                            for (int i = 0; i < 16; ++i) w16[i] = __float_as_uint(__uint_as_float(v[h * 16 + i]) * alpha);
                            tmem_st16(tmem + kColO + hf * 64 + q2 * 32 + h * 16 + lane_off, w16);
                        }
                    }
                    tmem_st_wait();
                }
                const float mref = (m == -INFINITY) ? 0.f : m;
                // P of this half tile (bf16, two per TMEM column) into P[lt & 1]
                if (lt >= 2) mbar_wait(&misc->p_empty[sb], ((lt - 2) >> 1) & 1);
                tc_fence_after();
                float l4[4] = {0.f, 0.f, 0.f, 0.f};
#pragma unroll
                for (int c16 = 0; c16 < 2; ++c16) {
                    uint32_t w16[16];
#pragma unroll
                    for (int i = 0; i < 16; ++i) {
                        const uint32_t pk = pack_bf16x2(ex2(fmaf(x[c16 * 32 + 2 * i], p.scale_log2, -mref)),
                                                        ex2(fmaf(x[c16 * 32 + 2 * i + 1], p.scale_log2, -mref)));
                        w16[i] = pk;
                        l4[i & 3] += __uint_as_float(pk << 16) + __uint_as_float(pk & 0xFFFF0000u);
                    }
                    tmem_st16(tmem + kColP + sb * 64 + hf * 32 + c16 * 16 + lane_off, w16);
                }
                l += (l4[0] + l4[1]) + (l4[2] + l4[3]);
                tmem_st_wait();
                tc_fence_before();
                __syncwarp();
                if (lane == 0) mbar_arrive(&misc->p_full[sb]);
                if (r == 0 && hf == 0) SPI_TRACE(5);

                if (t == sd.end - 1) {
                    // ============ epilogue of this segment (per row, per dim half) ============
                    misc->psum[hf][r] = l;
                    mbar_wait(&misc->p_empty[sb], (lt >> 1) & 1);  // last PV done
                    tc_fence_after();
                    named_bar_sync(pair_bar, 64);
                    const float lrow = l + misc->psum[hf ^ 1][r];
                    if (r == 0 && hf == 0) SPI_TRACE(6);
                    const bool full = (sd.begin == sd.ib) && (sd.end == sd.ie);
                    if (full) {
                        const float inv = 1.0f / lrow;
                        __nv_bfloat16 *orow = p.out + (((size_t)b * p.Nmax + node) * p.Hq + g * G + hl) * kHeadDim + hf * 64;
#pragma unroll
                        for (int q2 = 0; q2 < 2; ++q2) {
                            uint32_t v[32];
                            tmem_ld32(tmem + kColO + hf * 64 + q2 * 32 + lane_off, v);
                            tmem_ld_wait();
                            if (row_valid) {
#pragma unroll
                                for (int i = 0; i < 32; i += 8) {
                                    uint4 o4;
                                    o4.x = pack_bf16x2(__uint_as_float(v[i]) * inv, __uint_as_float(v[i + 1]) * inv);
                                    o4.y = pack_bf16x2(__uint_as_float(v[i + 2]) * inv, __uint_as_float(v[i + 3]) * inv);
                                    o4.z = pack_bf16x2(__uint_as_float(v[i + 4]) * inv, __uint_as_float(v[i + 5]) * inv);
                                    o4.w = pack_bf16x2(__uint_as_float(v[i + 6]) * inv, __uint_as_float(v[i + 7]) * inv);
                                    *reinterpret_cast<uint4 *>(orow + q2 * 32 + i) = o4;
                                }
                            }
                        }
                    } else {
                        const int slot = (sd.begin == t0) ? 0 : 1;
                        float *po = p.part_o + (((size_t)blockIdx.x * 2 + slot) * RB + r) * kHeadDim + hf * 64;
#pragma unroll
                        for (int q2 = 0; q2 < 2; ++q2) {
                            uint32_t v[32];
                            tmem_ld32(tmem + kColO + hf * 64 + q2 * 32 + lane_off, v);
                            tmem_ld_wait();
#pragma unroll
                            for (int i = 0; i < 32; i += 4)
                                *reinterpret_cast<float4 *>(po + q2 * 32 + i) =
                                    make_float4(__uint_as_float(v[i]), __uint_as_float(v[i + 1]),
                                                __uint_as_float(v[i + 2]), __uint_as_float(v[i + 3]));
                        }
                        float *pml = p.part_ml + ((size_t)blockIdx.x * 2 + slot) * 2 * RB;
                        if (hf == 0) {
                            pml[r] = m;
                            pml[RB + r] = lrow;
                        }
                        __threadfence();
                        named_bar_sync(1, 256);
                        if (r == 0 && hf == 0) {
                            const int c_first = cta_of_tile(sd.ib, T, NC);
                            const int c_last = cta_of_tile(sd.ie - 1, T, NC);
                            int npieces = 0;
                            for (int cc = c_first; cc <= c_last; ++cc)
                                npieces += cta_start(cc + 1, T, NC) > cta_start(cc, T, NC);
                            const unsigned old = atomicAdd(&p.item_cnt[sd.x], 1u);
                            misc->bcast = (old == (unsigned)(npieces - 1)) ? 1 : 0;
                            if (misc->bcast) p.item_cnt[sd.x] = 0u;  // ready for the next launch
                        }
                        named_bar_sync(1, 256);
                        if (misc->bcast) {
                            // last piece: merge every piece's (m, l, O row half) by log-sum-exp
                            __threadfence();
                            const int c_first = cta_of_tile(sd.ib, T, NC);
                            const int c_last = cta_of_tile(sd.ie - 1, T, NC);
                            float M = -INFINITY;
                            for (int cc = c_first; cc <= c_last; ++cc) {
                                const int s0 = cta_start(cc, T, NC);
                                if (cta_start(cc + 1, T, NC) <= s0) continue;
                                const size_t po2 = (size_t)cc * 2 + ((s0 >= sd.ib) ? 0 : 1);
                                M = fmaxf(M, ldcg_f32(p.part_ml + po2 * 2 * RB + r));
                            }
                            float L = 0.f;
                            for (int cc = c_first; cc <= c_last; ++cc) {
                                const int s0 = cta_start(cc, T, NC);
                                if (cta_start(cc + 1, T, NC) <= s0) continue;
                                const size_t po2 = (size_t)cc * 2 + ((s0 >= sd.ib) ? 0 : 1);
                                const float mp = ldcg_f32(p.part_ml + po2 * 2 * RB + r);
                                if (mp != -INFINITY) L += ex2(mp - M) * ldcg_f32(p.part_ml + po2 * 2 * RB + RB + r);
                            }
                            const float inv = 1.0f / L;
                            __nv_bfloat16 *orow = p.out + (((size_t)b * p.Nmax + node) * p.Hq + g * G + hl) * kHeadDim + hf * 64;
                            for (int q2 = 0; q2 < 2; ++q2) {
                                float acc[32];
#pragma unroll
                                for (int i = 0; i < 32; ++i) acc[i] = 0.f;
                                for (int cc = c_first; cc <= c_last; ++cc) {
                                    const int s0 = cta_start(cc, T, NC);
                                    if (cta_start(cc + 1, T, NC) <= s0) continue;
                                    const size_t po2 = (size_t)cc * 2 + ((s0 >= sd.ib) ? 0 : 1);
                                    const float mp = ldcg_f32(p.part_ml + po2 * 2 * RB + r);
                                    if (mp == -INFINITY) continue;
                                    const float w = ex2(mp - M) * inv;
                                    const float4 *src = reinterpret_cast<const float4 *>(
                                        p.part_o + (po2 * RB + r) * kHeadDim + hf * 64 + q2 * 32);
#pragma unroll
                                    for (int i = 0; i < 8; ++i) {
                                        const float4 o4 = __ldcg(src + i);
                                        acc[4 * i] += w * o4.x;
                                        acc[4 * i + 1] += w * o4.y;
                                        acc[4 * i + 2] += w * o4.z;
                                        acc[4 * i + 3] += w * o4.w;
                                    }
                                }
                                if (row_valid) {
#pragma unroll
                                    for (int i = 0; i < 32; i += 8) {
                                        uint4 o4;
                                        o4.x = pack_bf16x2(acc[i], acc[i + 1]);
                                        o4.y = pack_bf16x2(acc[i + 2], acc[i + 3]);
                                        o4.z = pack_bf16x2(acc[i + 4], acc[i + 5]);
                                        o4.w = pack_bf16x2(acc[i + 6], acc[i + 7]);
                                        *reinterpret_cast<uint4 *>(orow + q2 * 32 + i) = o4;
                                    }
                                }
                            }
                        }
                    }
                    tc_fence_before();
                    named_bar_sync(pair_bar, 64);  // psum of this segment read by both halves
                    if (r == 0 && hf == 0) SPI_TRACE(7);
                }
            }
            ++ls;
        }
    }

    tc_fence_before();
    __syncthreads();
    if (warp == 1) {
        tc_fence_after();
        tmem_dealloc<kTmemCols>(tmem);
    }
    if (threadIdx.x == 0) SPI_TRACE_K(1);
}

static size_t rows_smem_bytes(int num_slots) {
    return 1024 + (size_t)num_slots * kSlotBytes + 2 * rows::kQBuf + sizeof(rows::Misc);
}

cudaError_t launch_tree_attention_rows(const AttnParams &prm0, const void *q, const void *k, const void *v,
                                       int num_ctas, size_t max_smem, cudaStream_t stream) {
    AttnParams prm = prm0;
    CUtensorMap tq, tk, tv, tk16, tv16, tk4, tv4, tk1, tv1;
    const uint64_t rows = (uint64_t)prm.B * prm.Hkv * prm.Smax;
    if (!encode_q(&tq, q, prm.Hq, (uint64_t)prm.B * prm.Nmax, prm.G, prm.npc) ||
        !encode_2d(&tk, k, rows, kKeyTile) || !encode_2d(&tv, v, rows, kKeyTile) ||
        !encode_2d(&tk16, k, rows, 16) || !encode_2d(&tv16, v, rows, 16) || !encode_2d(&tk4, k, rows, 4) ||
        !encode_2d(&tv4, v, rows, 4) || !encode_2d(&tk1, k, rows, 1) || !encode_2d(&tv1, v, rows, 1))
        return cudaErrorInvalidValue;
    int ns = 2 * kMaxSlots;
    while (ns > 2 && rows_smem_bytes(ns) > max_smem) --ns;
    ns = min(ns, 6);
    prm.nk_slots = ns / 2;
    prm.nv_slots = ns - ns / 2;
    const size_t smem = rows_smem_bytes(ns);
    static bool attr_set = false;
    if (!attr_set) {
        cudaError_t e = cudaFuncSetAttribute(tree_attn_rows_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                             (int)max_smem);
        if (e != cudaSuccess) return e;
        attr_set = true;
    }
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(num_ctas);
    cfg.blockDim = dim3(352);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = stream;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, tree_attn_rows_kernel, tq, tk, tv, tk16, tv16, tk4, tv4, tk1, tv1, prm);
}

}  // namespace specinfer
