// tree_attention_rows.cu — K2 tree attention for wide trees / GQA groups (G * Nmax > 64 query rows
// per kv-head), sm_100a.  Same computation and schedule as tree_attention.cu (Def. 4.1
// L594-598, Eq. 1-4, topology-aware mask L645-674), different tiling:
//  * a work item is (request, kv-head, block of 128 query rows); the UMMA M dimension is the query
//    rows (one TMEM lane per row), N = 128 keys for S = Q K^T and N = 128 dims for O += P V, so the
//    MMAs run at full rate (N = 128) instead of the A-read-bound N <= 64 of the swapped kernel;
//  * two softmax groups of 4 warps own alternate KV tiles (tile parity), each with its own S
//    buffer, O accumulator and running (m, l) per row, merged by log-sum-exp at the segment end:
//    the groups run out of phase, so one group's TMEM / barrier latency hides behind the other's
//    exponentials; every row's softmax is thread-local (exact tile max, stale running max with a
//    2^8 tolerance, O row rescaled in TMEM by its own thread when it moves);
//  * P (bf16 pairs) is written over the first 64 columns of its own S buffer and feeds the PV
//    MMA as the A operand ("TS" form): TMEM = S0 S1 O0 O1, smem holds only Q and the K / V rings;
//  * lane mode (schedule_kernel): the row blocks of one (request, kv-head) run on `lanes` CTAs in
//    lock-step over the same tile range, so each KV tile is read from HBM once;
//  * tree keys are masked with the ancestor-or-self bitset of the row's node (tree_prepare);
//  * the stream-K schedule, producers, segment ring, row-exact tail loads, split combine and PDL
//    are shared with the swapped kernel (attn_shared.cuh).
#include "attn_shared.cuh"

namespace specinfer {

namespace rows {

constexpr int RB = kRowsBlock;              // 128 query rows per item
constexpr int kQBuf = 2 * RB * 128;          // one Q buffer: 2 halves x 128 rows x 128 B
constexpr int kTmemCols = 512;               // S0 S1 (P aliased over S) | O0 O1
constexpr int kColS = 0, kColO = 256;

constexpr int kMaxRing = 6;                  // unified K/V tile ring (slots of 32 KB)

struct Misc {
    uint64_t full[kMaxRing], empty[kMaxRing];
    uint64_t q_full[2], q_empty[2];
    uint64_t s_full[2];
    uint64_t p_full[2], p_empty[2];
    uint64_t seg_full[kSegRing];
    SegDesc seg[kSegRing];
    uint32_t tmem_base;
    int32_t bcast;
    float2 xch[RB];        // [row] (m, l) exchange between the two softmax groups at a segment's end
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

// Row max of one 128-key S tile (this thread's TMEM lane), optionally under the visibility mask.
template <bool kMask>
__device__ __forceinline__ void tile_max(uint32_t s_col, const uint32_t (&vis)[4], float (&tm4)[4]) {
#pragma unroll
    for (int h = 0; h < 2; ++h) {
        uint32_t v[2][32];
        tmem_ld32(s_col + h * 64, v[0]);
        tmem_ld32(s_col + h * 64 + 32, v[1]);
        tmem_ld_wait();
#pragma unroll
        for (int q = 0; q < 2; ++q) {
#pragma unroll
            for (int i = 0; i < 32; ++i) {
                float x = __uint_as_float(v[q][i]);
                if (kMask) x = ((vis[2 * h + q] >> i) & 1u) ? x : -INFINITY;
                tm4[i & 3] = fmaxf(tm4[i & 3], x);
            }
        }
    }
}

// P = 2^(s * scale_log2 - mref) of one S tile, packed to bf16 pairs over the first 64 columns of the
// same TMEM buffer; accumulates the fp32 row sum.
template <bool kMask>
__device__ __forceinline__ void tile_exp(uint32_t s_col, const uint32_t (&vis)[4], float scale_log2, float mref,
                                         float (&l4)[4]) {
    const uint64_t sc2 = f2_bits(scale_log2, scale_log2), nm2 = f2_bits(-mref, -mref);
    uint64_t la = f2_bits(0.f, 0.f), lb = f2_bits(0.f, 0.f);  // paired row-sum accumulators
#pragma unroll
    for (int h = 0; h < 2; ++h) {
        uint32_t v[2][32];
        tmem_ld32(s_col + h * 64, v[0]);
        tmem_ld32(s_col + h * 64 + 32, v[1]);
        tmem_ld_wait();
#pragma unroll
        for (int q = 0; q < 2; ++q) {
            uint32_t w16[16];
#pragma unroll
            for (int i = 0; i < 16; ++i) {
                float x0 = __uint_as_float(v[q][2 * i]), x1 = __uint_as_float(v[q][2 * i + 1]);
                if (kMask) {
                    x0 = ((vis[2 * h + q] >> (2 * i)) & 1u) ? x0 : -INFINITY;
                    x1 = ((vis[2 * h + q] >> (2 * i + 1)) & 1u) ? x1 : -INFINITY;
                }
                const uint64_t y = ffma2(f2_bits(x0, x1), sc2, nm2);
                const float e0 = ex2(__uint_as_float((uint32_t)y));
                const float e1 = ex2(__uint_as_float((uint32_t)(y >> 32)));
                w16[i] = pack_bf16x2(e0, e1);
                if (i & 1) lb = fadd2(lb, f2_bits(e0, e1));
                else la = fadd2(la, f2_bits(e0, e1));
            }
            tmem_st16(s_col + (2 * h + q) * 16, w16);
        }
    }
    l4[0] += __uint_as_float((uint32_t)la);
    l4[1] += __uint_as_float((uint32_t)(la >> 32));
    l4[2] += __uint_as_float((uint32_t)lb);
    l4[3] += __uint_as_float((uint32_t)(lb >> 32));
}

}  // namespace rows

__global__ void __launch_bounds__(352, 1)
    tree_attn_rows_kernel(const __grid_constant__ CUtensorMap tm_q, const __grid_constant__ CUtensorMap tm_k,
                          const __grid_constant__ CUtensorMap tm_v, const __grid_constant__ CUtensorMap tm_k16,
                          const __grid_constant__ CUtensorMap tm_v16, const __grid_constant__ CUtensorMap tm_k4,
                          const __grid_constant__ CUtensorMap tm_v4, const __grid_constant__ CUtensorMap tm_k1,
                          const __grid_constant__ CUtensorMap tm_v1, const AttnParams p) {
    using namespace rows;
    // dynamic smem starts 1024-aligned (no static smem; the 1 KB system reservation precedes it):
    // the launch budgets no alignment slack, so a misaligned base is a hard error
    extern __shared__ __align__(1024) uint8_t smem[];
    if ((smem_u32(smem) & 1023u) != 0u) __trap();
    const int NS = p.nk_slots;                 // unified ring: K and V tiles in MMA consumption order
    uint8_t *s_ring = smem;
    uint8_t *s_q = s_ring + (size_t)NS * kSlotBytes;
    Misc *misc = reinterpret_cast<Misc *>(s_q + 2 * kQBuf);

    const int warp = threadIdx.x >> 5;
    const int lane = threadIdx.x & 31;
    const int NC = gridDim.x / p.lanes;        // CTA groups splitting the unit tile stream
    const int cl = blockIdx.x % p.lanes;       // this CTA's chunk lane
    if (threadIdx.x == 0) SPI_TRACE_K(0);

    if (threadIdx.x == 0) {
        for (int i = 0; i < NS; ++i) {
            mbar_init(&misc->full[i], 1);
            mbar_init(&misc->empty[i], 1);
        }
        for (int i = 0; i < 2; ++i) {
            mbar_init(&misc->q_full[i], 1);
            mbar_init(&misc->q_empty[i], 1);
            mbar_init(&misc->s_full[i], 1);
            mbar_init(&misc->p_full[i], 4);
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
        // rows past a request's last key are never loaded: slots must hold finite data (0 * NaN)
        for (int i = threadIdx.x - 96; i < NS * kSlotBytes / 16; i += 256)
            reinterpret_cast<uint4 *>(s_ring)[i] = make_uint4(0, 0, 0, 0);
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
        // ============================ TMA producer (one thread) ============================
        // Loads K and V tiles into one ring in exactly the order the MMA issuer consumes them:
        // K(0), K(1), then V(j), K(j + 2) for j = 0, 1, ...  (S(lt + 2) follows PV(lt)).  The K
        // cursor publishes the segment descriptors and loads each segment's Q; the V cursor follows
        // the published descriptors.
        // lane mode: the other chunks of the unit read the same tiles shortly after, from L2
        const uint64_t pol = p.lanes > 1 ? l2_evict_normal_policy() : l2_evict_first_policy();
        if (lane == 0) {
            int x = x_first;
            int4 next_info = first_info;
            int lsk = 0, lsv = 0;           // segments opened by the K / V cursors
            int li = 0;                     // ring loads issued
            SegDesc dk{}, dv{};
            int tk = 0, tv = 0;
            bool kdone = false, vdone = false;
            // next non-empty segment of this CTA's range -> ring slot lsk (terminal if none)
            auto publish = [&]() {
                SegDesc d{};
                d.x = -1;
                for (;; x += p.lanes) {
                    const int4 info = next_info;
                    if (info.x >= t1) break;  // (the sentinel item_info[n_items] starts at T)
                    next_info = __ldg(p.item_info + min(x + p.lanes, p.n_items));
                    const int begin = max(t0, info.x), end = min(t1, info.y);
                    if (end <= begin || info.w == 0) continue;  // no tiles here / empty chunk of the unit
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
                    x += p.lanes;
                    break;
                }
                misc->seg[lsk % kSegRing] = d;
                mbar_arrive(&misc->seg_full[lsk % kSegRing]);
                if (d.x >= 0) {
                    const int qb = lsk & 1;
                    if (lsk >= 2) mbar_wait(&misc->q_empty[qb], ((lsk >> 1) - 1) & 1);
                    mbar_arrive_expect_tx(&misc->q_full[qb], 2u * (uint32_t)(p.G * p.npc) * 128u);
                    uint8_t *qdst = s_q + qb * kQBuf;
                    const int node0 = d.b * p.Nmax + d.c * p.npc;
                    tma_load_3d(qdst, &tm_q, &misc->q_full[qb], 0, d.g * p.G, node0);
                    tma_load_3d(qdst + RB * 128, &tm_q, &misc->q_full[qb], 64, d.g * p.G, node0);
                }
                dk = d;
                tk = d.begin;
                kdone = d.x < 0;
                ++lsk;
            };
            auto open_v = [&]() {
                dv = misc->seg[lsv % kSegRing];  // published earlier by this thread
                tv = dv.begin;
                vdone = dv.x < 0;
                ++lsv;
            };
            // one tile of K (is_v = 0) or V (1) of segment d, tile t, into the next ring slot
            auto load = [&](const SegDesc &d, int t, bool is_v) {
                const int Kend = d.P + d.n;
                const int key0 = (t - d.ib) * kKeyTile;
                const int nv = min(kKeyTile, Kend - key0);
                const int row0 = kv_tile_row(p, d.b, d.g, key0);
                const int slot = li % NS, f = li / NS;
                if (f >= 1) mbar_wait(&misc->empty[slot], (f - 1) & 1);
                if (li == 0) SPI_TRACE_K(2);
                uint8_t *dst = s_ring + (size_t)slot * kSlotBytes;
                uint64_t *bar = &misc->full[slot];
                const CUtensorMap *m = is_v ? &tm_v : &tm_k;
                if (SPI_FLAGS(p) & 1) {  // experiment: no K/V traffic (results invalid)
                    mbar_arrive(bar);
                } else if (nv == kKeyTile) {
                    mbar_arrive_expect_tx(bar, kSlotBytes);
                    tma_load_2d(dst, m, bar, 0, row0, pol);
                    tma_load_2d(dst + kHalfBytes, m, bar, 64, row0, pol);
                } else if (is_v) {
                    tma_load_rows(dst, bar, nv, row0, pol, &tm_v16, &tm_v4, &tm_v1);
                } else {
                    tma_load_rows(dst, bar, nv, row0, pol, &tm_k16, &tm_k4, &tm_k1);
                }
                ++li;
            };
            int lt_k = 0, lt_v = 0;
            auto step_k = [&]() {
                {
                    const int lt = lt_k;
                    SPI_TRACE(0);
                }
                load(dk, tk, false);
                ++lt_k;
                if (++tk == dk.end) publish();
            };
            auto step_v = [&]() {
                {
                    const int lt = lt_v;
                    SPI_TRACE(1);
                }
                load(dv, tv, true);
                ++lt_v;
                if (++tv == dv.end) open_v();
            };
            publish();
            open_v();
            for (int i = 0; i < 2 && !kdone; ++i) step_k();
            while (!vdone) {
                step_v();
                if (!kdone) step_k();
            }
            grid_launch_dependents();
        }
    } else if (warp == 1) {
        // ===================== S issuer: S = Q K^T (M = 128 rows, N = 128 keys) =====================
        // S(lt) goes to buffer lt & 1; P(lt) is written over the same columns, so the buffer is
        // free again once PV(lt - 2) has completed (p_empty).  K(j) is ring load j (j < 2) or
        // 2j - 1 (the producer's order K0 K1 V0 K2 V1 K3 ...).
        if (lane == 0) {
            const uint32_t idesc_s = make_idesc_bf16(128, 128, false, false);
            const uint32_t ring_addr = smem_u32(s_ring), q_addr = smem_u32(s_q);
            int lt = 0, ls = 0;
            while (true) {
                mbar_wait(&misc->seg_full[ls % kSegRing], (ls / kSegRing) & 1);
                const SegDesc d = misc->seg[ls % kSegRing];
                if (d.x < 0) break;
                const int qb = ls & 1;
                mbar_wait(&misc->q_full[qb], (ls >> 1) & 1);
                for (int t = d.begin; t < d.end; ++t, ++lt) {
                    const int li = lt < 2 ? lt : 2 * lt - 1;
                    const int slot = li % NS;
                    mbar_wait(&misc->full[slot], (li / NS) & 1);
                    const int sb = lt & 1;
                    if (lt >= 2) mbar_wait(&misc->p_empty[sb], ((lt - 2) >> 1) & 1);
                    tc_fence_after();
                    SPI_TRACE(2);
                    const uint32_t kbase = ring_addr + slot * kSlotBytes;
                    const uint32_t qbase = q_addr + qb * kQBuf;
#pragma unroll
                    for (int kk = 0; kk < kHeadDim / 16; ++kk) {
                        const uint32_t off = (kk >> 2) * (RB * 128) + (kk & 3) * 32;
                        const uint64_t adesc = make_smem_desc(qbase + off, 16, 1024, kSw128);
                        const uint64_t bdesc = make_smem_desc(kbase + (kk >> 2) * kHalfBytes + (kk & 3) * 32, 16,
                                                              1024, kSw128);
                        if (!(SPI_FLAGS(p) & 2))
                            umma_bf16_ss(tmem + kColS + sb * 128, adesc, bdesc, idesc_s, kk > 0 ? 1u : 0u);
                    }
                    umma_commit(&misc->s_full[sb]);
                    umma_commit(&misc->empty[slot]);
                    if (t == d.end - 1) umma_commit(&misc->q_empty[qb]);
                }
                ++ls;
            }
        }
    } else if (warp == 2) {
        // ========== PV issuer: O_{lt&1} += P V (A = P in TMEM over S(lt), N = 128 dims) ==========
        // V(j) is ring load 2j + 2, except the CTA's last tile (2j + 1: no K load follows it).
        if (lane == 0) {
            const uint32_t idesc_o = make_idesc_bf16(128, 128, false, true);
            const uint32_t ring_addr = smem_u32(s_ring);
            int lt = 0, ls = 0;
            mbar_wait(&misc->seg_full[0], 0);
            SegDesc d = misc->seg[0];
            while (d.x >= 0) {
                SegDesc dn{};
                bool have_next = false;
                for (int t = d.begin; t < d.end; ++t, ++lt) {
                    const int pb = lt & 1;
                    mbar_wait(&misc->p_full[pb], (lt >> 1) & 1);
                    bool last = false;
                    if (t == d.end - 1) {
                        // the next descriptor is published right after this segment's last K load
                        mbar_wait(&misc->seg_full[(ls + 1) % kSegRing], ((ls + 1) / kSegRing) & 1);
                        dn = misc->seg[(ls + 1) % kSegRing];
                        have_next = true;
                        last = dn.x < 0;
                    }
                    const int li = last ? 2 * lt + 1 : 2 * lt + 2;
                    const int slot = li % NS;
                    mbar_wait(&misc->full[slot], (li / NS) & 1);
                    tc_fence_after();
                    SPI_TRACE(3);
                    const uint32_t vbase = ring_addr + slot * kSlotBytes;
                    const bool first = (t - d.begin) < 2;  // first tile of group pb in this segment
#pragma unroll
                    for (int kk = 0; kk < kKeyTile / 16; ++kk) {
                        const uint64_t bdesc = make_smem_desc(vbase + kk * 16 * 128, kHalfBytes, 1024, kSw128);
                        if (!(SPI_FLAGS(p) & 2))
                            umma_bf16_ts(tmem + kColO + pb * 128, tmem + kColS + pb * 128 + kk * 8, bdesc, idesc_o,
                                         (first && kk == 0) ? 0u : 1u);
                    }
                    umma_commit(&misc->p_empty[pb]);
                    umma_commit(&misc->empty[slot]);
                }
                ++ls;
                if (!have_next) {  // (empty segments do not exist; kept for safety)
                    mbar_wait(&misc->seg_full[ls % kSegRing], (ls / kSegRing) & 1);
                    dn = misc->seg[ls % kSegRing];
                }
                d = dn;
            }
        }
    } else {
        // ============ softmax / epilogue: two groups of 4 warps, alternating KV tiles ============
        // group g (warps 3 + 4g .. 6 + 4g) owns the tiles with lt & 1 == g: S buffer g, its own
        // accumulator O_g and running (m, l) per row; thread = one query row (TMEM lane).  The
        // groups run out of phase, so one group's TMEM / barrier latency hides behind the other's
        // exponentials.  At a segment's end the two partial softmax states are merged by
        // log-sum-exp (group g writes dims [64 g, 64 g + 64) of the row).
        const int sw = warp - 3;               // 0..7
        const int grp = sw >> 2;               // tile parity owned by this group
        const int qd = warp & 3;               // TMEM lane quarter
        const int r = qd * 32 + lane;          // query row of the item = TMEM lane
        const uint32_t lane_off = (uint32_t)(qd * 32) << 16;
        const uint32_t pair_bar = 2 + qd;      // named barrier of the two warps of lane quarter qd
        const uint32_t s_col = tmem + kColS + grp * 128 + lane_off;
        const uint32_t o_col = tmem + kColO + grp * 128 + lane_off;
        int lt = 0, ls = 0;
        while (true) {
            mbar_wait(&misc->seg_full[ls % kSegRing], (ls / kSegRing) & 1);
            const SegDesc sd = misc->seg[ls % kSegRing];
            if (sd.x < 0) break;
            const int b = sd.b, g = sd.g, c = sd.c, P = sd.P, n = sd.n;
            const int Kend = P + n;
            const int G = p.G;
            const int rc = G * p.npc;
            const int node = c * p.npc + r / G, hl = r % G;
            const bool row_valid = (r < rc) && (node < n);
            // ancestor-or-self bitset of this row's node, read on masked tiles only (rows without a
            // node use node 0's root path, which keeps them finite; they are never written)
            const uint32_t *anc = p.anc + ((size_t)b * p.Nmax + (row_valid ? node : 0)) * kBitWords;
            float m = -INFINITY, l = 0.f;  // this group's running row max (log2 units) and sum
            int last_own = -1;
            for (int t = sd.begin; t < sd.end; ++t, ++lt) {
                if ((lt & 1) != grp) continue;
                const int key0 = (t - sd.ib) * kKeyTile;
                mbar_wait(&misc->s_full[grp], (lt >> 1) & 1);
                tc_fence_after();
                if (r == 0) SPI_TRACE(4 + grp);
                // visibility of the tile's 128 keys (4 words): committed keys visible; tree keys by
                // the ancestor bitset; keys past the request's end: none
                uint32_t vis[4] = {0xFFFFFFFFu, 0xFFFFFFFFu, 0xFFFFFFFFu, 0xFFFFFFFFu};
                const bool masked = key0 + kKeyTile > P;
                if (masked) {
#pragma unroll
                    for (int q = 0; q < 4; ++q) {
                        const int j0 = key0 + 32 * q - P;  // tree index of the group's first key
                        if (j0 + 32 > 0) {
                            const int jb = max(j0, 0);
                            const int wi = jb >> 5, sh = jb & 31;
                            const uint32_t lo = __ldg(anc + wi);
                            const uint32_t hi = wi + 1 < kBitWords ? __ldg(anc + wi + 1) : 0u;
                            uint32_t bits = sh ? ((lo >> sh) | (hi << (32 - sh))) : lo;
                            if (j0 < 0) bits = (bits << (-j0)) | ((1u << (-j0)) - 1u);
                            const int nvalid = Kend - (key0 + 32 * q);
                            if (nvalid < 32) bits &= nvalid <= 0 ? 0u : ((1u << nvalid) - 1u);
                            vis[q] = bits;
                        }
                    }
                }
                // pass 1: tile row max (unmasked tiles, the common case, take the select-free path)
                float tm4[4] = {-INFINITY, -INFINITY, -INFINITY, -INFINITY};
                if (masked) tile_max<true>(s_col, vis, tm4);
                else if (SPI_FLAGS(p) & 4) tm4[0] = 1.f;  // experiment: no S loads (results invalid)
                else tile_max<false>(s_col, vis, tm4);
                const float tm = fmaxf(fmaxf(tm4[0], tm4[1]), fmaxf(tm4[2], tm4[3])) * p.scale_log2;
                // stale running max: move it only when this tile exceeds it by more than 2^8
                float alpha = 1.f;
                if (tm > m + kRescaleThreshold) {
                    alpha = (m == -INFINITY) ? 0.f : ex2(m - tm);
                    m = tm;
                    l *= alpha;
                }
                if (__any_sync(0xffffffffu, alpha != 1.f) && t - sd.begin >= 2) {
                    // rescale O_g rows: PV of this group's previous tile must be complete
                    mbar_wait(&misc->p_empty[grp], ((lt - 2) >> 1) & 1);
                    tc_fence_after();
#pragma unroll
                    for (int q2 = 0; q2 < 4; ++q2) {
                        uint32_t v[32];
                        tmem_ld32(o_col + q2 * 32, v);
                        tmem_ld_wait();
                        uint32_t w16[16];
#pragma unroll
                        for (int h = 0; h < 2; ++h) {
#pragma unroll
                            for (int i = 0; i < 16; ++i) w16[i] = __float_as_uint(__uint_as_float(v[h * 16 + i]) * alpha);
                            tmem_st16(o_col + q2 * 32 + h * 16, w16);
                        }
                    }
                    tmem_st_wait();
                }
                const float mref = (m == -INFINITY) ? 0.f : m;
                // pass 2: P = 2^(s * scale - m) as bf16 pairs over the first 64 columns of S(lt)
                // (keys 32 q .. 32 q + 31 -> columns 16 q .. 16 q + 15: always already read)
                float l4[4] = {0.f, 0.f, 0.f, 0.f};
                if (masked) tile_exp<true>(s_col, vis, p.scale_log2, mref, l4);
                else if (SPI_FLAGS(p) & 8) l4[0] = 1.f;  // experiment: no softmax work (results invalid)
                else tile_exp<false>(s_col, vis, p.scale_log2, mref, l4);
                l += (l4[0] + l4[1]) + (l4[2] + l4[3]);
                tmem_st_wait();
                tc_fence_before();
                __syncwarp();
                if (lane == 0) mbar_arrive(&misc->p_full[grp]);
                if (r == 0) SPI_TRACE(6 + grp);
                last_own = lt;
            }

            // ============ epilogue of this segment: merge the two groups, store ============
            if (last_own >= 0) mbar_wait(&misc->p_empty[grp], (last_own >> 1) & 1);  // own last PV done
            // (m, l) exchange through one float2 per row: group 1 publishes, group 0 reads it and
            // publishes its own after a second barrier
            if (grp == 1) misc->xch[r] = make_float2(m, l);
            tc_fence_before();
            named_bar_sync(pair_bar, 64);
            tc_fence_after();
            const float2 other = misc->xch[r];
            named_bar_sync(pair_bar, 64);
            if (grp == 0) misc->xch[r] = make_float2(m, l);
            named_bar_sync(pair_bar, 64);
            const float2 mine = make_float2(m, l);
            const float2 g0 = (grp == 0) ? mine : misc->xch[r];
            const float2 g1 = (grp == 1) ? mine : other;
            if (r == 0 && grp == 0) SPI_TRACE(8);
            const float mA = g0.x, mB = g1.x;
            const float M = fmaxf(mA, mB);
            const float wA = (mA == -INFINITY) ? 0.f : ex2(mA - M);
            const float wB = (mB == -INFINITY) ? 0.f : ex2(mB - M);
            const float lrow = wA * g0.y + wB * g1.y;
            const bool useA = mA != -INFINITY, useB = mB != -INFINITY;
            const uint32_t oA = tmem + kColO + grp * 64 + lane_off;        // dims [64 grp, 64 grp + 64)
            const uint32_t oB = tmem + kColO + 128 + grp * 64 + lane_off;
            const bool full = (sd.begin == sd.ib) && (sd.end == sd.ie);
            // merged, unnormalised O row half (16 dims at a time)
            auto merged = [&](int q4, float (&o)[16]) {
                uint32_t va[16], vb[16];
                tmem_ld16(oA + q4 * 16, va);
                tmem_ld16(oB + q4 * 16, vb);
                tmem_ld_wait();
#pragma unroll
                for (int i = 0; i < 16; ++i)
                    o[i] = (useA ? wA * __uint_as_float(va[i]) : 0.f) + (useB ? wB * __uint_as_float(vb[i]) : 0.f);
            };
            if (full) {
                const float inv = 1.0f / lrow;
                __nv_bfloat16 *orow = p.out + (((size_t)b * p.Nmax + node) * p.Hq + g * G + hl) * kHeadDim + grp * 64;
#pragma unroll 1
                for (int q4 = 0; q4 < 4; ++q4) {
                    float o[16];
                    merged(q4, o);
                    if (row_valid) {
#pragma unroll
                        for (int i = 0; i < 16; i += 8) {
                            uint4 o4;
                            o4.x = pack_bf16x2(o[i] * inv, o[i + 1] * inv);
                            o4.y = pack_bf16x2(o[i + 2] * inv, o[i + 3] * inv);
                            o4.z = pack_bf16x2(o[i + 4] * inv, o[i + 5] * inv);
                            o4.w = pack_bf16x2(o[i + 6] * inv, o[i + 7] * inv);
                            *reinterpret_cast<uint4 *>(orow + q4 * 16 + i) = o4;
                        }
                    }
                }
            } else {
                const int slot = (sd.begin == t0) ? 0 : 1;
                float *po = p.part_o + (((size_t)blockIdx.x * 2 + slot) * RB + r) * kHeadDim + grp * 64;
#pragma unroll 1
                for (int q4 = 0; q4 < 4; ++q4) {
                    float o[16];
                    merged(q4, o);
#pragma unroll
                    for (int i = 0; i < 16; i += 4)
                        *reinterpret_cast<float4 *>(po + q4 * 16 + i) = make_float4(o[i], o[i + 1], o[i + 2], o[i + 3]);
                }
                float *pml = p.part_ml + ((size_t)blockIdx.x * 2 + slot) * 2 * RB;
                if (grp == 0) {
                    pml[r] = M;
                    pml[RB + r] = lrow;
                }
                __threadfence();
                named_bar_sync(1, 256);
                if (r == 0 && grp == 0) {
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
                    float Mx = -INFINITY;
                    for (int cc = c_first; cc <= c_last; ++cc) {
                        const int s0 = cta_start(cc, T, NC);
                        if (cta_start(cc + 1, T, NC) <= s0) continue;
                        const size_t po2 = ((size_t)cc * p.lanes + cl) * 2 + ((s0 >= sd.ib) ? 0 : 1);
                        Mx = fmaxf(Mx, ldcg_f32(p.part_ml + po2 * 2 * RB + r));
                    }
                    float Ls = 0.f;
                    for (int cc = c_first; cc <= c_last; ++cc) {
                        const int s0 = cta_start(cc, T, NC);
                        if (cta_start(cc + 1, T, NC) <= s0) continue;
                        const size_t po2 = ((size_t)cc * p.lanes + cl) * 2 + ((s0 >= sd.ib) ? 0 : 1);
                        const float mp = ldcg_f32(p.part_ml + po2 * 2 * RB + r);
                        if (mp != -INFINITY) Ls += ex2(mp - Mx) * ldcg_f32(p.part_ml + po2 * 2 * RB + RB + r);
                    }
                    const float inv = 1.0f / Ls;
                    __nv_bfloat16 *orow = p.out + (((size_t)b * p.Nmax + node) * p.Hq + g * G + hl) * kHeadDim + grp * 64;
                    for (int q2 = 0; q2 < 2; ++q2) {
                        float acc[32];
#pragma unroll
                        for (int i = 0; i < 32; ++i) acc[i] = 0.f;
                        for (int cc = c_first; cc <= c_last; ++cc) {
                            const int s0 = cta_start(cc, T, NC);
                            if (cta_start(cc + 1, T, NC) <= s0) continue;
                            const size_t po2 = ((size_t)cc * p.lanes + cl) * 2 + ((s0 >= sd.ib) ? 0 : 1);
                            const float mp = ldcg_f32(p.part_ml + po2 * 2 * RB + r);
                            if (mp == -INFINITY) continue;
                            const float w = ex2(mp - Mx) * inv;
                            const float4 *src = reinterpret_cast<const float4 *>(
                                p.part_o + (po2 * RB + r) * kHeadDim + grp * 64 + q2 * 32);
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
            named_bar_sync(pair_bar, 64);  // both O accumulators and (m, l) read before reuse
            if (r == 0 && grp == 0) SPI_TRACE(9);
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
    return (size_t)num_slots * kSlotBytes + 2 * rows::kQBuf + sizeof(rows::Misc);
}

cudaError_t launch_tree_attention_rows(const AttnParams &prm0, const void *q, const void *k, const void *v,
                                       int num_ctas, size_t max_smem, cudaStream_t stream) {
    AttnParams prm = prm0;
    CUtensorMap tq, tk, tv, tk16, tv16, tk4, tv4, tk1, tv1;
    const uint64_t rows = prm.page_table ? (uint64_t)prm.n_pages * prm.Hkv * kKeyTile
                                         : (uint64_t)prm.B * prm.Hkv * prm.Smax;
    if (!encode_q(&tq, q, prm.Hq, (uint64_t)prm.B * prm.Nmax, prm.G, prm.npc) ||
        !encode_2d(&tk, k, rows, kKeyTile) || !encode_2d(&tv, v, rows, kKeyTile) ||
        !encode_2d(&tk16, k, rows, 16) || !encode_2d(&tv16, v, rows, 16) || !encode_2d(&tk4, k, rows, 4) ||
        !encode_2d(&tv4, v, rows, 4) || !encode_2d(&tk1, k, rows, 1) || !encode_2d(&tv1, v, rows, 1))
        return cudaErrorInvalidValue;
    int ns = rows::kMaxRing;
    while (ns > 2 && rows_smem_bytes(ns) > max_smem) --ns;
    prm.nk_slots = ns;  // unified K/V ring
    prm.nv_slots = 0;
    const size_t smem = rows_smem_bytes(ns);
    {
        const cudaError_t e = ensure_max_smem_attr((const void *)tree_attn_rows_kernel, 3, max_smem);
        if (e != cudaSuccess) return e;
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
