// tree_attention_rows.cu — K2 tree attention for wide trees / GQA groups (G * Nmax > 64 query rows
// per kv-head), sm_100a.  Same computation and schedule as tree_attention.cu (Def. 4.1
// L594-598, Eq. 1-4, topology-aware mask L645-674), different tiling:
//  * a work item is (request, kv-head, block of 128 query rows); the UMMA M dimension is the query
//    rows (one TMEM lane per row), N = 128 keys for S = Q K^T and N = 128 dims for O += P V;
//  * TMEM = S0 | S1 | O | P0 | P1 (128 + 128 + 128 + 64 + 64 columns): S double-buffered, ONE O
//    accumulator, P (bf16 pairs) in its own columns.  The softmax reads a tile's 128 scores per row
//    into registers ONCE and releases the S buffer right there, so S(t + 2) is issued while tile t's
//    softmax runs (round 1 aliased P over S: S -> softmax -> PV -> S(t + 2) was one chain);
//  * 8 softmax warps in two groups of 4 (one warp per TMEM lane quarter each, thread = query row);
//    group g owns the tiles with t & 1 == g and both accumulate into the one O, so every P(t) uses
//    the row reference the previous tile left: the owner of tile t reads decision(t - 1) from the
//    other group (shared memory + one named barrier per direction and lane quarter), may raise it
//    (stale max: only beyond 2^8, then O is rescaled in TMEM after PV(t - 1)), publishes decision(t)
//    and only then computes its exponentials into registers; only their TMEM store waits for PV(t - 2)
//    to have released the P buffer -- the groups run out of phase;
//  * segment end: the non-owner group hands its row sums to the owner of the last tile (mbarriers,
//    neither group blocks), the owner hands the combined (row sum, reference) to an EPILOGUE
//    WARPGROUP, which waits for the segment's last PV, reads O and writes the rows (a whole item) or
//    the fp32 partial (a split piece; the last piece merges) -- the softmax groups go straight on with
//    the next segment, whose PVs wait only until the epilogue has read O;
//  * K and V in separate TMA rings fed by two producer warps; S issuer and PV issuer threads;
//  * warpgroups: 0-1 softmax, 2 control (producers, issuers), 3 epilogue; setmaxnreg moves registers
//    from the control and epilogue warpgroups (56 per thread) to the softmax warpgroups (200: the
//    scores stay in registers);
//  * schedule: with at least half an item per CTA, whole items claimed dynamically (item blockIdx.x
//    first, then tickets from an atomic counter reset by tree_prepare): the row blocks of one (request,
//    kv-head) are consecutive tickets, so they stream the same KV tiles at about the same time and the
//    second reads them from L2 (ncu: DRAM bytes = the algorithmic bytes).  Fewer items: the static
//    stream-K split in lane mode -- the row blocks of a (request, kv-head) on `lanes` CTAs in lock-step
//    over the same tile range;
//  * tree keys are masked with the ancestor-or-self bitset of the row's node (tree_prepare);
//  * the stream-K schedule, segment descriptors, row-exact tail loads, split combine and PDL are
//    shared with the swapped kernel (attn_shared.cuh).
#include "attn_shared.cuh"

namespace specinfer {

namespace rows {

constexpr int RB = kRowsBlock;              // 128 query rows per item
constexpr int kQBuf = 2 * RB * 128;          // one Q buffer: 2 halves x 128 rows x 128 B
constexpr int kTmemCols = 512;
constexpr int kColS = 0, kColO = 256, kColP = 384;
// warp roles: 0-7 softmax (two groups of 4, warp & 3 = TMEM lane quarter), 8 Q / K producer, 9 S issuer
// (+ TMEM allocation), 10 PV issuer, 11 V producer, 12-15 epilogue (warp & 3 = TMEM lane quarter).  The
// control (8-11) and epilogue (12-15) warpgroups give registers to the softmax warpgroups (setmaxnreg):
// 128 per thread at launch -> 56 / 56 / 200
constexpr int kThreads = 512;
constexpr int kWarpProd = 8, kWarpS = 9, kWarpPV = 10, kWarpV = 11;
constexpr int kRegsCtl = 56, kRegsEpi = 56, kRegsSoftmax = 200;
constexpr int kMaxK = 4, kMaxV = 4;          // ring slots (the launch picks 3 K + 2 V)

struct Misc {
    uint64_t k_full[kMaxK], k_empty[kMaxK];
    uint64_t v_full[kMaxV], v_empty[kMaxV];
    uint64_t q_full[2], q_empty[2];
    uint64_t s_full[2], s_free[2];           // S(t) ready / S buffer t & 1 loaded by the softmax
    uint64_t p_full[2], pv_done[2];          // P(t) written / PV(t) complete (P buffer free, O advanced)
    uint64_t o_free;                         // the epilogue has read O (next segment may overwrite it)
    uint64_t o_full;                         // a segment's last PV complete (O final)
    uint64_t epi_full[2], epi_empty[2];      // fin[slot] written by the segment's owner group / read
    uint64_t xl_full[2], xl_empty[2];        // xl[slot] written by the non-owner group / read by the owner
    float xl[2][2][RB];                      // [segment & 1][non-owner row sum, its reference][row]
    float fin[2][2][RB];                     // [segment & 1][row sum, row reference][row] -> epilogue
    uint64_t seg_full[kSegRing];
    SegDesc seg[kSegRing];
    uint64_t stage_bar;                      // bulk staging of split pieces (CTA's last segment)
    uint32_t tmem_base;
    int32_t bcast;
    float mref[RB];                          // [row] the row reference after the latest decision
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

// The normalised bf16 output of one query row (TMEM columns of O), 32 dims per TMEM load: the warp
// releases O (arrives on `o_free`: the next segment's first PV may overwrite it) right after its last
// TMEM load; the 32-byte global stores stay off the critical path.
__device__ __forceinline__ void store_o_row(uint32_t o_col, float inv, bool row_valid, __nv_bfloat16 *orow,
                                            uint64_t *o_free) {
    const bool al32 = (reinterpret_cast<uintptr_t>(orow) & 31u) == 0;
#pragma unroll 1
    for (int q = 0; q < 4; ++q) {
        uint32_t o[32];
        tmem_ld32(o_col + q * 32, o);
        tmem_ld_wait();
        if (q == 3) {
            tc_fence_before();
            __syncwarp();
            if ((threadIdx.x & 31) == 0) mbar_arrive(o_free);
        }
        if (!row_valid) continue;
        uint32_t w[16];
#pragma unroll
        for (int i = 0; i < 16; ++i) w[i] = pack_bf16x2(__uint_as_float(o[2 * i]) * inv, __uint_as_float(o[2 * i + 1]) * inv);
        __nv_bfloat16 *dst = orow + q * 32;
        if (al32) {
#pragma unroll
            for (int k = 0; k < 2; ++k)
                asm volatile("st.global.v8.b32 [%0], {%1, %2, %3, %4, %5, %6, %7, %8};" ::"l"(dst + k * 16),
                             "r"(w[8 * k]), "r"(w[8 * k + 1]), "r"(w[8 * k + 2]), "r"(w[8 * k + 3]), "r"(w[8 * k + 4]),
                             "r"(w[8 * k + 5]), "r"(w[8 * k + 6]), "r"(w[8 * k + 7])
                             : "memory");
        } else {
#pragma unroll
            for (int k = 0; k < 4; ++k)
                *reinterpret_cast<uint4 *>(dst + k * 8) = make_uint4(w[4 * k], w[4 * k + 1], w[4 * k + 2], w[4 * k + 3]);
        }
    }
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

// 2^x for a pair of x <= 8 on the FMA/ALU pipes (round-to-nearest split x = n + f, f in [-1/2, 1/2],
// degree-4 Taylor polynomial of 2^f: relative error < 5e-5, far below the bf16 rounding of P)
__device__ __forceinline__ uint64_t exp2_poly2(uint64_t x2) {
    const float x0 = fmaxf(__uint_as_float((uint32_t)x2), -126.f);
    const float x1 = fmaxf(__uint_as_float((uint32_t)(x2 >> 32)), -126.f);
    const uint64_t xm = f2_bits(x0, x1);
    const uint64_t magic = f2_bits(12582912.f, 12582912.f);   // 1.5 * 2^23: rint via the fp adder
    const uint64_t t = fadd2(xm, magic);
    const uint64_t nf = fadd2(t, f2_bits(-12582912.f, -12582912.f));
    const uint64_t f = fadd2(xm, nf ^ 0x8000000080000000ull);   // x - n
    uint64_t q = f2_bits(0.009618129f, 0.009618129f);
    q = ffma2(q, f, f2_bits(0.05550411f, 0.05550411f));
    q = ffma2(q, f, f2_bits(0.2402265f, 0.2402265f));
    q = ffma2(q, f, f2_bits(0.6931472f, 0.6931472f));
    q = ffma2(q, f, f2_bits(1.f, 1.f));
    const uint32_t n0 = (uint32_t)t - 0x4B400000u, n1 = (uint32_t)(t >> 32) - 0x4B400000u;
    return (uint64_t)((uint32_t)q + (n0 << 23)) | ((uint64_t)((uint32_t)(q >> 32) + (n1 << 23)) << 32);
}

// P = 2^(s * scale_log2 - mref) of 32 keys as 16 bf16 pairs (into w, not yet stored); returns the fp32
// sum of the bf16-ROUNDED values, so the normalisation matches the numerator the PV MMA computes.
// kMax: also the max of the (raw) s values, for the deferred stale-max check.
template <bool kMax>
__device__ __forceinline__ float exp32(const uint32_t (&v)[32], uint64_t sc2, uint64_t nm2, uint32_t (&w)[16],
                                       float &pm) {
    float acc[4] = {0.f, 0.f, 0.f, 0.f};
    float m2[2] = {-INFINITY, -INFINITY};
#pragma unroll
    for (int i = 0; i < 16; ++i) {
        const float x0 = __uint_as_float(v[2 * i]), x1 = __uint_as_float(v[2 * i + 1]);
        if (kMax) m2[i & 1] = fmaxf(m2[i & 1], fmaxf(x0, x1));
        const uint64_t y = ffma2(f2_bits(x0, x1), sc2, nm2);
        float e0, e1;
#ifdef ROWS_POLY_EXP
        if ((i & 3) == 3) {   // a quarter of the exponentials on the FMA pipe (MUFU relief)
            const uint64_t e = exp2_poly2(y);
            e0 = __uint_as_float((uint32_t)e);
            e1 = __uint_as_float((uint32_t)(e >> 32));
        } else
#endif
        {
            e0 = ex2(__uint_as_float((uint32_t)y));
            e1 = ex2(__uint_as_float((uint32_t)(y >> 32)));
        }
        w[i] = pack_bf16x2(e0, e1);
        // row sum of the rounded values: the bf16 halves added in place (no unpacking)
        acc[2 * (i & 1)] = add_bf16lo(w[i], acc[2 * (i & 1)]);
        acc[2 * (i & 1) + 1] = add_bf16hi(w[i], acc[2 * (i & 1) + 1]);
    }
    if (kMax) pm = fmaxf(pm, fmaxf(m2[0], m2[1]));
    return (acc[0] + acc[1]) + (acc[2] + acc[3]);
}

// masks 32 S values in place (invisible -> -inf)
__device__ __forceinline__ void mask32(uint32_t (&v)[32], uint32_t vis) {
#pragma unroll
    for (int i = 0; i < 32; ++i)
        if (!((vis >> i) & 1u)) v[i] = __float_as_uint(-INFINITY);
}

}  // namespace rows

__global__ void __launch_bounds__(rows::kThreads, 1)
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
    const int NK = p.nk_slots, NV = p.nv_slots;
    uint8_t *s_k = smem;
    uint8_t *s_v = s_k + (size_t)NK * kSlotBytes;
    uint8_t *s_q = s_v + (size_t)NV * kSlotBytes;
    Misc *misc = reinterpret_cast<Misc *>(s_q + 2 * kQBuf);

    const int warp = threadIdx.x >> 5;
    const int lane = threadIdx.x & 31;
    const int NC = gridDim.x / p.lanes;        // CTA groups splitting the unit tile stream
    const int cl = blockIdx.x % p.lanes;       // this CTA's chunk lane
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
            mbar_init(&misc->s_free[i], 4);
            mbar_init(&misc->p_full[i], 4);
            mbar_init(&misc->pv_done[i], 1);
        }
        mbar_init(&misc->o_free, 4);   // the epilogue warpgroup's 4 warps
        mbar_init(&misc->o_full, 1);
        for (int i = 0; i < 2; ++i) {
            mbar_init(&misc->epi_full[i], 4);
            mbar_init(&misc->epi_empty[i], 4);
            mbar_init(&misc->xl_full[i], 4);
            mbar_init(&misc->xl_empty[i], 4);
        }
        mbar_init(&misc->stage_bar, 1);
        for (int i = 0; i < kSegRing; ++i) mbar_init(&misc->seg_full[i], 1);
        fence_barrier_init();
    }
    if (warp == kWarpProd && lane == 0) {
        tma_prefetch_desc(&tm_q);
        tma_prefetch_desc(&tm_k);
        tma_prefetch_desc(&tm_v);
    }
    if (warp < 8) {
        // Q rows beyond an item's G*npc rows are never written by TMA: keep them zero
        for (int i = threadIdx.x; i < 2 * kQBuf / 16; i += 256)
            reinterpret_cast<uint4 *>(s_q)[i] = make_uint4(0, 0, 0, 0);
        // rows past a request's last key are never loaded: slots must hold finite data (0 * NaN)
        for (int i = threadIdx.x; i < (NK + NV) * kSlotBytes / 16; i += 256)
            reinterpret_cast<uint4 *>(s_k)[i] = make_uint4(0, 0, 0, 0);
        fence_proxy_async_smem();
    }
    if (warp == kWarpS) tmem_alloc<kTmemCols>(&misc->tmem_base);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem = misc->tmem_base;

    // Programmatic dependent launch (see tree_attention.cu): the producer warp may stage
    // committed-prefix tiles of its first segment before the dependency resolves (early_prefix)
    const bool early = p.early_prefix != 0 && (warp == kWarpProd || warp == kWarpV);
    if (!early) grid_dependency_wait();
    const int4 ci = __ldg(p.cta_info + 2 * blockIdx.x);
    const int4 first_info = __ldg(p.cta_info + 2 * blockIdx.x + 1);
    const int t0 = ci.x, t1 = ci.y, x_first = ci.z, T = ci.w;
    const int ntiles = p.dyn ? 1 : t1 - t0;   // (dynamic mode: every CTA starts with item blockIdx.x)

    if (warp >= 12) {
        // epilogue warpgroup (warp & 3 = TMEM lane quarter): its registers go to the softmax warps
        setmaxnreg_dec<kRegsEpi>();
        if (ntiles > 0) {
            // ====== epilogue: per segment, once the owner group handed over (row sum, reference) and the
            // segment's last PV completed, O -> normalised bf16 rows (a whole item) or the fp32 partial of a
            // split piece (the last piece merges every piece); O is released after its TMEM loads ======
            const int qd = warp & 3;
            const int r = qd * 32 + lane;
            const uint32_t lane_off = (uint32_t)(qd * 32) << 16;
            const uint32_t o_col = tmem + kColO + lane_off;
            int ls = 0, lt_end = 0;
            for (;;) {
                mbar_wait(&misc->seg_full[ls % kSegRing], (ls / kSegRing) & 1);
                const SegDesc sd = misc->seg[ls % kSegRing];
                if (sd.x < 0) break;
                lt_end += sd.end - sd.begin;
                const int lt = lt_end - 1;   // (trace slots: the segment's last tile)
                const int b = sd.b, g = sd.g, c = sd.c, n = sd.n;
                const int G = p.G;
                const int rc = G * p.npc;
                const int node = c * p.npc + r / G, hl = r % G;
                const bool row_valid = (r < rc) && (node < n);
                const bool full = (sd.begin == sd.ib) && (sd.end == sd.ie);
                const int fs = ls & 1;
                mbar_wait(&misc->epi_full[fs], (ls >> 1) & 1);
                if (r == 0) SPI_TRACE(10);
                const float lrow = misc->fin[fs][0][r], m = misc->fin[fs][1][r];
                __syncwarp();
                if (lane == 0) mbar_arrive(&misc->epi_empty[fs]);
                mbar_wait(&misc->o_full, ls & 1);   // one phase per segment, consumed in order
                tc_fence_after();
                if (r == 0) SPI_TRACE(11);
                if (full) {
                    store_o_row(o_col, 1.0f / lrow, row_valid,
                                p.out + (((size_t)b * p.Nmax + node) * p.Hq + g * G + hl) * kHeadDim, &misc->o_free);
                } else {
                    // a piece of a split item: unnormalised O row, (m, l) of the row, then the last piece
                    // merges every piece by log-sum-exp
                    const int slot = (sd.begin == t0) ? 0 : 1;
                    float *po = p.part_o + (((size_t)blockIdx.x * 2 + slot) * RB + r) * kHeadDim;
#pragma unroll 1
                    for (int q2 = 0; q2 < 4; ++q2) {
                        uint32_t o[32];
                        tmem_ld32(o_col + q2 * 32, o);
                        tmem_ld_wait();
#pragma unroll
                        for (int i = 0; i < 32; i += 8)   // 32-byte stores (part_o rows are 512-byte aligned)
                            asm volatile("st.global.v8.b32 [%0], {%1, %2, %3, %4, %5, %6, %7, %8};" ::"l"(po + q2 * 32 + i),
                                         "r"(o[i]), "r"(o[i + 1]), "r"(o[i + 2]), "r"(o[i + 3]), "r"(o[i + 4]),
                                         "r"(o[i + 5]), "r"(o[i + 6]), "r"(o[i + 7])
                                         : "memory");
                    }
                    tc_fence_before();
                    __syncwarp();
                    if (lane == 0) mbar_arrive(&misc->o_free);
                    float *pml = p.part_ml + ((size_t)blockIdx.x * 2 + slot) * 2 * RB;
                    pml[r] = m;
                    pml[RB + r] = lrow;
                    __threadfence();
                    named_bar_sync(14, 128);   // the epilogue warpgroup
                    if (r == 0) {
                        const int c_first = cta_of_tile(sd.ib, T, NC);
                        const int c_last = cta_of_tile(sd.ie - 1, T, NC);
                        int npieces = 0;
                        for (int cc = c_first; cc <= c_last; ++cc)
                            npieces += cta_start(cc + 1, T, NC) > cta_start(cc, T, NC);
                        const unsigned old = atomicAdd(&p.item_cnt[sd.x], 1u);
                        misc->bcast = (old == (unsigned)(npieces - 1)) ? 1 : 0;
                        if (misc->bcast) p.item_cnt[sd.x] = 0u;  // ready for the next launch
                    }
                    named_bar_sync(14, 128);
                    if (misc->bcast) {
                        // last piece: merge every piece's (m, l, O row) by log-sum-exp
                        __threadfence();
                        const int c_first = cta_of_tile(sd.ib, T, NC);
                        const int c_last = cta_of_tile(sd.ie - 1, T, NC);
                        auto piece = [&](int cc) -> long long {   // partial slot of CTA cc's piece, -1 if empty
                            const int s0 = cta_start(cc, T, NC);
                            if (cta_start(cc + 1, T, NC) <= s0) return -1;
                            return ((long long)cc * p.lanes + cl) * 2 + ((s0 >= sd.ib) ? 0 : 1);
                        };
                        // (compact, rolled loops: this code runs cold in the instruction cache, once per item,
                        // and its length -- not its loads -- set the cost: ~350 ns per missed 128-B line)
                        if (sd.end == t1) {
                            // the CTA's last segment: K / V rings and Q buffers are idle -> stage the pieces with
                            // bulk copies (all in flight at once) instead of one L2 round trip per (piece, chunk):
                            // (m, l) of every piece, then up to `cap` 64 KB O blocks per round; each warp merges
                            // its 32 rows with lane = 4 dims (conflict-free, coalesced 256 B output rows)
                            uint8_t *area = smem;
                            const size_t area_bytes = (size_t)(NK + NV) * kSlotBytes + 2 * kQBuf;
                            constexpr uint32_t kOB = RB * kHeadDim * 4, kMLB = 2 * RB * 4;
                            int npc = 0;
                            for (int cc = c_first; cc <= c_last; ++cc) npc += piece(cc) >= 0;
                            float *sml = reinterpret_cast<float *>(area + area_bytes) - (size_t)npc * 3 * RB;  // [npc][m, l, w][RB]
                            const int cap = (int)(((size_t)((uint8_t *)sml - area)) / kOB);
                            uint32_t ph = 0;
                            if (r == 0) {
                                fence_proxy_async_global();
                                mbar_arrive_expect_tx(&misc->stage_bar, (uint32_t)npc * kMLB);
                                int k = 0;
                                for (int cc = c_first; cc <= c_last; ++cc) {
                                    const long long po2 = piece(cc);
                                    if (po2 < 0) continue;
                                    bulk_load_g2s(sml + (size_t)k * 3 * RB, p.part_ml + po2 * 2 * RB, kMLB, &misc->stage_bar);
                                    ++k;
                                }
                            }
                            mbar_wait(&misc->stage_bar, ph);
                            ph ^= 1u;
                            float Mx = -INFINITY, Ls = 0.f;
                            for (int k = 0; k < npc; ++k) Mx = fmaxf(Mx, sml[(size_t)k * 3 * RB + r]);
                            for (int k = 0; k < npc; ++k) {
                                const float mk = sml[(size_t)k * 3 * RB + r];
                                const float w = (mk == -INFINITY) ? 0.f : ex2(mk - Mx);
                                Ls += w * sml[(size_t)k * 3 * RB + RB + r];
                                sml[(size_t)k * 3 * RB + 2 * RB + r] = w;
                            }
                            const float inv = 1.0f / Ls;
                            for (int k = 0; k < npc; ++k) sml[(size_t)k * 3 * RB + 2 * RB + r] *= inv;
                            named_bar_sync(14, 128);   // weights visible to the whole group
                            // rows in 4 batches of 8 (registers: the epilogue warpgroup runs on a small budget);
                            // all pieces staged once when they fit the area, else re-staged per batch and round
                            const int wrow0 = qd * 32;   // this warp's rows
                            const bool one_round = npc <= cap;
#pragma unroll 1
                            for (int rb = 0; rb < 4; ++rb) {
                                float4 acc[8];   // [row of the batch] lane's 4 dims
#pragma unroll
                                for (int i = 0; i < 8; ++i) acc[i] = make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll 1
                                for (int k0 = 0; k0 < npc; k0 += cap) {
                                    const int kn = min(cap, npc - k0);
                                    if (rb == 0 || !one_round) {
                                        if (r == 0) {
                                            mbar_arrive_expect_tx(&misc->stage_bar, (uint32_t)kn * kOB);
                                            int k = 0;
                                            for (int cc = c_first; cc <= c_last; ++cc) {
                                                const long long po2 = piece(cc);
                                                if (po2 < 0) continue;
                                                if (k >= k0 && k < k0 + kn)
                                                    bulk_load_g2s(area + (size_t)(k - k0) * kOB, p.part_o + po2 * RB * kHeadDim,
                                                                  kOB, &misc->stage_bar);
                                                ++k;
                                            }
                                        }
                                        mbar_wait(&misc->stage_bar, ph);
                                        ph ^= 1u;
                                    }
#pragma unroll 1
                                    for (int k = 0; k < kn; ++k) {
                                        const float *blk = reinterpret_cast<const float *>(area + (size_t)k * kOB);
                                        const float *wk = sml + (size_t)(k0 + k) * 3 * RB + 2 * RB + wrow0 + rb * 8;
#pragma unroll
                                        for (int i = 0; i < 8; ++i) {
                                            const float4 x = *reinterpret_cast<const float4 *>(
                                                blk + (size_t)(wrow0 + rb * 8 + i) * kHeadDim + 4 * lane);
                                            const float w = wk[i];
                                            acc[i].x += w * x.x;
                                            acc[i].y += w * x.y;
                                            acc[i].z += w * x.z;
                                            acc[i].w += w * x.w;
                                        }
                                    }
                                    if (!one_round) named_bar_sync(14, 128);   // the staging area is reused
                                }
                                // rows of this batch: row wrow0 + rb * 8 + i -> its node / head (padding rows skipped)
#pragma unroll
                                for (int i = 0; i < 8; ++i) {
                                    const int rr = wrow0 + rb * 8 + i;
                                    const int nd = c * p.npc + rr / G, hh = rr % G;
                                    if (rr < rc && nd < n) {
                                        uint2 o2;
                                        o2.x = pack_bf16x2(acc[i].x, acc[i].y);
                                        o2.y = pack_bf16x2(acc[i].z, acc[i].w);
                                        *reinterpret_cast<uint2 *>(p.out + (((size_t)b * p.Nmax + nd) * p.Hq + g * G + hh) *
                                                                               kHeadDim + 4 * lane) = o2;
                                    }
                                }
                            }
                        } else {
                            float Mx = -INFINITY, Ls = 0.f;
#pragma unroll 1
                            for (int cc = c_first; cc <= c_last; ++cc) {
                                const long long po2 = piece(cc);
                                if (po2 < 0) continue;
                                const float mp = ldcg_f32(p.part_ml + po2 * 2 * RB + r);
                                const float lp = ldcg_f32(p.part_ml + po2 * 2 * RB + RB + r);
                                if (mp == -INFINITY) continue;
                                const float nM = fmaxf(Mx, mp);
                                Ls = (Mx == -INFINITY ? 0.f : Ls * ex2(Mx - nM)) + ex2(mp - nM) * lp;
                                Mx = nM;
                            }
                            const float inv = 1.0f / Ls;
                            __nv_bfloat16 *orow = p.out + (((size_t)b * p.Nmax + node) * p.Hq + g * G + hl) * kHeadDim;
#pragma unroll 1
                            for (int q2 = 0; q2 < 8; ++q2) {   // 16 dims at a time
                                float4 a0 = make_float4(0.f, 0.f, 0.f, 0.f), a1 = a0, a2 = a0, a3 = a0;
#pragma unroll 1
                                for (int cc = c_first; cc <= c_last; ++cc) {
                                    const long long po2 = piece(cc);
                                    if (po2 < 0) continue;
                                    const float mp = ldcg_f32(p.part_ml + po2 * 2 * RB + r);
                                    const float4 *src = reinterpret_cast<const float4 *>(
                                        p.part_o + (po2 * RB + r) * kHeadDim + q2 * 16);
                                    const float4 x0 = __ldcg(src), x1 = __ldcg(src + 1), x2 = __ldcg(src + 2),
                                                 x3 = __ldcg(src + 3);
                                    const float w = (mp == -INFINITY) ? 0.f : ex2(mp - Mx) * inv;
                                    a0.x += w * x0.x; a0.y += w * x0.y; a0.z += w * x0.z; a0.w += w * x0.w;
                                    a1.x += w * x1.x; a1.y += w * x1.y; a1.z += w * x1.z; a1.w += w * x1.w;
                                    a2.x += w * x2.x; a2.y += w * x2.y; a2.z += w * x2.z; a2.w += w * x2.w;
                                    a3.x += w * x3.x; a3.y += w * x3.y; a3.z += w * x3.z; a3.w += w * x3.w;
                                }
                                if (row_valid) {
                                    uint4 o4;
                                    o4.x = pack_bf16x2(a0.x, a0.y);
                                    o4.y = pack_bf16x2(a0.z, a0.w);
                                    o4.z = pack_bf16x2(a1.x, a1.y);
                                    o4.w = pack_bf16x2(a1.z, a1.w);
                                    *reinterpret_cast<uint4 *>(orow + q2 * 16) = o4;
                                    o4.x = pack_bf16x2(a2.x, a2.y);
                                    o4.y = pack_bf16x2(a2.z, a2.w);
                                    o4.z = pack_bf16x2(a3.x, a3.y);
                                    o4.w = pack_bf16x2(a3.z, a3.w);
                                    *reinterpret_cast<uint4 *>(orow + q2 * 16 + 8) = o4;
                                }
                            }
                        }
                    }

                }
                ++ls;
            }
        }
    } else if (warp >= 8) {
        // control warpgroup: its registers go to the softmax warps (all 4 warps execute this one
        // instruction; no code path below rejoins the softmax path)
        setmaxnreg_dec<kRegsCtl>();
        if (ntiles <= 0) {
            if (early) grid_dependency_wait();
        } else if (warp == kWarpProd || warp == kWarpV) {
            // ============================ TMA producers ============================
            // warp 8: segment descriptors, Q and the K ring; warp 11: the V ring (follows the descriptors)
            const uint64_t pol = (p.lanes > 1 || (p.dyn && p.chunks > 1)) ? l2_evict_normal_policy() : l2_evict_first_policy();
            auto issue = [&](const SegDesc &d, int t, int lt, bool is_v) {
                const int key0 = (t - d.ib) * kKeyTile;
                const int nv = min(kKeyTile, d.P + d.n - key0);
                const int row0 = kv_tile_row(p, d.b, d.g, key0);
                const int NS = is_v ? NV : NK;
                const int slot = lt % NS, f = lt / NS;
                if (f >= 1) mbar_wait(is_v ? &misc->v_empty[slot] : &misc->k_empty[slot], (f - 1) & 1);
                if (!is_v) {
                    SPI_TRACE(0);
                    if (lt == 0) SPI_TRACE_K(2);
                } else {
                    SPI_TRACE(1);
                }
                uint8_t *dst = (is_v ? s_v : s_k) + (size_t)slot * kSlotBytes;
                uint64_t *bar = is_v ? &misc->v_full[slot] : &misc->k_full[slot];
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
            };
            auto n_early = [&](const SegDesc &d, int NS) {
                int c = 0;
                while (c < NS && d.begin + c < d.end && (d.begin + c - d.ib + 1) * kKeyTile <= d.P) ++c;
                return c;
            };
            if (warp == kWarpProd && lane == 0 && p.dyn) {
                // dynamic mode: whole items; the first is item blockIdx.x, the next ones are claimed from the
                // ticket counter (after the dependency wait), each one while the current item streams.  Every
                // launch draws exactly n_items tickets (n_items - grid claims + one failing claim per CTA) and
                // launches draw in turn, so ticket t names item grid + t mod n_items (>= n_items: none left).
                bool waited = !early;
                auto claim = [&]() -> int {
                    if (!waited) {
                        grid_dependency_wait();
                        waited = true;
                    }
                    const uint32_t t = atomicAdd(p.dyn_ctr, 1u);
                    const int idx = (int)(t % (uint32_t)p.n_items) + (int)gridDim.x;
                    return idx < p.n_items ? idx : -1;
                };
                int dx = (int)blockIdx.x < p.n_items ? (int)blockIdx.x : -1;
                int ls = 0, lt = 0;
                for (;;) {
                    SegDesc d{};
                    d.x = -1;
                    while (dx >= 0) {
                        const int4 info = __ldg(p.item_info + dx);
                        if (info.y > info.x && info.w > 0) {
                            d.x = dx;
                            d.begin = d.ib = info.x;
                            d.end = d.ie = info.y;
                            d.c = dx % p.chunks;
                            d.g = (dx / p.chunks) % p.Hkv;
                            d.b = dx / (p.chunks * p.Hkv);
                            d.P = info.z;
                            d.n = info.w;
                            break;
                        }
                        dx = claim();   // an empty item (invalid tree / padding chunk)
                    }
                    misc->seg[ls % kSegRing] = d;
                    mbar_arrive(&misc->seg_full[ls % kSegRing]);
                    if (d.x < 0) {
                        if (!waited) grid_dependency_wait();
                        break;
                    }
                    int pre = 0;
                    if (!waited) {   // (early mode, first item: committed-prefix tiles before the wait)
                        pre = n_early(d, NK);
                        for (int i = 0; i < pre; ++i) issue(d, d.begin + i, i, false);
                        grid_dependency_wait();
                        waited = true;
                    }
                    dx = claim();   // the next item (the atomic's latency overlaps this item's loads)
                    const int qb = ls & 1;
                    if (ls >= 2) mbar_wait(&misc->q_empty[qb], ((ls >> 1) - 1) & 1);
                    mbar_arrive_expect_tx(&misc->q_full[qb], 2u * (uint32_t)(p.G * p.npc) * 128u);
                    uint8_t *qdst = s_q + qb * kQBuf;
                    const int node0 = d.b * p.Nmax + d.c * p.npc;
                    tma_load_3d(qdst, &tm_q, &misc->q_full[qb], 0, d.g * p.G, node0);
                    tma_load_3d(qdst + RB * 128, &tm_q, &misc->q_full[qb], 64, d.g * p.G, node0);
                    lt += pre;
                    for (int t = d.begin + pre; t < d.end; ++t, ++lt) issue(d, t, lt, false);
                    ++ls;
                }
                grid_launch_dependents();
            } else if (warp == kWarpProd && lane == 0) {
                int x = x_first, ls = 0, lt = 0;
                int4 next_info = first_info;
                for (;;) {
                    // next non-empty segment of this CTA's range (terminal descriptor if none)
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
                    misc->seg[ls % kSegRing] = d;
                    mbar_arrive(&misc->seg_full[ls % kSegRing]);
                    if (d.x < 0) {
                        if (early && ls == 0) grid_dependency_wait();
                        break;
                    }
                    int pre = 0;
                    if (early && ls == 0) {
                        pre = n_early(d, NK);
                        for (int i = 0; i < pre; ++i) issue(d, d.begin + i, i, false);
                        grid_dependency_wait();
                    }
                    const int qb = ls & 1;
                    if (ls >= 2) mbar_wait(&misc->q_empty[qb], ((ls >> 1) - 1) & 1);
                    mbar_arrive_expect_tx(&misc->q_full[qb], 2u * (uint32_t)(p.G * p.npc) * 128u);
                    uint8_t *qdst = s_q + qb * kQBuf;
                    const int node0 = d.b * p.Nmax + d.c * p.npc;
                    tma_load_3d(qdst, &tm_q, &misc->q_full[qb], 0, d.g * p.G, node0);
                    tma_load_3d(qdst + RB * 128, &tm_q, &misc->q_full[qb], 64, d.g * p.G, node0);
                    lt += pre;
                    for (int t = d.begin + pre; t < d.end; ++t, ++lt) issue(d, t, lt, false);
                    ++ls;
                }
                grid_launch_dependents();
            } else if (warp == kWarpV && lane == 0) {
                int ls = 0, lt = 0;
                for (;;) {
                    mbar_wait(&misc->seg_full[ls % kSegRing], (ls / kSegRing) & 1);
                    const SegDesc d = misc->seg[ls % kSegRing];
                    if (d.x < 0) {
                        if (early && ls == 0) grid_dependency_wait();
                        break;
                    }
                    int pre = 0;
                    if (early && ls == 0) {
                        pre = n_early(d, NV);
                        for (int i = 0; i < pre; ++i) issue(d, d.begin + i, i, true);
                        grid_dependency_wait();
                    }
                    lt += pre;
                    for (int t = d.begin + pre; t < d.end; ++t, ++lt) issue(d, t, lt, true);
                    ++ls;
                }
            }
        } else if (warp == kWarpS) {
            // ===================== S issuer: S(t) = Q K(t)^T into S buffer t & 1 =====================
            // (the buffer is free once the softmax of tile t - 2 has loaded it: s_free)
            if (lane == 0) {
                const uint32_t idesc_s = make_idesc_bf16(128, 128, false, false);
                const uint32_t k_addr = smem_u32(s_k), q_addr = smem_u32(s_q);
                int lt = 0, ls = 0;
                for (;;) {
                    mbar_wait(&misc->seg_full[ls % kSegRing], (ls / kSegRing) & 1);
                    const SegDesc d = misc->seg[ls % kSegRing];
                    if (d.x < 0) break;
                    const int qb = ls & 1;
                    mbar_wait(&misc->q_full[qb], (ls >> 1) & 1);
                    for (int t = d.begin; t < d.end; ++t, ++lt) {
                        const int sb = lt & 1;
                        if (lt >= 2) mbar_wait(&misc->s_free[sb], ((lt - 2) >> 1) & 1);
                        const int slot = lt % NK;
                        mbar_wait(&misc->k_full[slot], (lt / NK) & 1);
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
                            if (!(SPI_FLAGS(p) & 2))
                                umma_bf16_ss(tmem + kColS + sb * 128, adesc, bdesc, idesc_s, kk > 0 ? 1u : 0u);
                        }
                        umma_commit(&misc->s_full[sb]);
                        umma_commit(&misc->k_empty[slot]);
                        if (t == d.end - 1) umma_commit(&misc->q_empty[qb]);
                    }
                    ++ls;
                }
            }
        } else if (warp == kWarpPV) {
            // ============ PV issuer: O += P(t) V(t) (A = P from TMEM, N = 128 dims), in tile order ============
            if (lane == 0) {
                const uint32_t idesc_o = make_idesc_bf16(128, 128, false, true);
                const uint32_t v_addr = smem_u32(s_v);
                int lt = 0, ls = 0;
                for (;;) {
                    mbar_wait(&misc->seg_full[ls % kSegRing], (ls / kSegRing) & 1);
                    const SegDesc d = misc->seg[ls % kSegRing];
                    if (d.x < 0) break;
                    for (int t = d.begin; t < d.end; ++t, ++lt) {
                        const int pb = lt & 1;
                        mbar_wait(&misc->p_full[pb], (lt >> 1) & 1);
                        const bool first = (t == d.begin);
                        if (first && ls > 0) mbar_wait(&misc->o_free, (ls - 1) & 1);  // previous segment's O read
                        const int slot = lt % NV;
                        mbar_wait(&misc->v_full[slot], (lt / NV) & 1);
                        tc_fence_after();
                        SPI_TRACE(3);
                        const uint32_t vbase = v_addr + slot * kSlotBytes;
    #pragma unroll
                        for (int kk = 0; kk < kKeyTile / 16; ++kk) {
                            const uint64_t bdesc = make_smem_desc(vbase + kk * 16 * 128, kHalfBytes, 1024, kSw128);
                            if (!(SPI_FLAGS(p) & 2))
                                umma_bf16_ts(tmem + kColO, tmem + kColP + pb * 64 + kk * 8, bdesc, idesc_o,
                                             (first && kk == 0) ? 0u : 1u);
                        }
                        umma_commit(&misc->pv_done[pb]);
                        umma_commit(&misc->v_empty[slot]);
                        if (t == d.end - 1) umma_commit(&misc->o_full);   // the segment's O is final
                    }
                    ++ls;
                }
            }
        }
    } else {
        setmaxnreg_inc<kRegsSoftmax>();
        if (ntiles > 0) {
                // ====== softmax / epilogue: two groups of 4 warps on alternating tiles, ONE shared O ======
                // group g (warps 3 + 4g .. 6 + 4g) owns the tiles with lt & 1 == g; thread = one query row (TMEM
                // lane).  Both groups accumulate into the same O, so every P(t) must use the row reference the
                // previous tile left: the owner of tile t reads decision(t - 1) (the other group's, through
                // shared memory + a producer/consumer named barrier per lane quarter), may raise it (stale
                // max: only beyond 2^8, then O is rescaled after PV(t - 1)), publishes decision(t) and only then
                // computes its exponentials -- the groups run out of phase, so one group's loads / maxima /
                // handshake overlap the other's exponentials.  The owner of a segment's last tile writes the
                // rows (the other group hands over its partial row sums through shared memory).
                const int sw = warp;                   // 0..7
                const int grp = sw >> 2;               // tile parity owned by this group
                const int qd = warp & 3;               // TMEM lane quarter
                const int r = qd * 32 + lane;          // query row of the item = TMEM lane
                const uint32_t lane_off = (uint32_t)(qd * 32) << 16;
                // decision(t) hand-over between the two warps of quarter qd: one named barrier PER DIRECTION.
                // (With a single barrier, the publisher's arrive(t) and its own sync at tile t + 2 could complete
                // the barrier together whenever the other warp reached its sync for t + 1 late -- the publisher
                // would then read a stale reference.  Per direction, arrivals and syncs strictly alternate.)
                const uint32_t dec_out = grp == 0 ? 6 + qd : 1 + qd;   // the decisions this group publishes
                const uint32_t dec_in = grp == 0 ? 1 + qd : 6 + qd;    // the other group's decisions
                const uint32_t o_col = tmem + kColO + lane_off;
                float *mref_s = misc->mref;            // [row] the row reference after the latest decision
                int lt = 0, ls = 0;
                for (;;) {
                    mbar_wait(&misc->seg_full[ls % kSegRing], (ls / kSegRing) & 1);
                    const SegDesc sd = misc->seg[ls % kSegRing];
                    if (sd.x < 0) break;
                    const int b = sd.b, c = sd.c, P = sd.P, n = sd.n;
                    const int Kend = P + n;
                    const int G = p.G;
                    const int rc = G * p.npc;
                    const int node = c * p.npc + r / G;
                    const bool row_valid = (r < rc) && (node < n);
                    // ancestor-or-self bitset of this row's node, read on masked tiles only (rows without a
                    // node use node 0's root path, which keeps them finite; they are never written)
                    const uint32_t *anc = p.anc + ((size_t)b * p.Nmax + (row_valid ? node : 0)) * kBitWords;
                    // the masked (tree) tiles come last in a segment: pull the row's bitset into L1 now, so their
                    // __ldg's hit L1 instead of paying an L2 round trip on the softmax critical path
                    asm volatile("prefetch.global.L1 [%0];" ::"l"(anc));
                    float m = -INFINITY, l = 0.f;      // latest known row reference (log2 units), this group's sum
                    const int lt0 = lt;
                    for (int t = sd.begin; t < sd.end; ++t, ++lt) {
                        if ((lt & 1) != grp) continue;
                        const int sb = lt & 1;
                        const int key0 = (t - sd.ib) * kKeyTile;
                        mbar_wait(&misc->s_full[sb], (lt >> 1) & 1);
                        tc_fence_after();
                        if (r == 0) SPI_TRACE(4 + grp);
                        const uint32_t s_col = tmem + kColS + sb * 128 + lane_off;
                        // visibility of the tile's 128 keys (4 words): committed keys visible; tree keys by the
                        // ancestor bitset; keys past the request's end: none
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
                        // pass 1: this row's tile max
                        float tm;
                        uint32_t sv[4][32];   // the row's 128 scores stay in registers for pass 2
                        {
                            float m4[4] = {-INFINITY, -INFINITY, -INFINITY, -INFINITY};
#pragma unroll
                            for (int q = 0; q < 4; ++q) tmem_ld32(s_col + q * 32, sv[q]);
                            tmem_ld_wait();
                            // S buffer t & 1 is free now: S(t + 2) may overwrite it while this tile's softmax runs
                            tc_fence_before();
                            __syncwarp();
                            if (lane == 0) mbar_arrive(&misc->s_free[sb]);
#pragma unroll
                            for (int q = 0; q < 4; ++q) {
                                if (masked) rows::mask32(sv[q], vis[q]);
#pragma unroll
                                for (int i = 0; i < 32; ++i) m4[i & 3] = fmaxf(m4[i & 3], __uint_as_float(sv[q][i]));
                            }
                            tm = fmaxf(fmaxf(m4[0], m4[1]), fmaxf(m4[2], m4[3])) * p.scale_log2;
                        }
                        // decision(t - 1): the reference P(t - 1) used (ignored at a segment's first tile: new rows)
                        if (lt > 0) {
                            named_bar_sync(dec_in, 64);
                            const float mp = mref_s[r];
                            if (lt > lt0 && mp != m) {   // the other group raised it: rebase this group's sum
                                l = (m == -INFINITY) ? 0.f : l * ex2(m - mp);
                                m = mp;
                            }
                        }
                        if (r == 0) SPI_TRACE(8 + grp);
                        // decision(t): stale running max, moved only when this tile exceeds it by more than 2^8
                        float alpha = 1.f;
                        if (tm > m + kRescaleThreshold) {
                            alpha = (m == -INFINITY) ? 0.f : ex2(m - tm);
                            m = tm;
                            l *= alpha;
                        }
                        const bool moved = __any_sync(0xffffffffu, alpha != 1.f) && lt > lt0;
                        // O holds PV(<= t - 1) against the old reference: rescale it once PV(t - 1) completed and
                        // before PV(t) is issued (p_full).  This group last observed pv_done of ITS parity (PV(t - 4));
                        // the other barrier may still be a phase behind PV(t - 1)'s, which a parity wait cannot tell
                        // apart from "complete": first PV(t - 2) (own barrier, one phase ahead), which implies PV(t - 3).
                        auto rescale_o = [&]() {
                            if (lt >= 2) mbar_wait(&misc->pv_done[lt & 1], ((lt - 2) >> 1) & 1);
                            mbar_wait(&misc->pv_done[(lt - 1) & 1], ((lt - 1) >> 1) & 1);
                            tc_fence_after();
#pragma unroll 1
                            for (int q2 = 0; q2 < 4; ++q2) {
                                uint32_t v[32];
                                tmem_ld32(o_col + q2 * 32, v);
                                tmem_ld_wait();
                                uint32_t w16[16];
#pragma unroll
                                for (int hh = 0; hh < 2; ++hh) {
#pragma unroll
                                    for (int i = 0; i < 16; ++i) w16[i] = __float_as_uint(__uint_as_float(v[hh * 16 + i]) * alpha);
                                    tmem_st16(o_col + q2 * 32 + hh * 16, w16);
                                }
                            }
                        };
                        mref_s[r] = m;
                        named_bar_arrive(dec_out, 64);   // decision(t) -> the owner of tile t + 1
                        // pass 2: P(t) = 2^(s * scale - m) as bf16 pairs, row sum of the rounded values; every
                        // exponential is computed into registers first, and only the TMEM stores into P buffer t & 1
                        // wait for PV(t - 2) to have read it (that wait overlaps the exponentials)
                        {
                            const float mref = (m == -INFINITY) ? 0.f : m;
                            const uint64_t sc2 = f2_bits(p.scale_log2, p.scale_log2), nm2 = f2_bits(-mref, -mref);
                            const uint32_t p_col = tmem + kColP + sb * 64 + lane_off;
                            float ls2 = 0.f;
                            uint32_t w16[4][16];
#pragma unroll
                            for (int q = 0; q < 4; ++q) {
                                float dummy = 0.f;
                                ls2 += rows::exp32<false>(sv[q], sc2, nm2, w16[q], dummy);
                            }
                            if (lt >= 2) mbar_wait(&misc->pv_done[sb], ((lt - 2) >> 1) & 1);
                            tc_fence_after();
#pragma unroll
                            for (int q = 0; q < 4; ++q) tmem_st16(p_col + q * 16, w16[q]);
                            l += (SPI_FLAGS(p) & 8) ? 1.f : ls2;
                        }
                        if (moved) rescale_o();   // (the scores' registers are dead by now)
                        tmem_st_wait();
                        tc_fence_before();
                        __syncwarp();
                        if (lane == 0) mbar_arrive(&misc->p_full[sb]);
                        if (r == 0) SPI_TRACE(6 + grp);
                    }

                    // ============ end of this segment ============
                    // The non-owner group hands its (row sum, reference) to the owner of the segment's last tile
                    // through xl[segment & 1] (mbarriers: neither group blocks on the other here); the owner
                    // combines both and hands (row sum, reference) to the epilogue warpgroup, which reads O once
                    // the last PV completed.  Neither softmax group waits for that PV or touches O here.
                    const int llast = lt - 1;
                    const int owner = llast & 1;
                    const int fs = ls & 1;
                    if (grp != owner) {
                        if (ls >= 2) mbar_wait(&misc->xl_empty[fs], ((ls >> 1) - 1) & 1);
                        misc->xl[fs][0][r] = l;
                        misc->xl[fs][1][r] = m;
                        __syncwarp();
                        if (lane == 0) mbar_arrive(&misc->xl_full[fs]);
                    } else {
                        mbar_wait(&misc->xl_full[fs], (ls >> 1) & 1);
                        const float lo_ = misc->xl[fs][0][r], mo = misc->xl[fs][1][r];
                        __syncwarp();
                        if (lane == 0) mbar_arrive(&misc->xl_empty[fs]);
                        const float lrow = l + ((mo == -INFINITY || lo_ == 0.f) ? 0.f : lo_ * ex2(mo - m));
                        if (ls >= 2) mbar_wait(&misc->epi_empty[fs], ((ls >> 1) - 1) & 1);
                        misc->fin[fs][0][r] = lrow;
                        misc->fin[fs][1][r] = m;
                        __syncwarp();
                        if (lane == 0) mbar_arrive(&misc->epi_full[fs]);
                    }
                    ++ls;
                }
                // the last tile's decision has no next owner: consume it so every barrier phase completes
                if (lt > 0 && ((lt - 1) & 1) != grp) named_bar_sync(dec_in, 64);
        }
    }

    tc_fence_before();
    __syncthreads();
    if (warp == kWarpS) {
        tc_fence_after();
        tmem_dealloc<kTmemCols>(tmem);
    }
    if (threadIdx.x == 0) SPI_TRACE_K(1);
#ifdef SPECINFER_DEBUG_HOOKS
    if (threadIdx.x == 0 && SPI_TRACING(p)) {   // slot 3 (unused here): the SM this CTA ran on
        uint32_t smid;
        asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
        p.trace[(size_t)kTraceCtas * kTraceTiles * kTraceEv + blockIdx.x * 8 + 3] = smid + 1;
    }
#endif
}

static size_t rows_smem_bytes(int nk, int nv) {
    return (size_t)(nk + nv) * kSlotBytes + 2 * rows::kQBuf + sizeof(rows::Misc);
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
    // K ring 3 slots (K is released right after S), V ring 2 (held until PV); fewer if smem is short
    int nk = 3, nv = 2;
    while (rows_smem_bytes(nk, nv) > max_smem && nk + nv > 2) {
        if (nk > nv) --nk; else --nv;
    }
    if (rows_smem_bytes(nk, nv) > max_smem) return cudaErrorInvalidConfiguration;
    prm.nk_slots = nk;
    prm.nv_slots = nv;
    const size_t smem = rows_smem_bytes(nk, nv);
    {
        const cudaError_t e = ensure_max_smem_attr((const void *)tree_attn_rows_kernel, 3, max_smem);
        if (e != cudaSuccess) return e;
    }
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(num_ctas);
    cfg.blockDim = dim3(rows::kThreads);
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
