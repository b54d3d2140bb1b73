// tree_attention.cu — K2 tree attention for sm_100a.
//
// What it computes (Def. 4.1, Eq. 1-4; readings R1, R2,
// R20): for request b, kv-head g, every query row r = (node i, q-head g*G + hl):
//     out = sum_j softmax_j(sm_scale * q . k_j) v_j
// over the committed keys [0, P_b) and the tree keys P_b + a with a an ancestor-or-self of i
// (the topology-aware causal mask, one fused kernel for all tree tokens, L657-674).
//
// How (B200-first design):
//  * Work = the whole KV stream of one layer, B*Hkv items x ceil((P_b+n_b)/128) tiles of 128
//    keys, split evenly over a persistent grid (one CTA per SM) at tile granularity
//    (stream-K).  Items cut by a CTA boundary write fp32 partials (O, m, l) and the last piece
//    to finish merges them (log-sum-exp), so one launch per layer and no tail wave.
//  * Each KV tile is read from HBM once by TMA (128B-swizzled, 2 x 16 KB boxes per tile) into
//    a ring of 32 KB smem slots and shared by ALL G*n_b query rows of the kv-head.
//  * "Swapped" tensor-core formulation for few query rows: S^T = K Q^T (UMMA M = 128 keys,
//    N = NT query rows, K = 128 dims) and O^T += V^T P^T (M = 128 dims, N = NT, K = 128 keys),
//    tcgen05.mma kind::f16 issued by one thread, fp32 accumulators in TMEM.
//  * 4 softmax warps own one key (TMEM lane) each: fp32 scale + mask (ancestor bitsets from
//    tree_prepare) + exp2, P rounded to bf16 into smem (MN-major, swizzled) for the PV MMA.
//    Running row maxima are kept "stale" until a tile raises some row by more than 2^8
//    (exactly rescaled then, O^T rescaled in TMEM), so the common path needs no reduction
//    across lanes other than the row sums (transpose-reduce with warp shuffles).
//  * warp 0: TMA producer; warp 1: TMEM allocator + MMA issuer; warps 2-5: softmax/epilogue.
#include "common.cuh"

namespace specinfer {

struct AttnParams {
    const int32_t *prefix_len;
    const int32_t *n_nodes;
    const int32_t *item_start;
    uint32_t *item_cnt;
    const uint32_t *desc;
    float *part_o;
    float *part_ml;
    __nv_bfloat16 *out;
    int B, Nmax, Hq, Hkv, G, Smax, chunks, npc, n_items, num_slots;
    float scale_log2;
};

constexpr int kSlotBytes = kKeyTile * kHeadDim * 2;  // 32 KB: one K or V tile
constexpr int kHalfBytes = kSlotBytes / 2;            // 16 KB: 128 keys x 64 dims
constexpr int kTailRows = 16;                          // row granularity of partial tiles
constexpr float kRescaleThreshold = 8.0f;              // log2 units: stale max tolerance

template <int NT>
struct SmemPlan {
    static constexpr int kQBuf = 2 * NT * 128;         // one Q buffer: 2 halves x NT rows x 128 B
    static constexpr int kPBuf = kKeyTile * NT * 2;    // one P^T buffer: 128 keys x NT bf16
    static constexpr uint32_t kPSwizzle = NT == 64 ? kSw128 : (NT == 32 ? kSw64 : kSw32);
    static constexpr uint32_t kPMask = NT == 64 ? 7u : (NT == 32 ? 3u : 1u);
    static constexpr int kTmemCols = (3 * NT <= 32) ? 32 : (3 * NT <= 64 ? 64 : (3 * NT <= 128 ? 128 : 256));
};

struct SmemMisc {
    uint64_t slot_full[16];
    uint64_t slot_empty[16];
    uint64_t q_full[2], q_empty[2];
    uint64_t s_full[2], s_empty[2];
    uint64_t p_full[2], p_empty[2];
    uint32_t tmem_base;
    int32_t flags[2][4];
    int32_t bcast;
    alignas(16) float m_run[64];
    alignas(16) float alpha[64];
    alignas(16) float l_part[4][64];
    alignas(16) float wred[4][64];
};

// Iterates the (item, tile-range) segments of this CTA's contiguous tile range [t0, t1).
struct SegIter {
    const int32_t *item_start;
    int t0, t1, x;
    int begin, end, ib, ie;
    __device__ void init(const int32_t *is, int n_items, int t0_, int t1_) {
        item_start = is;
        t0 = t0_;
        t1 = t1_;
        // last item with start <= t0
        int lo = 0, hi = n_items;  // answer in [0, n_items)
        while (hi - lo > 1) {
            const int mid = (lo + hi) >> 1;
            if (item_start[mid] <= t0) lo = mid; else hi = mid;
        }
        x = lo - 1;
    }
    __device__ bool next() {
        for (;;) {
            ++x;
            ib = item_start[x];
            if (ib >= t1) return false;
            ie = item_start[x + 1];
            begin = max(t0, ib);
            end = min(t1, ie);
            if (end > begin) return true;
        }
    }
};

__device__ __forceinline__ int cta_start(long long c, long long T, long long NC) {
    return (int)((c * T) / NC);
}

__device__ __forceinline__ int cta_of_tile(int t, int T, int NC) {
    int c = (int)(((long long)t * NC) / T);
    if (c >= NC) c = NC - 1;
    while (c + 1 < NC && cta_start(c + 1, T, NC) <= t) ++c;
    while (c > 0 && cta_start(c, T, NC) > t) --c;
    return c;
}

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

template <int NT>
__global__ void __launch_bounds__(192, 1)
    tree_attn_kernel(const __grid_constant__ CUtensorMap tm_q, const __grid_constant__ CUtensorMap tm_k,
                     const __grid_constant__ CUtensorMap tm_v, const __grid_constant__ CUtensorMap tm_k16,
                     const __grid_constant__ CUtensorMap tm_v16, const AttnParams p) {
    using Plan = SmemPlan<NT>;
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    uint8_t *smem = reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
    const int NS = p.num_slots;
    uint8_t *s_slots = smem;
    uint8_t *s_q = s_slots + (size_t)NS * kSlotBytes;
    uint8_t *s_p = s_q + 2 * Plan::kQBuf;
    SmemMisc *misc = reinterpret_cast<SmemMisc *>(s_p + 2 * Plan::kPBuf);

    const int warp = threadIdx.x >> 5;
    const int lane = threadIdx.x & 31;

    const int T = p.item_start[p.n_items];
    const int NC = gridDim.x;
    const int t0 = cta_start(blockIdx.x, T, NC);
    const int t1 = cta_start(blockIdx.x + 1, T, NC);
    if (t1 <= t0) return;  // uniform across the CTA

    if (threadIdx.x == 0) {
        for (int i = 0; i < NS; ++i) {
            mbar_init(&misc->slot_full[i], 1);
            mbar_init(&misc->slot_empty[i], 1);
        }
        for (int i = 0; i < 2; ++i) {
            mbar_init(&misc->q_full[i], 1);
            mbar_init(&misc->q_empty[i], 1);
            mbar_init(&misc->s_full[i], 1);
            mbar_init(&misc->s_empty[i], 128);
            mbar_init(&misc->p_full[i], 4);
            mbar_init(&misc->p_empty[i], 1);
        }
        fence_barrier_init();
        fence_proxy_async_smem();
    }
    if (warp == 0 && lane == 0) {
        tma_prefetch_desc(&tm_q);
        tma_prefetch_desc(&tm_k);
        tma_prefetch_desc(&tm_v);
        tma_prefetch_desc(&tm_k16);
        tma_prefetch_desc(&tm_v16);
    }
    if (warp == 1) tmem_alloc<Plan::kTmemCols>(&misc->tmem_base);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem = misc->tmem_base;
    const uint32_t tm_S0 = tmem, tm_O = tmem + 2 * NT;

    SegIter it;
    it.init(p.item_start, p.n_items, t0, t1);

    if (warp == 0) {
        // ============================ TMA producer ============================
        if (lane == 0) {
            const uint64_t pol = l2_evict_first_policy();
            int lt = 0, ls = 0;
            while (it.next()) {
                const int x = it.x;
                const int c = x % p.chunks;
                const int g = (x / p.chunks) % p.Hkv;
                const int b = x / (p.chunks * p.Hkv);
                const int Kend = p.prefix_len[b] + p.n_nodes[b];
                const int qb = ls & 1;
                if (ls >= 2) mbar_wait(&misc->q_empty[qb], ((ls >> 1) - 1) & 1);
                const uint32_t qbytes = 2u * (uint32_t)(p.G * p.npc) * 128u;
                mbar_arrive_expect_tx(&misc->q_full[qb], qbytes);
                uint8_t *qdst = s_q + qb * Plan::kQBuf;
                const int node0 = b * p.Nmax + c * p.npc;
                tma_load_3d(qdst, &tm_q, &misc->q_full[qb], 0, g * p.G, node0);
                tma_load_3d(qdst + NT * 128, &tm_q, &misc->q_full[qb], 64, g * p.G, node0);
                const long long rowbase = (long long)(b * p.Hkv + g) * p.Smax;
                for (int t = it.begin; t < it.end; ++t, ++lt) {
                    const int key0 = (t - it.ib) * kKeyTile;
                    const int nv = min(kKeyTile, Kend - key0);
                    const int row0 = (int)(rowbase + key0);
#pragma unroll
                    for (int which = 0; which < 2; ++which) {
                        const int seq = 2 * lt + which;
                        const int slot = seq % NS;
                        const int f = seq / NS;
                        if (f >= 1) mbar_wait(&misc->slot_empty[slot], (f - 1) & 1);
                        uint8_t *dst = s_slots + (size_t)slot * kSlotBytes;
                        uint64_t *bar = &misc->slot_full[slot];
                        if (nv == kKeyTile) {
                            mbar_arrive_expect_tx(bar, kSlotBytes);
                            const CUtensorMap *m = which ? &tm_v : &tm_k;
                            tma_load_2d(dst, m, bar, 0, row0, pol);
                            tma_load_2d(dst + kHalfBytes, m, bar, 64, row0, pol);
                        } else {
                            const int nb = (nv + kTailRows - 1) / kTailRows;
                            mbar_arrive_expect_tx(bar, (uint32_t)nb * kTailRows * 128u * 2u);
                            const CUtensorMap *m = which ? &tm_v16 : &tm_k16;
                            for (int i = 0; i < nb; ++i) {
                                tma_load_2d(dst + i * kTailRows * 128, m, bar, 0, row0 + i * kTailRows, pol);
                                tma_load_2d(dst + kHalfBytes + i * kTailRows * 128, m, bar, 64,
                                            row0 + i * kTailRows, pol);
                            }
                        }
                    }
                }
                ++ls;
            }
        }
    } else if (warp == 1) {
        // ============================ MMA issuer ==============================
        if (lane == 0) {
            const uint32_t idesc_s = make_idesc_bf16(128, NT, false, false);
            const uint32_t idesc_o = make_idesc_bf16(128, NT, true, true);
            const uint32_t slots_addr = smem_u32(s_slots);
            const uint32_t q_addr = smem_u32(s_q);
            const uint32_t p_addr = smem_u32(s_p);
            int lt = 0, ls = 0;
            bool prev_first = false;  // tile lt-1 was the first of its segment
            auto issue_pv = [&](int u, bool first) {
                mbar_wait(&misc->p_full[u & 1], (u >> 1) & 1);
                const int seq = 2 * u + 1;
                const int slot = seq % NS;
                mbar_wait(&misc->slot_full[slot], (seq / NS) & 1);
                tc_fence_after();
                const uint32_t vbase = slots_addr + slot * kSlotBytes;
                const uint32_t pbase = p_addr + (u & 1) * Plan::kPBuf;
#pragma unroll
                for (int kk = 0; kk < kKeyTile / 16; ++kk) {
                    const uint64_t adesc = make_smem_desc(vbase + kk * 16 * 128, kHalfBytes, 1024, kSw128);
                    const uint64_t bdesc = make_smem_desc(pbase + kk * 16 * (NT * 2), Plan::kPBuf,
                                                          8 * NT * 2, Plan::kPSwizzle);
                    umma_bf16_ss(tm_O, adesc, bdesc, idesc_o, (first && kk == 0) ? 0u : 1u);
                }
                umma_commit(&misc->p_empty[u & 1]);
                umma_commit(&misc->slot_empty[slot]);
            };
            while (it.next()) {
                const int qb = ls & 1;
                mbar_wait(&misc->q_full[qb], (ls >> 1) & 1);
                for (int t = it.begin; t < it.end; ++t, ++lt) {
                    const int seq = 2 * lt;
                    const int slot = seq % NS;
                    mbar_wait(&misc->slot_full[slot], (seq / NS) & 1);
                    const int sb = lt & 1;
                    if (lt >= 2) mbar_wait(&misc->s_empty[sb], ((lt - 2) >> 1) & 1);
                    tc_fence_after();
                    const uint32_t kbase = slots_addr + slot * kSlotBytes;
                    const uint32_t qbase = q_addr + qb * Plan::kQBuf;
#pragma unroll
                    for (int kk = 0; kk < kHeadDim / 16; ++kk) {
                        const uint32_t koff = (kk >> 2) * kHalfBytes + (kk & 3) * 32;
                        const uint32_t qoff = (kk >> 2) * (NT * 128) + (kk & 3) * 32;
                        const uint64_t adesc = make_smem_desc(kbase + koff, 16, 1024, kSw128);
                        const uint64_t bdesc = make_smem_desc(qbase + qoff, 16, 1024, kSw128);
                        umma_bf16_ss(tm_S0 + sb * NT, adesc, bdesc, idesc_s, kk > 0 ? 1u : 0u);
                    }
                    umma_commit(&misc->s_full[sb]);
                    umma_commit(&misc->slot_empty[slot]);
                    if (t == it.end - 1) umma_commit(&misc->q_empty[qb]);
                    if (lt >= 1) issue_pv(lt - 1, prev_first);
                    prev_first = (t == it.begin);
                }
                ++ls;
            }
            if (lt >= 1) issue_pv(lt - 1, prev_first);
        }
    } else {
        // ======================= softmax / epilogue warps =======================
        const int st = threadIdx.x - 64;       // 0..127
        const int qd = warp & 3;               // TMEM lane quarter of this warp
        const int kt = qd * 32 + lane;         // key within tile (S^T lane) / head dim (O^T lane)
        const uint32_t lane_off = (uint32_t)(qd * 32) << 16;
        int lt = 0;
        while (it.next()) {
            const int x = it.x;
            const int c = x % p.chunks;
            const int g = (x / p.chunks) % p.Hkv;
            const int b = x / (p.chunks * p.Hkv);
            const int P = p.prefix_len[b];
            const int n = p.n_nodes[b];
            const int Kend = P + n;
            const int node0 = c * p.npc;
            const int G = p.G;
            const int rc = G * p.npc;               // rows used in this chunk
            // rows whose node exists
            uint64_t row_valid = 0;
            for (int r = 0; r < rc; ++r)
                if (node0 + r / G < n) row_valid |= 1ull << r;
            // reset row statistics
            if (qd == 0) {
                for (int r = lane; r < NT; r += 32) misc->m_run[r] = -INFINITY;
            }
            for (int r = lane; r < NT; r += 32) misc->l_part[qd][r] = 0.f;
            named_bar_sync(1, 128);

            for (int t = it.begin; t < it.end; ++t, ++lt) {
                const int key0 = (t - it.ib) * kKeyTile;
                const int kk = key0 + kt;
                const int sb = lt & 1;
                // ---- S^T row of this key ----
                mbar_wait(&misc->s_full[sb], (lt >> 1) & 1);
                tc_fence_after();
                float xv[NT];
                {
                    uint32_t r16[16];
#pragma unroll
                    for (int c16 = 0; c16 < NT / 16; ++c16) {
                        tmem_ld16(tm_S0 + sb * NT + c16 * 16 + lane_off, r16);
                        tmem_ld_wait();
#pragma unroll
                        for (int i = 0; i < 16; ++i) xv[c16 * 16 + i] = __uint_as_float(r16[i]);
                    }
                }
                tc_fence_before();
                mbar_arrive(&misc->s_empty[sb]);
                // ---- mask + scale ----
                uint64_t vis;
                if (kk < P) {
                    vis = row_valid;
                } else if (kk < Kend) {
                    const int j = kk - P;
                    const uint4 *dp = reinterpret_cast<const uint4 *>(p.desc + ((size_t)b * p.Nmax + j) * kBitWords);
                    const uint4 d0 = __ldg(dp), d1 = __ldg(dp + 1);
                    const uint32_t dw[8] = {d0.x, d0.y, d0.z, d0.w, d1.x, d1.y, d1.z, d1.w};
                    uint64_t m = 0;
                    for (int nd = 0; nd < p.npc; ++nd) {
                        const int node = node0 + nd;
                        if (node < kMaxNodes && ((dw[node >> 5] >> (node & 31)) & 1u)) {
                            const uint64_t run = (G >= 64) ? ~0ull : ((1ull << G) - 1ull);
                            m |= run << (nd * G);
                        }
                    }
                    vis = m & row_valid;
                } else {
                    vis = 0;
                }
#pragma unroll
                for (int r = 0; r < NT; ++r)
                    xv[r] = ((vis >> r) & 1ull) ? xv[r] * p.scale_log2 : -INFINITY;
                // ---- does this tile raise some row max beyond the stale tolerance? ----
                bool need = false;
#pragma unroll
                for (int r = 0; r < NT; r += 4) {
                    const float4 m4 = *reinterpret_cast<const float4 *>(&misc->m_run[r]);
                    need |= xv[r] > m4.x + kRescaleThreshold;
                    need |= xv[r + 1] > m4.y + kRescaleThreshold;
                    need |= xv[r + 2] > m4.z + kRescaleThreshold;
                    need |= xv[r + 3] > m4.w + kRescaleThreshold;
                }
                const unsigned ballot = __ballot_sync(0xffffffffu, need);
                if (lane == 0) misc->flags[sb][qd] = ballot != 0u;
                named_bar_sync(1, 128);
                const bool rescale = (misc->flags[sb][0] | misc->flags[sb][1] | misc->flags[sb][2] |
                                      misc->flags[sb][3]) != 0;
                if (rescale) {
                    // exact tile max per row: transpose-reduce within the warp, combine 4 warps
                    float mx[NT];
#pragma unroll
                    for (int r = 0; r < NT; ++r) mx[r] = xv[r];
#pragma unroll
                    for (int blk = 0; blk < (NT + 31) / 32; ++blk) {
                        constexpr int W = NT < 32 ? NT : 32;
                        transpose_reduce<W, true>(mx + blk * 32);
                        const int row = blk * 32 + (lane & (W - 1));
                        if (lane < W) misc->wred[qd][row] = mx[blk * 32];
                    }
                    named_bar_sync(1, 128);
                    if (qd == 0) {
                        for (int r = lane; r < NT; r += 32) {
                            const float tm = fmaxf(fmaxf(misc->wred[0][r], misc->wred[1][r]),
                                                   fmaxf(misc->wred[2][r], misc->wred[3][r]));
                            const float mo = misc->m_run[r];
                            const float mn = fmaxf(mo, tm);
                            misc->alpha[r] = (mo == -INFINITY) ? 0.f : ex2(mo - mn);
                            misc->m_run[r] = mn;
                        }
                    }
                    named_bar_sync(1, 128);
                    for (int r = lane; r < NT; r += 32) misc->l_part[qd][r] *= misc->alpha[r];
                    if (t != it.begin) {
                        // O^T columns (rows of Q) scaled by alpha: wait for PV of tile lt-1
                        mbar_wait(&misc->p_empty[(lt - 1) & 1], ((lt - 1) >> 1) & 1);
                        tc_fence_after();
                        uint32_t r16[16];
#pragma unroll
                        for (int c16 = 0; c16 < NT / 16; ++c16) {
                            tmem_ld16(tm_O + c16 * 16 + lane_off, r16);
                            tmem_ld_wait();
#pragma unroll
                            for (int i = 0; i < 16; ++i)
                                r16[i] = __float_as_uint(__uint_as_float(r16[i]) * misc->alpha[c16 * 16 + i]);
                            tmem_st16(tm_O + c16 * 16 + lane_off, r16);
                        }
                        tmem_st_wait();
                    }
                }
                // ---- probabilities (bf16) ----
#pragma unroll
                for (int r = 0; r < NT; r += 4) {
                    const float4 m4 = *reinterpret_cast<const float4 *>(&misc->m_run[r]);
                    const float mr[4] = {m4.x, m4.y, m4.z, m4.w};
#pragma unroll
                    for (int i = 0; i < 4; ++i) {
                        const float ref = (mr[i] == -INFINITY) ? 0.f : mr[i];
                        const float e = ex2(xv[r + i] - ref);
                        xv[r + i] = __bfloat162float(__float2bfloat16_rn(e));
                    }
                }
                // V rows of keys beyond the request's last key must be finite zeros (0 * NaN)
                if (kk >= Kend) {
                    const int seq = 2 * lt + 1;
                    const int slot = seq % NS;
                    mbar_wait(&misc->slot_full[slot], (seq / NS) & 1);
                    uint4 *v0 = reinterpret_cast<uint4 *>(s_slots + (size_t)slot * kSlotBytes + kt * 128);
                    uint4 *v1 = reinterpret_cast<uint4 *>(s_slots + (size_t)slot * kSlotBytes + kHalfBytes + kt * 128);
#pragma unroll
                    for (int i = 0; i < 8; ++i) {
                        v0[i] = make_uint4(0, 0, 0, 0);
                        v1[i] = make_uint4(0, 0, 0, 0);
                    }
                }
                // ---- P^T row (this key) into smem, MN-major + swizzle ----
                if (lt >= 2) mbar_wait(&misc->p_empty[sb], ((lt - 2) >> 1) & 1);
                {
                    uint8_t *pb = s_p + sb * Plan::kPBuf;
#pragma unroll
                    for (int c8 = 0; c8 < NT / 8; ++c8) {
                        const uint32_t o = (uint32_t)kt * (NT * 2) + c8 * 16;
                        const uint32_t phys = o ^ (((o >> 7) & Plan::kPMask) << 4);
                        uint4 v;
                        v.x = pack_bf16x2(xv[c8 * 8 + 0], xv[c8 * 8 + 1]);
                        v.y = pack_bf16x2(xv[c8 * 8 + 2], xv[c8 * 8 + 3]);
                        v.z = pack_bf16x2(xv[c8 * 8 + 4], xv[c8 * 8 + 5]);
                        v.w = pack_bf16x2(xv[c8 * 8 + 6], xv[c8 * 8 + 7]);
                        *reinterpret_cast<uint4 *>(pb + phys) = v;
                    }
                }
                fence_proxy_async_smem();
                tc_fence_before();
                __syncwarp();
                if (lane == 0) mbar_arrive(&misc->p_full[sb]);
                // ---- row sums of this tile (in key order over the 4 warps) ----
#pragma unroll
                for (int blk = 0; blk < (NT + 31) / 32; ++blk) {
                    constexpr int W = NT < 32 ? NT : 32;
                    transpose_reduce<W, false>(xv + blk * 32);
                    const int row = blk * 32 + (lane & (W - 1));
                    if (lane < W) misc->l_part[qd][row] += xv[blk * 32];
                }

                if (t == it.end - 1) {
                    // ============ epilogue of this segment ============
                    mbar_wait(&misc->p_empty[sb], (lt >> 1) & 1);  // last PV done
                    tc_fence_after();
                    float o[NT];
                    {
                        uint32_t r16[16];
#pragma unroll
                        for (int c16 = 0; c16 < NT / 16; ++c16) {
                            tmem_ld16(tm_O + c16 * 16 + lane_off, r16);
                            tmem_ld_wait();
#pragma unroll
                            for (int i = 0; i < 16; ++i) o[c16 * 16 + i] = __uint_as_float(r16[i]);
                        }
                    }
                    tc_fence_before();
                    named_bar_sync(1, 128);  // all l_part updates visible
                    const int d = kt;
                    const bool full = (it.begin == it.ib) && (it.end == it.ie);
                    if (full) {
#pragma unroll
                        for (int r = 0; r < NT; ++r) {
                            if (!((row_valid >> r) & 1ull)) continue;
                            const float l = misc->l_part[0][r] + misc->l_part[1][r] + misc->l_part[2][r] + misc->l_part[3][r];
                            const int node = node0 + r / G, hl = r % G;
                            p.out[(((size_t)b * p.Nmax + node) * p.Hq + g * G + hl) * kHeadDim + d] =
                                __float2bfloat16_rn(o[r] / l);
                        }
                    } else {
                        const int slot = (it.begin == t0) ? 0 : 1;
                        float *po = p.part_o + (((size_t)blockIdx.x * 2 + slot) * NT) * kHeadDim;
#pragma unroll
                        for (int r = 0; r < NT; ++r) po[(size_t)r * kHeadDim + d] = o[r];
                        float *pml = p.part_ml + ((size_t)blockIdx.x * 2 + slot) * 2 * NT;
                        if (st < NT) {
                            pml[st] = misc->m_run[st];
                            pml[NT + st] = misc->l_part[0][st] + misc->l_part[1][st] + misc->l_part[2][st] + misc->l_part[3][st];
                        }
                        __threadfence();
                        named_bar_sync(1, 128);
                        if (st == 0) {
                            const int c_first = cta_of_tile(it.ib, T, NC);
                            const int c_last = cta_of_tile(it.ie - 1, T, NC);
                            int npieces = 0;
                            for (int cc = c_first; cc <= c_last; ++cc)
                                npieces += cta_start(cc + 1, T, NC) > cta_start(cc, T, NC);
                            const unsigned old = atomicAdd(&p.item_cnt[x], 1u);
                            misc->bcast = (old == (unsigned)(npieces - 1)) ? 1 : 0;
                            if (misc->bcast) p.item_cnt[x] = 0u;  // ready for the next launch
                        }
                        named_bar_sync(1, 128);
                        if (misc->bcast) {
                            __threadfence();
                            const int c_first = cta_of_tile(it.ib, T, NC);
                            const int c_last = cta_of_tile(it.ie - 1, T, NC);
                            for (int r = 0; r < NT; ++r) {
                                if (!((row_valid >> r) & 1ull)) continue;
                                float M = -INFINITY;
                                for (int cc = c_first; cc <= c_last; ++cc) {
                                    const int s0 = cta_start(cc, T, NC);
                                    if (cta_start(cc + 1, T, NC) <= s0) continue;
                                    const int sl = (s0 >= it.ib) ? 0 : 1;
                                    M = fmaxf(M, ldcg_f32(p.part_ml + ((size_t)cc * 2 + sl) * 2 * NT + r));
                                }
                                float L = 0.f, O = 0.f;
                                for (int cc = c_first; cc <= c_last; ++cc) {
                                    const int s0 = cta_start(cc, T, NC);
                                    if (cta_start(cc + 1, T, NC) <= s0) continue;
                                    const int sl = (s0 >= it.ib) ? 0 : 1;
                                    const float *pm = p.part_ml + ((size_t)cc * 2 + sl) * 2 * NT;
                                    const float mp = ldcg_f32(pm + r);
                                    if (mp == -INFINITY) continue;
                                    const float w = ex2(mp - M);
                                    L += w * ldcg_f32(pm + NT + r);
                                    O += w * ldcg_f32(p.part_o + (((size_t)cc * 2 + sl) * NT + r) * kHeadDim + d);
                                }
                                const int node = node0 + r / G, hl = r % G;
                                p.out[(((size_t)b * p.Nmax + node) * p.Hq + g * G + hl) * kHeadDim + d] =
                                    __float2bfloat16_rn(O / L);
                            }
                        }
                    }
                    named_bar_sync(1, 128);  // stats read by everyone before the next reset
                }
            }
        }
    }

    tc_fence_before();
    __syncthreads();
    if (warp == 1) {
        tc_fence_after();
        tmem_dealloc<Plan::kTmemCols>(tmem);
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

template <int NT>
static size_t attn_smem_bytes(int num_slots) {
    using Plan = SmemPlan<NT>;
    return 1024 + (size_t)num_slots * kSlotBytes + 2 * Plan::kQBuf + 2 * Plan::kPBuf + sizeof(SmemMisc);
}

template <int NT>
static int pick_slots(size_t max_smem) {
    int ns = 16;
    while (ns > 2 && attn_smem_bytes<NT>(ns) > max_smem) --ns;
    return ns;
}

template <int NT>
static cudaError_t launch_nt(const AttnParams &prm0, const void *q, const void *k, const void *v,
                             int num_sms, size_t max_smem, cudaStream_t stream) {
    AttnParams prm = prm0;
    CUtensorMap tq, tk, tv, tk16, tv16;
    const uint64_t rows = (uint64_t)prm.B * prm.Hkv * prm.Smax;
    if (!encode_q(&tq, q, prm.Hq, (uint64_t)prm.B * prm.Nmax, prm.G, prm.npc) ||
        !encode_2d(&tk, k, rows, kKeyTile) || !encode_2d(&tv, v, rows, kKeyTile) ||
        !encode_2d(&tk16, k, rows, kTailRows) || !encode_2d(&tv16, v, rows, kTailRows))
        return cudaErrorInvalidValue;
    prm.num_slots = pick_slots<NT>(max_smem);
    const size_t smem = attn_smem_bytes<NT>(prm.num_slots);
    static bool attr_set = false;
    if (!attr_set) {
        cudaError_t e = cudaFuncSetAttribute(tree_attn_kernel<NT>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                             (int)max_smem);
        if (e != cudaSuccess) return e;
        attr_set = true;
    }
    tree_attn_kernel<NT><<<num_sms, 192, smem, stream>>>(tq, tk, tv, tk16, tv16, prm);
    return cudaGetLastError();
}

cudaError_t launch_tree_attention(const specinfer_shape_t &s, const WsLayout &w, const void *q,
                                  const void *k, const void *v, const int32_t *prefix_len,
                                  const int32_t *n_nodes, void *out, char *ws, int num_sms,
                                  size_t max_smem, cudaStream_t stream) {
    AttnParams prm{};
    prm.prefix_len = prefix_len;
    prm.n_nodes = n_nodes;
    prm.item_start = reinterpret_cast<const int32_t *>(ws + w.item_start);
    prm.item_cnt = reinterpret_cast<uint32_t *>(ws + w.item_cnt);
    prm.desc = reinterpret_cast<const uint32_t *>(ws + w.desc);
    prm.part_o = reinterpret_cast<float *>(ws + w.part_o);
    prm.part_ml = reinterpret_cast<float *>(ws + w.part_ml);
    prm.out = reinterpret_cast<__nv_bfloat16 *>(out);
    prm.B = s.batch;
    prm.Nmax = s.max_nodes;
    prm.Hq = s.num_q_heads;
    prm.Hkv = s.num_kv_heads;
    prm.G = s.num_q_heads / s.num_kv_heads;
    prm.Smax = s.max_seq;
    prm.chunks = w.chunks;
    prm.npc = w.npc;
    prm.n_items = w.n_items;
    const float sm_scale = s.sm_scale > 0.f ? s.sm_scale : 1.0f / sqrtf((float)s.head_dim);
    prm.scale_log2 = sm_scale * 1.4426950408889634f;
    const int grid = num_sms;  // persistent: one CTA per SM
    switch (w.nt) {
        case 16: return launch_nt<16>(prm, q, k, v, grid, max_smem, stream);
        case 32: return launch_nt<32>(prm, q, k, v, grid, max_smem, stream);
        default: return launch_nt<64>(prm, q, k, v, grid, max_smem, stream);
    }
}

}  // namespace specinfer
