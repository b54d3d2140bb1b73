// tree_attention.cu — K2 tree attention for sm_100a.
//
// What it computes (Def. 4.1, Eq. 1-4; readings R1, R2,
// R20): for request b, kv-head g, every query row r = (node i, q-head g*G + hl):
//     out = sum_j softmax_j(sm_scale * q . k_j) v_j
// over the committed keys [0, P_b) and the tree keys P_b + a with a an ancestor-or-self of i
// (the topology-aware causal mask, one fused kernel for all tree tokens, L657-674).
//
// How (B200-first design):
//  * Work = the whole KV stream of one layer: items (b, kv-head, row chunk) x ceil((P_b+n_b)/128)
//    tiles of 128 keys, split evenly over a persistent grid (one CTA per SM) at tile
//    granularity (stream-K).  Items cut by a CTA boundary write fp32 partials (O, m, l); the
//    last piece to finish merges them (log-sum-exp): one launch per layer, no tail wave.
//  * Each KV tile is read from HBM once by TMA (128B-swizzled 16 KB boxes) and shared by ALL
//    G*n_b query rows of the kv-head.  K and V have separate smem rings (K tiles are released
//    right after S = K Q^T, so K prefetch never waits for a PV), fed by two producer warps.
//  * "Swapped" tensor-core formulation for few query rows: S^T = K Q^T (UMMA M = 128 keys,
//    N = NT query rows, K = 128 dims) and O^T += V^T P^T (M = 128 dims, N = NT, K = 128 keys);
//    tcgen05.mma kind::f16 issued by one thread, fp32 accumulators in TMEM.
//  * 4 softmax warps own one key (TMEM lane) each: fp32 scale, tree mask (row masks from
//    tree_prepare; committed keys need none), exp2, P rounded to bf16 into smem (MN-major,
//    swizzled) for the PV MMA, row sums kept per thread and reduced once per segment.  The
//    running row maxima stay "stale" until a tile raises a row by more than 2^8; then they are
//    recomputed exactly and O^T is rescaled in TMEM (the rare path).
//  * Segment metadata is decoded once by the producer and passed through an smem ring, so no
//    consumer waits on a global load at item boundaries.
//  * warp 0: Q + K + segment ring producer; warp 1: TMEM allocator + S issuer; warp 2: PV issuer;
//    warps 3 .. (8 at NT >= 32, 4 at NT = 16): softmax / epilogue / split combine; last warp: V producer.
#include "attn_shared.cuh"

#include <cooperative_groups.h>

namespace specinfer {

template <int NT>
struct SmemPlan {
    static constexpr int kQBuf = 2 * NT * 128;         // one Q buffer: 2 halves x NT rows x 128 B
    static constexpr int kNQ = 2;                      // Q buffers (segment s uses s % kNQ)
    static constexpr int kPBuf = kKeyTile * NT * 2;    // one P^T buffer: 128 keys x NT bf16
    // P^T buffers: two (softmax(t) overlaps PV(t-1)) except at NT = 64, where the second 16 KB
    // would cost a K/V ring slot (measured: width-5 C2 tree 1% slower with two)
    static constexpr int kNP = NT == 64 ? 1 : 2;
    static constexpr uint32_t kPSwizzle = NT == 64 ? kSw128 : (NT == 32 ? kSw64 : kSw32);
    static constexpr uint32_t kPMask = NT == 64 ? 7u : (NT == 32 ? 3u : 1u);
    static constexpr int kTmemCols = (3 * NT <= 32) ? 32 : (3 * NT <= 64 ? 64 : (3 * NT <= 128 ? 128 : 256));
};

struct SmemMisc {
    uint64_t k_full[kMaxSlots], k_empty[kMaxSlots];
    uint64_t v_full[kMaxSlots], v_empty[kMaxSlots];
    uint64_t q_full[2], q_empty[2];
    uint64_t s_full[2], s_empty[2];
    uint64_t p_full[2], p_empty[2];  // P^T buffers: tile lt uses buffer lt % kNP, free once PV(lt-kNP) read it
    uint64_t cmb_bar;          // bulk staging of the split pieces (at most one merge per CTA uses it)
    uint64_t seg_full[kSegRing];
    SegDesc seg[kSegRing];
    uint32_t tmem_base;
    int32_t bcast;
    alignas(16) float m_thr[64];   // running row max + threshold (-inf: no key seen yet)
    alignas(16) float m_ref[64];   // running row max used as exp2 reference (0 if none yet)
    alignas(16) float alpha[64];
    alignas(16) float l_part[4][64];
    alignas(16) float wred[4][64];
    // split-combine state (the per-piece staging arrays live in the idle P^T buffer)
    alignas(16) float run_m[64];
    alignas(16) float run_l[64];
    size_t piece_off[kCombineBatch];
    int32_t npieces;
};

// warp roles: 0 Q / K producer, 1 S issuer (+ TMEM allocation), 2 PV issuer, 3 .. 3 + kSoft / 32 - 1
// softmax / epilogue, last: V producer (its own warp: as a second lane of warp 0, a lane spinning on
// one ring's empty barrier held the other ring's lane at the warp's divergence point -- at batch 2
// K and V loads were issued 1-2K cycles after their slots freed)
template <int NT>
struct SwRoles {
    static constexpr int kSoftWarps = NT >= 32 ? 8 : 4;
    static constexpr int kWarpV = 3 + kSoftWarps;
    static constexpr int kThreads = 32 * (kWarpV + 1);
};

template <int NT>
__global__ void __launch_bounds__(SwRoles<NT>::kThreads, 1)
    tree_attn_kernel(const __grid_constant__ CUtensorMap tm_q, const __grid_constant__ CUtensorMap tm_k,
                     const __grid_constant__ CUtensorMap tm_v, const __grid_constant__ CUtensorMap tm_k16,
                     const __grid_constant__ CUtensorMap tm_v16, const __grid_constant__ CUtensorMap tm_k4,
                     const __grid_constant__ CUtensorMap tm_v4, const __grid_constant__ CUtensorMap tm_k1,
                     const __grid_constant__ CUtensorMap tm_v1, const AttnParams p) {
    using Plan = SmemPlan<NT>;
    // NT >= 32: 8 softmax warps, two per TMEM lane quarter, each owning half of the query rows
    // (columns of S^T) of its key: half the registers and two warps per SMSP to hide latency
    constexpr int kSplit = NT >= 32 ? 2 : 1;
    constexpr int NTH = NT / kSplit;  // query rows per softmax thread
    constexpr int kSoft = 128 * kSplit;
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    // keep the pointer derived from smem_raw so the compiler emits LDS/STS, not generic LD/ST
    uint8_t *smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
    const int NK = p.nk_slots, NV = p.nv_slots;
    uint8_t *s_k = smem;
    uint8_t *s_v = s_k + (size_t)NK * kSlotBytes;
    uint8_t *s_q = s_v + (size_t)NV * kSlotBytes;
    uint8_t *s_p = s_q + Plan::kNQ * Plan::kQBuf;
    SmemMisc *misc = reinterpret_cast<SmemMisc *>(s_p + Plan::kNP * Plan::kPBuf);

    const int warp = threadIdx.x >> 5;
    const int lane = threadIdx.x & 31;

    if (threadIdx.x == 0) SPI_TRACE_K(0);
    const int NC = gridDim.x;
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
            mbar_init(&misc->s_empty[i], 4 * kSplit);
        }
        for (int i = 0; i < Plan::kNP; ++i) {
            mbar_init(&misc->p_full[i], 4 * kSplit);
            mbar_init(&misc->p_empty[i], 1);
        }
        mbar_init(&misc->cmb_bar, 1);
        for (int i = 0; i < kSegRing; ++i) mbar_init(&misc->seg_full[i], 1);
        fence_barrier_init();
    }
    if (warp == 0 && lane == 0) {
        tma_prefetch_desc(&tm_q);
        tma_prefetch_desc(&tm_k);
        tma_prefetch_desc(&tm_v);
        tma_prefetch_desc(&tm_k16);
        tma_prefetch_desc(&tm_v16);
        tma_prefetch_desc(&tm_k4);
        tma_prefetch_desc(&tm_v4);
        tma_prefetch_desc(&tm_k1);
        tma_prefetch_desc(&tm_v1);
    }
    constexpr int kWarpV = SwRoles<NT>::kWarpV;
    const bool softw = warp >= 3 && warp < kWarpV;   // softmax / epilogue warp
    if (softw) {
        // Q rows beyond a chunk's G*npc rows are never written by TMA: keep them zero
        for (int i = threadIdx.x - 96; i < Plan::kNQ * Plan::kQBuf / 16; i += kSoft)
            reinterpret_cast<uint4 *>(s_q)[i] = make_uint4(0, 0, 0, 0);
        // V rows past a request's last key are never loaded: they must hold finite data (0 * NaN)
        for (int i = threadIdx.x - 96; i < NV * kSlotBytes / 16; i += kSoft)
            reinterpret_cast<uint4 *>(s_v)[i] = make_uint4(0, 0, 0, 0);
        fence_proxy_async_smem();
    }
    if (warp == 1) tmem_alloc<Plan::kTmemCols>(&misc->tmem_base);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem = misc->tmem_base;
    const uint32_t tm_S0 = tmem, tm_O = tmem + 2 * NT;
    if (threadIdx.x == 0) SPI_TRACE_K(4);

    // Programmatic dependent launch: everything above overlapped the previous kernel's tail;
    // from here on we read inputs it may have produced.  With early_prefix (the caller guarantees
    // that neither the committed prefix of the caches nor the schedule in the workspace was written
    // by the immediately preceding kernel), the two producer threads first stage the committed-prefix
    // tiles of their first segment and only then wait; every other warp waits here.
    // (the whole producer warps skip this wait: a wait on lanes 1-31 alone would hold lane 0 at the
    // warp's reconvergence point; lane 0 waits after staging, lanes 1-31 read nothing)
    const bool early = p.early_prefix != 0 && (warp == 0 || warp == kWarpV);
    if (!early) grid_dependency_wait();
    if (threadIdx.x == 0) SPI_TRACE_K(5);
    // this CTA's slice of the tile sequence (precomputed by tree_prepare for this grid)
    const int4 ci = __ldg(p.cta_info + 2 * blockIdx.x);
    const int4 first_info = __ldg(p.cta_info + 2 * blockIdx.x + 1);
    const int t0 = ci.x, t1 = ci.y, x_first = ci.z, T = ci.w;
    const int ntiles = p.dyn ? 1 : t1 - t0;   // (dynamic mode: every CTA starts with item blockIdx.x)
    if (threadIdx.x == 0 && ntiles > -1000000) SPI_TRACE_K(6);

    if (ntiles <= 0) {
        // no work for this CTA (fewer tiles than CTAs)
        if (early) grid_dependency_wait();
    } else if (warp == 0 || warp == kWarpV) {
        // ============================ TMA producers ============================
        const uint64_t pol = l2_evict_first_policy();
        // one K (warp 0) or V (V warp) tile of segment d into ring slot lt % NS
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
            if (SPI_FLAGS(p) & 1) {
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
        // committed-prefix tiles of the first segment that fit the free ring slots (early mode)
        auto n_early = [&](const SegDesc &d, int NS) {
            int c = 0;
            while (c < NS && d.begin + c < d.end && (d.begin + c - d.ib + 1) * kKeyTile <= d.P) ++c;
            return c;
        };
        if (warp == 0 && lane == 0 && p.dyn) {
            // dynamic mode (see tree_attention_rows.cu): whole items, the first one is item blockIdx.x, the
            // next ones are claimed from the ticket counter after the dependency wait, each while the
            // current item streams; ticket t names item grid + t mod n_items (>= n_items: none left)
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
            int lt = 0, ls = 0;
            for (;;) {
                SegDesc d{};
                d.x = -1;
                while (dx >= 0) {
                    const int4 info = __ldg(p.item_info + dx);
                    if (info.y > info.x) {
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
                    dx = claim();   // an empty item
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
                const int qb = ls % Plan::kNQ;
                if (ls >= Plan::kNQ) mbar_wait(&misc->q_empty[qb], ((ls / Plan::kNQ) - 1) & 1);
                mbar_arrive_expect_tx(&misc->q_full[qb], 2u * (uint32_t)(p.G * p.npc) * 128u);
                uint8_t *qdst = s_q + qb * Plan::kQBuf;
                const int node0 = d.b * p.Nmax + d.c * p.npc;
                tma_load_3d(qdst, &tm_q, &misc->q_full[qb], 0, d.g * p.G, node0);
                tma_load_3d(qdst + NT * 128, &tm_q, &misc->q_full[qb], 64, d.g * p.G, node0);
                lt += pre;
                for (int t = d.begin + pre; t < d.end; ++t, ++lt) issue(d, t, lt, false);
                ++ls;
            }
            grid_launch_dependents();
        } else if (warp == 0 && lane == 0) {
            // segment descriptors for every role, Q, and the K tiles
            int lt = 0, ls = 0;
            int4 next_info = first_info;
            SPI_TRACE(12);
            for (int x = x_first; lt < ntiles; ++x) {
                const int4 info = next_info;  // {first tile, end tile, P, n}
                next_info = __ldg(p.item_info + x + 1);  // prefetched a segment ahead (sentinel-safe)
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
                if (ls == 0) SPI_TRACE(13);
                mbar_arrive(&misc->seg_full[ls % kSegRing]);  // release: descriptor visible
                int pre = 0;
                if (early && ls == 0) {
                    pre = n_early(d, NK);
                    for (int i = 0; i < pre; ++i) issue(d, d.begin + i, i, false);
                    grid_dependency_wait();   // q, tree keys and everything else: after the dependency
                }
                const int qb = ls % Plan::kNQ;
                if (ls >= Plan::kNQ) mbar_wait(&misc->q_empty[qb], ((ls / Plan::kNQ) - 1) & 1);
                mbar_arrive_expect_tx(&misc->q_full[qb], 2u * (uint32_t)(p.G * p.npc) * 128u);
                uint8_t *qdst = s_q + qb * Plan::kQBuf;
                const int node0 = d.b * p.Nmax + d.c * p.npc;
                tma_load_3d(qdst, &tm_q, &misc->q_full[qb], 0, d.g * p.G, node0);
                tma_load_3d(qdst + NT * 128, &tm_q, &misc->q_full[qb], 64, d.g * p.G, node0);
                if (ls == 0) SPI_TRACE(14);
                lt += pre;
                for (int t = d.begin + pre; t < d.end; ++t, ++lt) issue(d, t, lt, false);
                ++ls;
            }
            {   // terminal descriptor: the consumers stop here
                SegDesc d{};
                d.x = -1;
                misc->seg[ls % kSegRing] = d;
                mbar_arrive(&misc->seg_full[ls % kSegRing]);
            }
            grid_launch_dependents();  // all of this CTA's K loads are issued
        } else if (warp == kWarpV && lane == 0) {
            // V tiles, following the segment ring written by warp 0
            int lt = 0, ls = 0;
            for (;;) {
                mbar_wait(&misc->seg_full[ls % kSegRing], (ls / kSegRing) & 1);
                const SegDesc d = misc->seg[ls % kSegRing];
                if (d.x < 0) {   // terminal descriptor
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
    } else if (warp == 1) {
        // ===================== S issuer: S^T = K Q^T per tile =====================
        // (its own warp so that S(t+1) never queues behind PV(t) in one thread's program order)
        if (lane == 0) {
            const uint32_t idesc_s = make_idesc_bf16(128, NT, false, false);
            const uint32_t k_addr = smem_u32(s_k), q_addr = smem_u32(s_q);
            int lt = 0, ls = 0;
            for (;;) {
                mbar_wait(&misc->seg_full[ls % kSegRing], (ls / kSegRing) & 1);
                const SegDesc d = misc->seg[ls % kSegRing];
                if (d.x < 0) break;   // terminal descriptor
                const int qb = ls % Plan::kNQ;
                mbar_wait(&misc->q_full[qb], (ls / Plan::kNQ) & 1);
                for (int t = d.begin; t < d.end; ++t, ++lt) {
                    const int slot = lt % NK;
                    mbar_wait(&misc->k_full[slot], (lt / NK) & 1);
                    const int sb = lt & 1;
                    if (lt >= 2) mbar_wait(&misc->s_empty[sb], ((lt - 2) >> 1) & 1);
                    tc_fence_after();
                    SPI_TRACE(2);
                    const uint32_t kbase = k_addr + slot * kSlotBytes;
                    const uint32_t qbase = q_addr + qb * Plan::kQBuf;
#pragma unroll
                    for (int kk = 0; kk < kHeadDim / 16; ++kk) {
                        const uint32_t koff = (kk >> 2) * kHalfBytes + (kk & 3) * 32;
                        const uint32_t qoff = (kk >> 2) * (NT * 128) + (kk & 3) * 32;
                        const uint64_t adesc = make_smem_desc(kbase + koff, 16, 1024, kSw128);
                        const uint64_t bdesc = make_smem_desc(qbase + qoff, 16, 1024, kSw128);
                        if (!(SPI_FLAGS(p) & 2)) umma_bf16_ss(tm_S0 + sb * NT, adesc, bdesc, idesc_s, kk > 0 ? 1u : 0u);
                    }
                    umma_commit(&misc->s_full[sb]);
                    umma_commit(&misc->k_empty[slot]);
                    if (t == d.end - 1) umma_commit(&misc->q_empty[qb]);
                }
                ++ls;
            }
        }
    } else if (warp == 2) {
        // ===================== PV issuer: O^T += V^T P^T per tile ==================
        if (lane == 0) {
            const uint32_t idesc_o = make_idesc_bf16(128, NT, true, true);
            const uint32_t v_addr = smem_u32(s_v), p_addr = smem_u32(s_p);
            int lt = 0, ls = 0;
            for (;;) {
                mbar_wait(&misc->seg_full[ls % kSegRing], (ls / kSegRing) & 1);
                const SegDesc d = misc->seg[ls % kSegRing];
                if (d.x < 0) break;   // terminal descriptor
                for (int t = d.begin; t < d.end; ++t, ++lt) {
                    mbar_wait(&misc->p_full[lt % Plan::kNP], (lt / Plan::kNP) & 1);
                    const int slot = lt % NV;
                    mbar_wait(&misc->v_full[slot], (lt / NV) & 1);
                    tc_fence_after();
                    SPI_TRACE(3);
                    const uint32_t vbase = v_addr + slot * kSlotBytes;
                    const bool first = (t == d.begin);
#pragma unroll
                    for (int kk = 0; kk < kKeyTile / 16; ++kk) {
                        const uint64_t adesc = make_smem_desc(vbase + kk * 16 * 128, kHalfBytes, 1024, kSw128);
                        const uint64_t bdesc = make_smem_desc(p_addr + (lt % Plan::kNP) * Plan::kPBuf + kk * 16 * (NT * 2), Plan::kPBuf,
                                                              8 * NT * 2, Plan::kPSwizzle);
                        if (!(SPI_FLAGS(p) & 2)) umma_bf16_ss(tm_O, adesc, bdesc, idesc_o, (first && kk == 0) ? 0u : 1u);
                    }
                    umma_commit(&misc->p_empty[lt % Plan::kNP]);
                    umma_commit(&misc->v_empty[slot]);
                }
                ++ls;
            }
        }
    } else if (softw) {
        // ======================= softmax / epilogue warps =======================
        const int st = threadIdx.x - 96;       // 0..kSoft-1
        const int half = st >> 7;              // which half of the query rows (kSplit = 2)
        const int r0 = half * NTH;             // first query row (S^T / O^T column) of this thread
        const int qd = warp & 3;               // TMEM lane quarter of this warp
        const int kt = qd * 32 + lane;         // key within tile (S^T lane) / head dim (O^T lane)
        const int d = kt;
        const uint32_t lane_off = (uint32_t)(qd * 32) << 16;
        int lt = 0, ls = 0;
        for (;;) {
            mbar_wait(&misc->seg_full[ls % kSegRing], (ls / kSegRing) & 1);
            const SegDesc sd = misc->seg[ls % kSegRing];
            if (sd.x < 0) break;   // terminal descriptor
            const int b = sd.b, g = sd.g, c = sd.c, P = sd.P, n = sd.n;
            const int Kend = P + n;
            const int node0 = c * p.npc;
            const int G = p.G;
            // prefetch the tree row masks this thread needs in this segment (<= 3 tiles carry
            // tree keys): latency is hidden behind the prefix tiles
            const int tt_tree0 = P / kKeyTile;  // first item tile holding a tree key
            unsigned long long rm[3] = {0ull, 0ull, 0ull};
#pragma unroll
            for (int i = 0; i < 3; ++i) {
                const int tt = tt_tree0 + i;
                const int kk = tt * kKeyTile + kt;
                if (tt >= sd.begin - sd.ib && tt < sd.end - sd.ib && kk >= P && kk < Kend)
                    rm[i] = __ldg(p.rowmask + ((size_t)b * p.chunks + c) * p.Nmax + (kk - P));
            }
            // reset row statistics
            if (st < 32) {
                for (int r = lane; r < NT; r += 32) {
                    misc->m_thr[r] = -INFINITY;
                    misc->m_ref[r] = 0.f;
                }
            }
            float lsum[NTH];
#pragma unroll
            for (int r = 0; r < NTH; ++r) lsum[r] = 0.f;
            named_bar_sync(1, kSoft);
            if (st == 0) SPI_TRACE(10);

            for (int t = sd.begin; t < sd.end; ++t, ++lt) {
                const int tt = t - sd.ib;
                const int kk = tt * kKeyTile + kt;
                const int sb = lt & 1;
                // ---- S^T row of this key ----
                mbar_wait(&misc->s_full[sb], (lt >> 1) & 1);
                tc_fence_after();
                if (st == 0) SPI_TRACE(4);
                if (st == 0 && lt == 0) SPI_TRACE_K(7);
                float xv[NTH];
                {
                    uint32_t r16[NTH / 16][16];
#pragma unroll
                    for (int c16 = 0; c16 < NTH / 16; ++c16)
                        tmem_ld16(tm_S0 + sb * NT + r0 + c16 * 16 + lane_off, r16[c16]);
                    tmem_ld_wait();
#pragma unroll
                    for (int c16 = 0; c16 < NTH / 16; ++c16)
#pragma unroll
                        for (int i = 0; i < 16; ++i) xv[c16 * 16 + i] = __uint_as_float(r16[c16][i]) * p.scale_log2;
                }
                tc_fence_before();
                __syncwarp();
                if (lane == 0) mbar_arrive(&misc->s_empty[sb]);
                // ---- mask: committed keys are visible to every row (padded rows are harmless:
                // their Q rows are zero or belong to no output); tree keys use the row mask;
                // keys past the request's end are invisible ----
                if (kk >= P) {
                    unsigned long long vis = 0ull;
                    if (kk < Kend) {
                        const int i = tt - tt_tree0;
                        vis = i == 0 ? rm[0] : (i == 1 ? rm[1] : rm[2]);
                    }
#pragma unroll
                    for (int r = 0; r < NTH; ++r)
                        if (!((vis >> (r0 + r)) & 1ull)) xv[r] = -INFINITY;
                }
                // ---- does this tile raise a row max beyond the stale tolerance? ----
                bool need = false;
#pragma unroll
                for (int r = 0; r < NTH; r += 4) {
                    const float4 m4 = *reinterpret_cast<const float4 *>(&misc->m_thr[r0 + r]);
                    need |= (xv[r] > m4.x) | (xv[r + 1] > m4.y) | (xv[r + 2] > m4.z) | (xv[r + 3] > m4.w);
                }
                bulk_wait_read_all();  // output staging (P^T buffer) read by the bulk stores
                // one barrier instruction both synchronises the softmax warps and ORs their verdicts
                const bool rescale = named_bar_red_or(1, kSoft, need);
                if (rescale) {
                    // exact tile max per row: transpose-reduce within the warp, combine 4 warps
#pragma unroll
                    for (int blk = 0; blk < (NTH + 31) / 32; ++blk) {
                        constexpr int W = NTH < 32 ? NTH : 32;
                        float mx[W];
#pragma unroll
                        for (int r = 0; r < W; ++r) mx[r] = xv[blk * 32 + r];
                        transpose_reduce<W, true>(mx);
                        const int row = r0 + blk * 32 + (lane & (W - 1));
                        if (lane < W) misc->wred[qd][row] = mx[0];
                    }
                    named_bar_sync(1, kSoft);
                    if (st < 32) {
                        for (int r = lane; r < NT; r += 32) {
                            const float tmx = fmaxf(fmaxf(misc->wred[0][r], misc->wred[1][r]),
                                                    fmaxf(misc->wred[2][r], misc->wred[3][r]));
                            const float mo = misc->m_thr[r] - kRescaleThreshold;  // -inf stays -inf
                            const float mn = fmaxf(mo, tmx);
                            misc->alpha[r] = (mo == -INFINITY) ? 0.f : ex2(mo - mn);
                            misc->m_thr[r] = mn + kRescaleThreshold;
                            misc->m_ref[r] = (mn == -INFINITY) ? 0.f : mn;
                        }
                    }
                    named_bar_sync(1, kSoft);
#pragma unroll
                    for (int r = 0; r < NTH; ++r) lsum[r] *= misc->alpha[r0 + r];
                    if (t != sd.begin) {
                        // O^T columns (query rows) scaled by alpha: wait for PV of tile lt-1
                        mbar_wait(&misc->p_empty[(lt - 1) % Plan::kNP], ((lt - 1) / Plan::kNP) & 1);
                        tc_fence_after();
                        uint32_t r16[16];
#pragma unroll
                        for (int c16 = 0; c16 < NTH / 16; ++c16) {
                            tmem_ld16(tm_O + r0 + c16 * 16 + lane_off, r16);
                            tmem_ld_wait();
#pragma unroll
                            for (int i = 0; i < 16; ++i)
                                r16[i] = __float_as_uint(__uint_as_float(r16[i]) * misc->alpha[r0 + c16 * 16 + i]);
                            tmem_st16(tm_O + r0 + c16 * 16 + lane_off, r16);
                        }
                        tmem_st_wait();
                    }
                }
                // ---- probabilities, row sums ----
#pragma unroll
                for (int r = 0; r < NTH; r += 4) {
                    const float4 m4 = *reinterpret_cast<const float4 *>(&misc->m_ref[r0 + r]);
                    xv[r] = ex2(xv[r] - m4.x);
                    xv[r + 1] = ex2(xv[r + 1] - m4.y);
                    xv[r + 2] = ex2(xv[r + 2] - m4.z);
                    xv[r + 3] = ex2(xv[r + 3] - m4.w);
                }
                // P rounded to bf16 once; the row sums use the rounded values so that the
                // normalisation matches the numerator the PV MMA computes
                uint32_t pk[NTH / 2];
#pragma unroll
                for (int i = 0; i < NTH / 2; ++i) {
                    pk[i] = pack_bf16x2(xv[2 * i], xv[2 * i + 1]);
                    lsum[2 * i] = add_bf16lo(pk[i], lsum[2 * i]);       // the bf16 halves added in place
                    lsum[2 * i + 1] = add_bf16hi(pk[i], lsum[2 * i + 1]);
                }
                // ---- P^T row (this key) into smem as bf16, MN-major + swizzle ----
                if (lt >= Plan::kNP)  // PV(t - kNP) has read this buffer
                    mbar_wait(&misc->p_empty[lt % Plan::kNP], ((lt - Plan::kNP) / Plan::kNP) & 1);
                {
                    uint8_t *pb = s_p + (lt % Plan::kNP) * Plan::kPBuf;
#pragma unroll
                    for (int c8 = 0; c8 < NTH / 8; ++c8) {
                        const uint32_t o = (uint32_t)kt * (NT * 2) + (half * (NTH / 8) + c8) * 16;
                        const uint32_t phys = o ^ (((o >> 7) & Plan::kPMask) << 4);
                        *reinterpret_cast<uint4 *>(pb + phys) =
                            make_uint4(pk[c8 * 4], pk[c8 * 4 + 1], pk[c8 * 4 + 2], pk[c8 * 4 + 3]);
                    }
                }
                fence_proxy_async_smem();
                tc_fence_before();
                __syncwarp();
                if (lane == 0) mbar_arrive(&misc->p_full[lt % Plan::kNP]);
                if (st == 0) SPI_TRACE(5);

                if (t == sd.end - 1) {
                    // ============ epilogue of this segment ============
                    // row sums over the 128 keys of every tile: reduce the per-thread partials
#pragma unroll
                    for (int blk = 0; blk < (NTH + 31) / 32; ++blk) {
                        constexpr int W = NTH < 32 ? NTH : 32;
                        transpose_reduce<W, false>(lsum + blk * 32);
                        const int row = r0 + blk * 32 + (lane & (W - 1));
                        if (lane < W) misc->l_part[qd][row] = lsum[blk * 32];
                    }
                    mbar_wait(&misc->p_empty[lt % Plan::kNP], (lt / Plan::kNP) & 1);  // last PV done (and every earlier one)
                    tc_fence_after();
                    if (st == 0) SPI_TRACE(6);
                    float o[NTH];
                    {
                        uint32_t r16[NTH / 16][16];
#pragma unroll
                        for (int c16 = 0; c16 < NTH / 16; ++c16)
                            tmem_ld16(tm_O + r0 + c16 * 16 + lane_off, r16[c16]);
                        tmem_ld_wait();
#pragma unroll
                        for (int c16 = 0; c16 < NTH / 16; ++c16)
#pragma unroll
                            for (int i = 0; i < 16; ++i) o[c16 * 16 + i] = __uint_as_float(r16[c16][i]);
                    }
                    tc_fence_before();
                    named_bar_sync(1, kSoft);  // all l_part visible
                    if (st < NT) {
                        const float l = misc->l_part[0][st] + misc->l_part[1][st] + misc->l_part[2][st] + misc->l_part[3][st];
                        misc->run_l[st] = l;           // row sum of this segment
                        misc->alpha[st] = 1.0f / l;    // its reciprocal (inf for rows with no key)
                    }
                    named_bar_sync(1, kSoft);
                    if (st == 0) SPI_TRACE(9);
                    // (split-KV mode: a part of a split item stages a partial, the cluster's rank 0
                    // merges; an item left whole on rank 0 is written here directly)
                    const bool full = (sd.begin == sd.ib) && (sd.end == sd.ie);
                    const int rc = G * p.npc;
                    if (full) {
                        // stage the bf16 rows in the idle P^T buffer (row r at r*256 B, rows of a
                        // node contiguous) and write each node's G rows with one bulk async copy
                        __nv_bfloat16 *stg = reinterpret_cast<__nv_bfloat16 *>(s_p);
#pragma unroll
                        for (int r = 0; r < NTH; r += 4) {
                            const float4 inv = *reinterpret_cast<const float4 *>(&misc->alpha[r0 + r]);
                            stg[(r0 + r + 0) * kHeadDim + d] = __float2bfloat16_rn(o[r + 0] * inv.x);
                            stg[(r0 + r + 1) * kHeadDim + d] = __float2bfloat16_rn(o[r + 1] * inv.y);
                            stg[(r0 + r + 2) * kHeadDim + d] = __float2bfloat16_rn(o[r + 2] * inv.z);
                            stg[(r0 + r + 3) * kHeadDim + d] = __float2bfloat16_rn(o[r + 3] * inv.w);
                        }
                        fence_proxy_async_smem();
                        named_bar_sync(1, kSoft);
                        const int nodes_here = min(p.npc, n - node0);
                        if (st < nodes_here) {
                            bulk_store_s2g(p.out + (((size_t)b * p.Nmax + node0 + st) * p.Hq + g * G) * kHeadDim,
                                           s_p + st * G * kHeadDim * 2, (uint32_t)(G * kHeadDim * 2));
                            bulk_commit();
                        }
                        if (st == 0) SPI_TRACE(8);
                    } else {
                      if (p.splitk > 1) {
                        // split-KV mode: stage this part's (O, m, l) in the idle K ring (its only
                        // segment is done); the cluster merges them at the end of the kernel
                        float *so = reinterpret_cast<float *>(s_k);
#pragma unroll
                        for (int r = 0; r < NTH; ++r) so[(size_t)(r0 + r) * kHeadDim + d] = o[r];
                        if (st < NT) {
                            const float mt = misc->m_thr[st];
                            so[NT * kHeadDim + st] = mt == -INFINITY ? -INFINITY : mt - kRescaleThreshold;
                            so[NT * kHeadDim + NT + st] = misc->run_l[st];
                        }
                      } else {
                        const int slot = (sd.begin == t0) ? 0 : 1;
                        float *po = p.part_o + (((size_t)blockIdx.x * 2 + slot) * NT) * kHeadDim;
#pragma unroll
                        for (int r = 0; r < NTH; ++r) po[(size_t)(r0 + r) * kHeadDim + d] = o[r];
                        float *pml = p.part_ml + ((size_t)blockIdx.x * 2 + slot) * 2 * NT;
                        if (st < NT) {
                            const float mt = misc->m_thr[st];
                            pml[st] = mt == -INFINITY ? -INFINITY : mt - kRescaleThreshold;
                            pml[NT + st] = misc->run_l[st];
                        }
                        // release: the CTA barrier orders every thread's partial stores before thread
                        // 0's gpu-scope fence and counter update (fence cumulativity, one fence per CTA)
                        named_bar_sync(1, kSoft);
                        if (st == 0) SPI_TRACE(8);
                        if (st == 0) {
                            __threadfence();
                            const int c_first = cta_of_tile(sd.ib, T, NC);
                            const int c_last = cta_of_tile(sd.ie - 1, T, NC);
                            int npieces = 0;
                            for (int cc = c_first; cc <= c_last; ++cc)
                                npieces += cta_start(cc + 1, T, NC) > cta_start(cc, T, NC);
                            const unsigned old = atomicAdd(&p.item_cnt[sd.x], 1u);
                            misc->bcast = (old == (unsigned)(npieces - 1)) ? 1 : 0;
                            if (misc->bcast) p.item_cnt[sd.x] = 0u;  // ready for the next launch
                        }
                        named_bar_sync(1, kSoft);
                        if (st == 0) SPI_TRACE(11);
                        if (misc->bcast) {
                            // last piece: merge all pieces' (m, l, O) by log-sum-exp
                            __threadfence();
// merge-phase trace points go to the (unused) row of tile lt + 1: 0 start, 1 pieces issued,
// 2 staged, 3 weights, 4 accumulated, 5 stored
#define SPI_TRACE2(ev) do { if (st == 0 && SPI_TRACING(p) && blockIdx.x < kTraceCtas && lt + 1 < kTraceTiles) \
    p.trace[((size_t)blockIdx.x * kTraceTiles + lt + 1) * kTraceEv + (ev)] = clock64(); } while (0)
                            SPI_TRACE2(0);
                            float acc[NTH];
#pragma unroll
                            for (int r = 0; r < NTH; ++r) acc[r] = 0.f;
                            // CTA's last segment => the K / V rings are idle: stage every piece's
                            // (O, m, l) there with bulk copies (one L2 round trip for all pieces).
                            // One thread enumerates the pieces; the rest of the merge is unrolled over
                            // this thread's rows (latency-bound code: 4 warps, ILP from the rows).
                            constexpr uint32_t kOBytes = NT * kHeadDim * 4, kMLBytes = 2 * NT * 4;
                            float *so = reinterpret_cast<float *>(s_k);
                            if (st == 0) {
                                int npcs = -1;
                                if (sd.end == t1 && !(SPI_FLAGS(p) & 32)) {  // no tile follows: rings idle (32: test the fallback)
                                    npcs = 0;
                                    const int cf = cta_of_tile(sd.ib, T, NC), cl2 = cta_of_tile(sd.ie - 1, T, NC);
                                    for (int cc = cf; cc <= cl2 && npcs <= kCombineBatch; ++cc) {
                                        const int s0 = cta_start(cc, T, NC);
                                        if (cta_start(cc + 1, T, NC) <= s0) continue;
                                        if (npcs < kCombineBatch) misc->piece_off[npcs] = (size_t)cc * 2 + ((s0 >= sd.ib) ? 0 : 1);
                                        ++npcs;
                                    }
                                    if (npcs > kCombineBatch ||
                                        (size_t)npcs * (kOBytes + kMLBytes) > (size_t)(NK + NV) * kSlotBytes)
                                        npcs = -1;
                                }
                                misc->npieces = npcs;
                                if (npcs > 0) {
                                    fence_proxy_async_global();
                                    mbar_arrive_expect_tx(&misc->cmb_bar, (uint32_t)npcs * (kOBytes + kMLBytes));
                                    float *sml = so + (size_t)npcs * NT * kHeadDim;
                                    for (int pc = 0; pc < npcs; ++pc) {
                                        const size_t off = misc->piece_off[pc];
                                        bulk_load_g2s(so + (size_t)pc * NT * kHeadDim, p.part_o + off * NT * kHeadDim,
                                                      kOBytes, &misc->cmb_bar);
                                        bulk_load_g2s(sml + pc * 2 * NT, p.part_ml + off * 2 * NT, kMLBytes, &misc->cmb_bar);
                                    }
                                }
                            }
                            named_bar_sync(1, kSoft);
                            const int npcs = misc->npieces;
                            SPI_TRACE2(1);
                            if (npcs > 0) {
                                const float *sml = so + (size_t)npcs * NT * kHeadDim;
                                float *cmb_w = reinterpret_cast<float *>(s_p);
                                mbar_wait(&misc->cmb_bar, 0);
                                SPI_TRACE2(2);
                                if (st < NT) {
                                    const int r = st;
                                    float M = -INFINITY;
                                    for (int pc = 0; pc < npcs; ++pc) M = fmaxf(M, sml[pc * 2 * NT + r]);
                                    float L = 0.f;
                                    for (int pc = 0; pc < npcs; ++pc) {
                                        const float mp = sml[pc * 2 * NT + r];
                                        const float w = (mp == -INFINITY) ? 0.f : ex2(mp - M);
                                        cmb_w[pc * NT + r] = w;
                                        L += w * sml[pc * 2 * NT + NT + r];
                                    }
                                    misc->run_l[r] = L;
                                }
                                named_bar_sync(1, kSoft);
                                SPI_TRACE2(3);
                                // rows in groups of 8 (rolled outer loops): this code is cold in the
                                // instruction cache once per launch, so it is kept small
                                int node = node0 + r0 / G, hl = r0 % G;
#pragma unroll 1
                                for (int r8 = 0; r8 < NTH; r8 += 8) {
                                    float a8[8] = {0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f};
#pragma unroll 1
                                    for (int pc = 0; pc < npcs; ++pc) {
                                        const float *po2 = so + ((size_t)pc * NT + r0 + r8) * kHeadDim + d;
                                        const float *wv = cmb_w + pc * NT + r0 + r8;
#pragma unroll
                                        for (int i = 0; i < 8; ++i) a8[i] += wv[i] * po2[(size_t)i * kHeadDim];
                                    }
#pragma unroll
                                    for (int i = 0; i < 8; ++i) {
                                        const int rr = r0 + r8 + i;
                                        if (rr < rc && node < n)
                                            p.out[(((size_t)b * p.Nmax + node) * p.Hq + g * G + hl) * kHeadDim + d] =
                                                __float2bfloat16_rn(__fdividef(a8[i], misc->run_l[rr]));
                                        if (++hl == G) {
                                            hl = 0;
                                            ++node;
                                        }
                                    }
                                }
                                SPI_TRACE2(4);
                            } else {
                            // pieces staged kCombineBatch at a time through the idle P^T buffer so every
                            // global load of a batch is in flight
                            if (st < NT) {
                                misc->run_m[st] = -INFINITY;
                                misc->run_l[st] = 0.f;
                            }
                            // the P^T buffer is idle during an epilogue (last PV done, next P not yet written)
                            float *cmb_m = reinterpret_cast<float *>(s_p);
                            float *cmb_l = cmb_m + kCombineBatch * NT;
                            float *cmb_w = cmb_l + kCombineBatch * NT;
                            int cc = 0, c_last = 0;
                            if (st == 0) {
                                cc = cta_of_tile(sd.ib, T, NC);
                                c_last = cta_of_tile(sd.ie - 1, T, NC);
                            }
                            for (;;) {
                                named_bar_sync(1, kSoft);
                                if (st == 0) {
                                    int nb = 0;
                                    while (cc <= c_last && nb < kCombineBatch) {
                                        const int s0 = cta_start(cc, T, NC);
                                        if (cta_start(cc + 1, T, NC) > s0) {
                                            misc->piece_off[nb] = ((size_t)cc * 2 + ((s0 >= sd.ib) ? 0 : 1));
                                            ++nb;
                                        }
                                        ++cc;
                                    }
                                    misc->bcast = nb;
                                }
                                named_bar_sync(1, kSoft);
                                const int nb = misc->bcast;
                                if (nb == 0) break;
                                for (int idx = st; idx < nb * NT; idx += kSoft) {
                                    const int pc = idx / NT, r = idx - pc * NT;
                                    const float *pm = p.part_ml + misc->piece_off[pc] * 2 * NT;
                                    cmb_m[pc * NT + r] = ldcg_f32(pm + r);
                                    cmb_l[pc * NT + r] = ldcg_f32(pm + NT + r);
                                }
                                named_bar_sync(1, kSoft);
                                if (st < NT) {
                                    const int r = st;
                                    float bm = -INFINITY;
                                    for (int pc = 0; pc < nb; ++pc) bm = fmaxf(bm, cmb_m[pc * NT + r]);
                                    const float mo = misc->run_m[r];
                                    const float mn = fmaxf(mo, bm);
                                    const float sc = (mo == -INFINITY) ? 0.f : ex2(mo - mn);
                                    float L = misc->run_l[r] * sc;
                                    for (int pc = 0; pc < nb; ++pc) {
                                        const float mp = cmb_m[pc * NT + r];
                                        const float w = (mp == -INFINITY) ? 0.f : ex2(mp - mn);
                                        cmb_w[pc * NT + r] = w;
                                        L += w * cmb_l[pc * NT + r];
                                    }
                                    misc->run_m[r] = mn;
                                    misc->run_l[r] = L;
                                    misc->alpha[r] = sc;
                                }
                                named_bar_sync(1, kSoft);
#pragma unroll
                                for (int r = 0; r < NTH; ++r) acc[r] *= misc->alpha[r0 + r];
                                for (int pc = 0; pc < nb; ++pc) {
                                    const float *po2 = p.part_o + misc->piece_off[pc] * NT * kHeadDim + d;
                                    float v[NTH];
#pragma unroll
                                    for (int r = 0; r < NTH; ++r) v[r] = ldcg_f32(po2 + (size_t)(r0 + r) * kHeadDim);
#pragma unroll
                                    for (int r = 0; r < NTH; ++r) acc[r] += cmb_w[pc * NT + r0 + r] * v[r];
                                }
                            }
                            }
                            // fallback: row rr = node_local * G + hl, walked incrementally (no division)
                            int node = node0 + r0 / G, hl = r0 % G;
#pragma unroll
                            for (int r = 0; r < NTH && npcs <= 0; ++r) {
                                const int rr = r0 + r;
                                if (rr < rc && node < n) {
                                    p.out[(((size_t)b * p.Nmax + node) * p.Hq + g * G + hl) * kHeadDim + d] =
                                        __float2bfloat16_rn(__fdividef(acc[r], misc->run_l[rr]));
                                }
                                if (++hl == G) {
                                    hl = 0;
                                    ++node;
                                }
                            }
                            SPI_TRACE2(5);
                        }
                      }
                    }
                    named_bar_sync(1, kSoft);  // stats read by everyone before the next reset
                    if (st == 0) SPI_TRACE(7);
                }
            }
            ++ls;
        }
    }

    if (softw) bulk_wait_all();  // output bulk stores complete before smem goes away
    tc_fence_before();
    __syncthreads();
    if (p.splitk > 1) {
        // ======== split-KV mode: merge the cluster's partials (DSMEM), rank 0 writes the rows ========
        namespace cg = cooperative_groups;
        cg::cluster_group cluster = cg::this_cluster();
        float *so = reinterpret_cast<float *>(s_k);
        if (ntiles <= 0 && threadIdx.x < NT) {  // no tiles for this part: it saw no key
            so[NT * kHeadDim + threadIdx.x] = -INFINITY;
            so[NT * kHeadDim + NT + threadIdx.x] = 0.f;
        }
        // partial k (O rows [NT][128] then m [NT], l [NT]) lives at kPart floats into rank 0's K/V rings
        constexpr int kPart = NT * kHeadDim + 2 * NT;
        cluster.sync();  // every rank's tiles done: rank 0's rings are idle, every part staged locally
        if (threadIdx.x == 0) SPI_TRACE_K(3);
        const int K = p.splitk;
        const int rank = (int)cluster.block_rank();
        if (rank != 0) {
            // push this part into rank 0's shared memory (fire-and-forget DSMEM stores, 16 B each)
            uint4 *dst = reinterpret_cast<uint4 *>(cluster.map_shared_rank(so, 0) + (size_t)rank * kPart);
            const uint4 *src = reinterpret_cast<const uint4 *>(so);
            for (int i = threadIdx.x; i < kPart / 4; i += blockDim.x) dst[i] = src[i];
        }
        cluster.sync();  // every part is in rank 0's shared memory; ranks != 0 may exit
        const int x = blockIdx.x / K;
        const int4 info = __ldg(p.item_info + x);
        const bool whole = t0 == info.x && t1 == info.y;  // rank 0 streamed (and wrote) the whole item
        if (rank == 0 && softw && !whole && info.y > info.x) {
            const int st = threadIdx.x - 96;
            const int r0 = (st >> 7) * NTH;
            const int d = (warp & 3) * 32 + lane;
            const int n = info.w, G = p.G, rc = G * p.npc;
            const int c = x % p.chunks, g = (x / p.chunks) % p.Hkv, b = x / (p.chunks * p.Hkv);
            const int node0 = c * p.npc;
            float *cmb_w = so + (size_t)K * kPart;  // [K][NT] merge weights, after the staged partials
            if (st < NT) {
                float M = -INFINITY;
                for (int k = 0; k < K; ++k) M = fmaxf(M, so[(size_t)k * kPart + NT * kHeadDim + st]);
                float L = 0.f;
                for (int k = 0; k < K; ++k) {
                    const float *rk = so + (size_t)k * kPart;
                    const float mk = rk[NT * kHeadDim + st];
                    const float w = (mk == -INFINITY) ? 0.f : ex2(mk - M);
                    cmb_w[k * NT + st] = w;
                    L += w * rk[NT * kHeadDim + NT + st];
                }
                misc->run_l[st] = L;
            }
            named_bar_sync(1, kSoft);
            float acc[NTH];
#pragma unroll
            for (int r = 0; r < NTH; ++r) acc[r] = 0.f;
            for (int k = 0; k < K; ++k) {
                const float *rk = so + (size_t)k * kPart + d;
#pragma unroll
                for (int r = 0; r < NTH; ++r) {
                    const float w = cmb_w[k * NT + r0 + r];
                    if (w != 0.f) acc[r] += w * rk[(size_t)(r0 + r) * kHeadDim];
                }
            }
            int node = node0 + r0 / G, hl = r0 % G;
#pragma unroll
            for (int r = 0; r < NTH; ++r) {
                const int rr = r0 + r;
                if (rr < rc && node < n && n > 0)
                    p.out[(((size_t)b * p.Nmax + node) * p.Hq + g * G + hl) * kHeadDim + d] =
                        __float2bfloat16_rn(__fdividef(acc[r], misc->run_l[rr]));
                if (++hl == G) {
                    hl = 0;
                    ++node;
                }
            }
        }
    }
    if (warp == 1) {
        tc_fence_after();
        tmem_dealloc<Plan::kTmemCols>(tmem);
    }
    if (threadIdx.x == 0) SPI_TRACE_K(1);
}

template <int NT>
static size_t attn_smem_bytes(int num_slots) {
    using Plan = SmemPlan<NT>;
    static_assert(3 * kCombineBatch * NT * 4 <= Plan::kPBuf, "combine staging must fit the P buffer");
    return 1024 + (size_t)num_slots * kSlotBytes + Plan::kNQ * Plan::kQBuf + Plan::kNP * Plan::kPBuf +
           sizeof(SmemMisc);
}

// bytes rank 0 of a split-KV cluster can stage partials in: its K/V rings, Q and P^T buffers
// (contiguous, all idle once its tiles are done)
template <int NT>
static size_t split_stage_bytes(int num_slots) {
    using Plan = SmemPlan<NT>;
    return (size_t)num_slots * kSlotBytes + Plan::kNQ * Plan::kQBuf + Plan::kNP * Plan::kPBuf;
}

template <int NT>
static cudaError_t launch_nt(const AttnParams &prm0, const void *q, const void *k, const void *v,
                             int num_sms, size_t max_smem, cudaStream_t stream) {
    AttnParams prm = prm0;
    CUtensorMap tq, tk, tv, tk16, tv16, tk4, tv4, tk1, tv1;
    const uint64_t rows = prm.page_table ? (uint64_t)prm.n_pages * prm.Hkv * kKeyTile
                                         : (uint64_t)prm.B * prm.Hkv * prm.Smax;
    if (!encode_q(&tq, q, prm.Hq, (uint64_t)prm.B * prm.Nmax, prm.G, prm.npc) ||
        !encode_2d(&tk, k, rows, kKeyTile) || !encode_2d(&tv, v, rows, kKeyTile) ||
        !encode_2d(&tk16, k, rows, 16) || !encode_2d(&tv16, v, rows, 16) || !encode_2d(&tk4, k, rows, 4) ||
        !encode_2d(&tv4, v, rows, 4) || !encode_2d(&tk1, k, rows, 1) || !encode_2d(&tv1, v, rows, 1))
        return cudaErrorInvalidValue;
    int ns = 2 * kMaxSlots;
    while (ns > 2 && attn_smem_bytes<NT>(ns) > max_smem) --ns;
    // split-KV mode: rank 0 gathers every part's partial (and the merge weights) in its idle buffers
    if (prm0.splitk > 1 && (size_t)prm0.splitk * (NT * kHeadDim + 3 * NT) * 4 > split_stage_bytes<NT>(ns))
        return cudaErrorInvalidConfiguration;
    // K tiles are released right after S = K Q^T; V tiles are held until PV: give V the extra slot
    ns = min(ns, 6);
    prm.nk_slots = ns / 2;
    prm.nv_slots = ns - ns / 2;
    const size_t smem = attn_smem_bytes<NT>(ns);
    {
        const cudaError_t e = ensure_max_smem_attr((const void *)tree_attn_kernel<NT>, NT == 16 ? 0 : (NT == 32 ? 1 : 2),
                                                   max_smem);
        if (e != cudaSuccess) return e;
    }
    // programmatic dependent launch: the prologue (barrier init, TMEM alloc, smem zeroing) of
    // this grid overlaps the tail of the previous kernel on the stream
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(num_sms);  // (the caller's grid: w.grid)
    cfg.blockDim = dim3(SwRoles<NT>::kThreads);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = stream;
    cudaLaunchAttribute attr[2];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    if (prm.splitk > 1) {  // split-KV mode: one cluster of splitk CTAs per item
        attr[1].id = cudaLaunchAttributeClusterDimension;
        attr[1].val.clusterDim.x = prm.splitk;
        attr[1].val.clusterDim.y = 1;
        attr[1].val.clusterDim.z = 1;
        cfg.numAttrs = 2;
    }
    return cudaLaunchKernelEx(&cfg, tree_attn_kernel<NT>, tq, tk, tv, tk16, tv16, tk4, tv4, tk1, tv1, prm);
}

cudaError_t launch_tree_attention_rows(const AttnParams &prm0, const void *q, const void *k, const void *v,
                                       int num_ctas, size_t max_smem, cudaStream_t stream);

#ifdef SPECINFER_DEBUG_HOOKS
unsigned long long *g_attn_trace = nullptr;  // debug build only (specinfer_debug_set_trace)
int g_attn_debug_flags = 0;                   // debug build only (SPECINFER_DEBUG_FLAGS, experiments)
#endif

cudaError_t launch_tree_attention(const specinfer_shape_t &s, const WsLayout &w, const void *q,
                                  const void *k, const void *v, const int32_t *prefix_len,
                                  const int32_t *n_nodes, void *out, char *ws, int num_sms,
                                  size_t max_smem, cudaStream_t stream, const int32_t *page_table,
                                  int num_pages, uint32_t flags) {
    AttnParams prm{};
    prm.early_prefix = (flags & SPECINFER_ATTN_EARLY_PREFIX) ? 1 : 0;
    prm.page_table = page_table;
    prm.max_pages = (s.max_seq + kKeyTile - 1) / kKeyTile;
    prm.n_pages = num_pages;
    prm.prefix_len = prefix_len;
    prm.n_nodes = n_nodes;
    prm.item_start = reinterpret_cast<const int32_t *>(ws + w.item_start);
    prm.item_cnt = reinterpret_cast<uint32_t *>(ws + w.item_cnt);
    prm.item_info = reinterpret_cast<const int4 *>(ws + w.item_info);
    prm.cta_info = reinterpret_cast<const int4 *>(ws + w.cta_info);
    prm.rowmask = reinterpret_cast<const unsigned long long *>(ws + w.rowmask);
    prm.anc = reinterpret_cast<const uint32_t *>(ws + w.anc);
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
    prm.lanes = w.lanes;
    const float sm_scale = s.sm_scale > 0.f ? s.sm_scale : 1.0f / sqrtf((float)s.head_dim);
    prm.scale_log2 = sm_scale * 1.4426950408889634f;
#ifdef SPECINFER_DEBUG_HOOKS
    prm.trace = g_attn_trace;
    prm.debug_flags = g_attn_debug_flags;
#endif
    prm.splitk = w.splitk;
    const int grid = w.grid;  // persistent one CTA per SM, or n_items x splitk in split-KV mode
    // enough items per CTA (and no split-KV clusters): dynamic whole-item claims instead of the static
    // stream-K split.  Per-CTA speed differs by ~10% across a B200's SMs, which a static split cannot see,
    // and whole items need no lock-step lanes or split merges: measured faster at every C3 / C4 batch from
    // 1.7 items per CTA up (bench A/B: C3 345 -> 314 us, C4 885 -> 787 us per launch) and for the swapped
    // kernel at C2 batch 16 (89.2 -> 87.3 us per layer; batch 8 unchanged).  Fewer items than CTAs keep
    // the stream-K split (long items spread over many CTAs).
    prm.dyn_ctr = reinterpret_cast<uint32_t *>(ws + w.dyn_ctr);
    // (the rows kernel's static path -- lock-step lanes, split merges -- costs more: it switches to whole
    // items from half an item per CTA up, C3 batch 4 48.3 -> 43.6 us; the swapped kernel keeps stream-K
    // below one item per CTA, C2 batch 4 24.3 vs 24.7 us)
    prm.dyn = (w.splitk == 1 && (w.nt == kRowsBlock ? 2 * w.n_items >= grid : w.n_items >= grid)) ? 1 : 0;
    switch (w.nt) {
        case 16: return launch_nt<16>(prm, q, k, v, grid, max_smem, stream);
        case 32: return launch_nt<32>(prm, q, k, v, grid, max_smem, stream);
        case 64: return launch_nt<64>(prm, q, k, v, grid, max_smem, stream);
        default: return launch_tree_attention_rows(prm, q, k, v, grid, max_smem, stream);
    }
}

}  // namespace specinfer
