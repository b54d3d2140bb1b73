// prepare.cu — K1 tree_prepare.
//
// Per request: validate the token tree (Def. 3.1: node u has parent p_u and
// S_u = S_{p_u} + t_u; nodes in topological order, reading R5), and build the bitsets of the
// topology-aware causal mask (L657-674): anc[i] = Anc*(i) = anc[parent[i]] U {i} and its
// transpose desc[j] = { i : j in Anc*(i) }.  Then one block builds the tree-attention work
// schedule: items (b, kv-head g, row chunk c) with ceil((P_b + n_b)/128) KV tiles each, and
// their exclusive tile prefix (a stream-K style split of the whole KV stream over the CTAs).
#include "common.cuh"

namespace specinfer {

constexpr int kPrepThreads = 512;

// Per request (one CTA): validate the tree and build its bitsets / row masks.  Parents and depths
// are staged in shared memory first (one round of loads), desc = the transpose of anc is built
// 32 x 32 bits at a time with warp ballots.
__device__ void validate_bitsets(
    int b, const int32_t *__restrict__ parent, const int32_t *__restrict__ depth,
    const int32_t *__restrict__ prefix_len, const int32_t *__restrict__ n_nodes, int Nmax,
    int max_depth, int Smax, int G, int npc, int chunks, int32_t *__restrict__ status, int32_t *__restrict__ req_ok,
    uint32_t *__restrict__ anc, uint32_t *__restrict__ desc, unsigned long long *__restrict__ rowmask) {
    __shared__ int32_t s_par[kMaxNodes], s_dep[kMaxNodes];
    __shared__ uint32_t s_anc[kMaxNodes][kBitWords];
    __shared__ int s_bad;
    const int n = n_nodes[b];
    const int P = prefix_len[b];
    if (threadIdx.x == 0) s_bad = (n < 1 || n > Nmax || P < 0 || (long long)P + n > Smax) ? 1 : 0;
    for (int i = threadIdx.x; i < Nmax; i += blockDim.x) {
        s_par[i] = parent[(size_t)b * Nmax + i];
        s_dep[i] = depth[(size_t)b * Nmax + i];
    }
    __syncthreads();
    const bool n_ok = !s_bad;
    for (int i = threadIdx.x; n_ok && i < n; i += blockDim.x) {
        const int p = s_par[i], d = s_dep[i];
        const bool bad = (i == 0) ? (p != -1 || d != 0)
                                  : (p < 0 || p >= i || d > max_depth || d != s_dep[p] + 1);
        if (bad) atomicOr(&s_bad, 1);
    }
    __syncthreads();
    const bool ok = !s_bad;
    // ancestor-or-self bitsets by walking to the root (<= Dmax + 1 steps on a valid tree)
    for (int i = threadIdx.x; i < Nmax; i += blockDim.x) {
        uint32_t w[kBitWords];
#pragma unroll
        for (int k = 0; k < kBitWords; ++k) w[k] = 0;
        if (ok && i < n) {
            int u = i;
            while (u >= 0) {
#pragma unroll
                for (int k = 0; k < kBitWords; ++k)
                    if ((u >> 5) == k) w[k] |= 1u << (u & 31);
                u = s_par[u];
            }
        }
#pragma unroll
        for (int k = 0; k < kBitWords; ++k) {
            s_anc[i][k] = w[k];
            anc[((size_t)b * Nmax + i) * kBitWords + k] = w[k];
        }
    }
    __syncthreads();
    // descendant-or-self bitsets: desc[j] bit i  <=>  anc[i] bit j; warp task (iw, jw) transposes
    // the 32 x 32 block of rows i in [32 iw, 32 iw + 32) and columns j in [32 jw, 32 jw + 32)
    {
        const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5, nw = blockDim.x >> 5;
        const int njw = (Nmax + 31) >> 5;
        for (int task = wid; task < njw * kBitWords; task += nw) {
            const int jw = task / kBitWords, iw = task % kBitWords;
            const int i = 32 * iw + lane;
            const uint32_t a = (i < Nmax) ? s_anc[i][jw] : 0u;   // rows past n / invalid trees are 0
            uint32_t mine = 0u;
#pragma unroll 8
            for (int k = 0; k < 32; ++k) {
                const uint32_t col = __ballot_sync(0xffffffffu, (a >> k) & 1u);
                if (lane == k) mine = col;
            }
            const int j = 32 * jw + lane;
            if (j < Nmax) desc[((size_t)b * Nmax + j) * kBitWords + iw] = mine;
        }
    }
    // row masks of the tree part for the attention kernel: bit r of rowmask[b][c][j] is set iff
    // query row r of chunk c (node c*npc + r/G) exists and has tree node j on its root path
    const int rc = G * npc;  // the row masks serve the swapped kernel (<= 64 rows per chunk)
    for (int idx = threadIdx.x; rc <= 64 && idx < chunks * Nmax; idx += blockDim.x) {
        const int c = idx / Nmax, j = idx - c * Nmax;
        unsigned long long m = 0ull;
        if (ok && j < n) {
            for (int r = 0; r < rc; ++r) {
                const int node = c * npc + r / G;
                if (node < n && ((s_anc[node][j >> 5] >> (j & 31)) & 1u)) m |= 1ull << r;
            }
        }
        rowmask[((size_t)b * chunks + c) * Nmax + j] = m;
    }
    if (threadIdx.x == 0) req_ok[b] = ok ? 1 : 0;   // (the schedule kernel sets the status words)
}

// Single block: tiles per schedule unit, exclusive scan, total; zero the split/verify counters.
// A unit is one item (lanes == 1) or the `lanes` row chunks of one (b, kv-head) (lanes == chunks,
// the rows-as-M kernel).  In lane mode CTA c runs chunk c % lanes of every unit in its tile range
// [t0, t1) of the unit stream, so the `lanes` CTAs of a group read the same KV tile at about the
// same time: one HBM read, the other chunks hit L2.
__device__ void schedule(
    const int32_t *__restrict__ prefix_len, const int32_t *__restrict__ n_nodes,
    const int32_t *req_ok, int B, int Hkv, int chunks, int npc, int lanes,
    int32_t *__restrict__ item_start, uint32_t *__restrict__ item_cnt, int4 *__restrict__ item_info,
    int4 *__restrict__ cta_info, int num_ctas, int splitk, uint32_t *__restrict__ verify_cnt,
    int32_t *__restrict__ status, int no_split_slack) {
    const int n_items = B * Hkv * chunks;
    const int n_units = n_items / lanes;
    const int per = (n_units + blockDim.x - 1) / blockDim.x;
    const int lo = threadIdx.x * per;
    const int hi = min(n_units, lo + per);
    // per-request (n, P, ok) and the unit tile prefix live in shared memory when they fit, so the
    // schedule is one round of global loads and then shared-memory work (this block runs on the
    // critical path of every step; each dependent L2 round trip is ~0.5 us)
    constexpr int kSmB = 1024, kSmU = 4096;
    __shared__ int s_n[kSmB], s_P[kSmB], s_ok[kSmB];
    __shared__ int s_start[kSmU + 1];
    const bool smB = B <= kSmB, smU = n_units <= kSmU;
    if (smB)
        for (int b = threadIdx.x; b < B; b += blockDim.x) {
            s_n[b] = n_nodes[b];
            s_P[b] = prefix_len[b];
            s_ok[b] = __ldcg(req_ok + b);   // written by the other CTAs of the launch
        }
    __syncthreads();
    // status words of this tree: [0] = bad-tree bit if any request failed validation (replaces every
    // earlier sticky bit), [1] = total tiles (below), [2..63] = 0
    int bad_local = 0;
    for (int b = threadIdx.x; b < B; b += blockDim.x) bad_local |= (smB ? s_ok[b] : __ldcg(req_ok + b)) == 0;
    const int any_bad = __syncthreads_or(bad_local);
    if (threadIdx.x == 0) status[0] = any_bad ? kStatusBadTree : 0;
    for (int i = 2 + threadIdx.x; i < 64; i += blockDim.x) status[i] = 0;
    auto N_of = [&](int b) { return smB ? s_n[b] : n_nodes[b]; };
    auto P_of = [&](int b) { return smB ? s_P[b] : prefix_len[b]; };
    auto ok_of = [&](int b) { return smB ? s_ok[b] : __ldcg(req_ok + b); };
    // tiles of unit u: a unit's chunks share its KV stream; an empty chunk (c * npc >= n) of a
    // lane-mode unit keeps the unit's tile range and is skipped by its CTAs (n field 0)
    auto tiles_of = [&](int u) -> int {
        const int x = u * lanes;
        const int c = x % chunks;
        const int b = x / (chunks * Hkv);
        if (!ok_of(b)) return 0;
        const int n = N_of(b);
        if (c * npc >= n) return 0;
        return (P_of(b) + n + kKeyTile - 1) / kKeyTile;
    };
    int local = 0, local_max = 0;
    for (int u = lo; u < hi; ++u) {
        const int tl = tiles_of(u);
        local += tl;
        local_max = max(local_max, tl);
    }
    __shared__ int s_max_tiles;
    if (threadIdx.x == 0) s_max_tiles = 0;
    __syncthreads();
    atomicMax(&s_max_tiles, local_max);
    // block exclusive scan of per-thread sums
    __shared__ int s_warp[32];
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    int v = local;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const int t = __shfl_up_sync(0xffffffffu, v, o);
        if (lane >= o) v += t;
    }
    if (lane == 31) s_warp[wid] = v;
    __syncthreads();
    if (wid == 0) {
        int w = (lane < (int)(blockDim.x >> 5)) ? s_warp[lane] : 0;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const int t = __shfl_up_sync(0xffffffffu, w, o);
            if (lane >= o) w += t;
        }
        s_warp[lane] = w;
    }
    __syncthreads();
    int run = v - local + (wid > 0 ? s_warp[wid - 1] : 0);
    for (int u = lo; u < hi; ++u) {
        const int tl = tiles_of(u);
        item_start[u] = run;
        if (smU) s_start[u] = run;
        for (int x = u * lanes; x < (u + 1) * lanes; ++x) {
            const int b = x / (chunks * Hkv);
            const int c = x % chunks;
            const int n = N_of(b);
            const bool empty = lanes > 1 && c * npc >= n;
            item_info[x] = make_int4(run, run + tl, P_of(b), empty ? 0 : n);
            item_cnt[x] = 0u;
        }
        run += tl;
    }
    __shared__ int s_total;
    if (threadIdx.x == blockDim.x - 1) {
        item_start[n_units] = run;
        if (smU) s_start[n_units] = run;
        item_info[n_items] = make_int4(run, run, 0, 0);
        status[1] = run;
        s_total = run;
    }
    for (int b = threadIdx.x; b < 2 * B; b += blockDim.x) verify_cnt[b] = 0u;
    __syncthreads();
    // per-CTA slice [t0, t1) of the unit tile sequence, and its first item.
    // Small problems (every unit fits a CTA group and the longest unit is at most kNoSplitSlack
    // tiles longer than an even stream-K share): one unit per CTA group, no split, so no split
    // combine -- its partial write / atomic / merge code runs cold once per launch (~10 us of
    // instruction-cache misses at the kernel's tail, measured) and costs more than the
    // parallelism it buys (C1: 2 tiles per unit; B = 1..4 at P = 2048: 17).  Otherwise even stream-K slices.
    const long long T = s_total;
    const int NCv = num_ctas / lanes;
    // (no_split_slack: 8 tiles for the swapped kernel; 24 for the rows kernel, whose split merge
    // reads 64 KB partials per piece -- a few L2 round trips -- so tiny stream-K pieces do not pay)
    const int kNoSplitSlack = no_split_slack;
    // whole units per CTA group (contiguous ranges of floor / ceil(n_units / NCv) units) when the
    // busiest group's upper bound exceeds an even share by at most kNoSplitSlack tiles
    const int upc = (n_units + NCv - 1) / NCv;
    const bool one_per_cta = n_units > 0 &&
        (long long)upc * s_max_tiles * NCv <= T + (long long)kNoSplitSlack * NCv;
    auto start_of = [&](int u) { return smU ? s_start[u] : item_start[u]; };
    auto info_of = [&](int x) -> int4 {   // == item_info[x], rebuilt from shared memory
        if (!smU || !smB) return item_info[x];
        const int u = x / lanes, b = x / (chunks * Hkv), c = x % chunks;
        const int n = s_n[b];
        const bool empty = lanes > 1 && c * npc >= n;
        return make_int4(s_start[u], s_start[u + 1], s_P[b], empty ? 0 : n);
    };
    for (int c = threadIdx.x; c < num_ctas; c += blockDim.x) {
        const int vc = c / lanes, cl = c % lanes;
        if (splitk > 1) {  // split-KV mode (lanes == 1): CTA c = part c % splitk of item c / splitk
            const int u = c / splitk, r = c % splitk;
            int t0 = (int)T, t1 = (int)T;
            if (u < n_units) {
                // short items stay whole on rank 0 (written directly, no merge): the cluster merge
                // costs about as much as streaming kMinSplitTiles tiles on one CTA
                constexpr int kMinSplitTiles = 12;
                const int s0 = start_of(u), len = start_of(u + 1) - s0;
                if (len < kMinSplitTiles) {
                    t0 = r == 0 ? s0 : s0 + len;
                    t1 = s0 + len;
                } else {
                    t0 = s0 + (int)((long long)r * len / splitk);
                    t1 = s0 + (int)((long long)(r + 1) * len / splitk);
                }
            }
            const int x0 = u < n_units ? u : n_items;
            cta_info[2 * c] = make_int4(t0, t1, x0, (int)T);
            cta_info[2 * c + 1] = x0 < n_items ? info_of(x0) : make_int4(0, 0, 0, 0);
            continue;
        }
        if (one_per_cta) {
            // (at most one unit per group: units on groups 0 .. n_units-1, measured 7.4 -> 6.8 us at C1)
            const int u_lo = n_units <= NCv ? min(vc, n_units) : (int)((long long)vc * n_units / NCv);
            const int u_hi = n_units <= NCv ? min(vc + 1, n_units) : (int)((long long)(vc + 1) * n_units / NCv);
            const int t0 = start_of(u_lo);
            const int t1 = start_of(u_hi);
            const int x0 = u_lo < u_hi ? u_lo * lanes + cl : n_items;
            cta_info[2 * c] = make_int4(t0, t1, x0, (int)T);
            cta_info[2 * c + 1] = x0 < n_items ? info_of(x0) : make_int4(0, 0, 0, 0);
            continue;
        }
        const int t0 = (int)((long long)vc * T / NCv);
        const int t1 = (int)((long long)(vc + 1) * T / NCv);
        int lo2 = 0, hi2 = n_units;  // last unit with start <= t0
        while (hi2 - lo2 > 1) {
            const int mid = (lo2 + hi2) >> 1;
            if (start_of(mid) <= t0) lo2 = mid; else hi2 = mid;
        }
        const int x0 = lo2 * lanes + cl;
        cta_info[2 * c] = make_int4(t0, t1, x0, (int)T);
        cta_info[2 * c + 1] = x0 < n_items ? info_of(x0) : make_int4(0, 0, 0, 0);
    }
}

// Two launches per tree, no memset: one CTA per request validates it and builds its bitsets; then
// one CTA builds the schedule and the status words from req_ok (the kernel boundary orders them).
__global__ void __launch_bounds__(kPrepThreads) tree_validate_kernel(
    const int32_t *__restrict__ parent, const int32_t *__restrict__ depth,
    const int32_t *__restrict__ prefix_len, const int32_t *__restrict__ n_nodes, int Nmax, int max_depth,
    int Smax, int G, int npc, int chunks, int32_t *__restrict__ status, int32_t *__restrict__ req_ok,
    uint32_t *__restrict__ anc, uint32_t *__restrict__ desc, unsigned long long *__restrict__ rowmask) {
    validate_bitsets(blockIdx.x, parent, depth, prefix_len, n_nodes, Nmax, max_depth, Smax, G, npc, chunks, status,
                     req_ok, anc, desc, rowmask);
}

__global__ void __launch_bounds__(kPrepThreads) schedule_kernel(
    const int32_t *__restrict__ prefix_len, const int32_t *__restrict__ n_nodes, const int32_t *req_ok, int B,
    int Hkv, int chunks, int npc, int lanes, int32_t *__restrict__ item_start, uint32_t *__restrict__ item_cnt,
    int4 *__restrict__ item_info, int4 *__restrict__ cta_info, int num_ctas, int splitk,
    uint32_t *__restrict__ verify_cnt, int32_t *__restrict__ status, int no_split_slack, uint32_t *dyn_ctr) {
    if (threadIdx.x == 0) *dyn_ctr = 0u;   // the rows kernel's item tickets start over every step
    schedule(prefix_len, n_nodes, req_ok, B, Hkv, chunks, npc, lanes, item_start, item_cnt, item_info, cta_info,
             num_ctas, splitk, verify_cnt, status, no_split_slack);
}

cudaError_t launch_tree_prepare(const specinfer_shape_t &s, const WsLayout &w,
                                const int32_t *parent, const int32_t *depth,
                                const int32_t *prefix_len, const int32_t *n_nodes, char *ws,
                                int num_ctas, cudaStream_t stream) {
    int32_t *status = reinterpret_cast<int32_t *>(ws + w.status);
    int32_t *req_ok = reinterpret_cast<int32_t *>(ws + w.req_ok);
    tree_validate_kernel<<<s.batch, kPrepThreads, 0, stream>>>(
        parent, depth, prefix_len, n_nodes, s.max_nodes, s.max_depth, s.max_seq,
        s.num_q_heads / s.num_kv_heads, w.npc, w.chunks, status, req_ok,
        reinterpret_cast<uint32_t *>(ws + w.anc), reinterpret_cast<uint32_t *>(ws + w.desc),
        reinterpret_cast<unsigned long long *>(ws + w.rowmask));
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
    schedule_kernel<<<1, kPrepThreads, 0, stream>>>(
        prefix_len, n_nodes, req_ok, s.batch, s.num_kv_heads, w.chunks, w.npc, w.lanes,
        reinterpret_cast<int32_t *>(ws + w.item_start), reinterpret_cast<uint32_t *>(ws + w.item_cnt),
        reinterpret_cast<int4 *>(ws + w.item_info), reinterpret_cast<int4 *>(ws + w.cta_info), num_ctas, w.splitk,
        reinterpret_cast<uint32_t *>(ws + w.verify_cnt), status, w.nt == kRowsBlock ? 24 : 8,
        reinterpret_cast<uint32_t *>(ws + w.dyn_ctr));
    return cudaGetLastError();
}

}  // namespace specinfer
