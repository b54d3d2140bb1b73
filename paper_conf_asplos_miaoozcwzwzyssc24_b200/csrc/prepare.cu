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

__global__ void __launch_bounds__(256) tree_validate_bitsets_kernel(
    const int32_t *__restrict__ parent, const int32_t *__restrict__ depth,
    const int32_t *__restrict__ prefix_len, const int32_t *__restrict__ n_nodes, int Nmax,
    int max_depth, int Smax, int32_t *__restrict__ status, int32_t *__restrict__ req_ok,
    uint32_t *__restrict__ anc, uint32_t *__restrict__ desc) {
    const int b = blockIdx.x;
    __shared__ int32_t s_par[kMaxNodes];
    __shared__ uint32_t s_anc[kMaxNodes][kBitWords];
    __shared__ int s_bad;
    const int n = n_nodes[b];
    const int P = prefix_len[b];
    if (threadIdx.x == 0) {
        int bad = (n < 1 || n > Nmax || P < 0 || (long long)P + n > Smax) ? 1 : 0;
        s_bad = bad;
    }
    __syncthreads();
    const bool n_ok = !s_bad;
    for (int i = threadIdx.x; i < Nmax; i += blockDim.x) {
        const int p = parent[(size_t)b * Nmax + i];
        s_par[i] = p;
        if (n_ok && i < n) {
            const int d = depth[(size_t)b * Nmax + i];
            bool bad;
            if (i == 0) {
                bad = (p != -1) || (d != 0);
            } else {
                bad = (p < 0) || (p >= i) || (d > max_depth) ||
                      (d != depth[(size_t)b * Nmax + p] + 1);
            }
            if (bad) atomicOr(&s_bad, 1);
        }
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
                w[u >> 5] |= 1u << (u & 31);
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
    // descendant-or-self bitsets: desc[j] bit i  <=>  anc[i] bit j
    for (int j = threadIdx.x; j < Nmax; j += blockDim.x) {
        uint32_t w[kBitWords];
#pragma unroll
        for (int k = 0; k < kBitWords; ++k) w[k] = 0;
        if (ok && j < n) {
            for (int i = j; i < n; ++i)
                if ((s_anc[i][j >> 5] >> (j & 31)) & 1u) w[i >> 5] |= 1u << (i & 31);
        }
#pragma unroll
        for (int k = 0; k < kBitWords; ++k) desc[((size_t)b * Nmax + j) * kBitWords + k] = w[k];
    }
    if (threadIdx.x == 0) {
        req_ok[b] = ok ? 1 : 0;
        if (!ok) atomicOr(status, kStatusBadTree);
    }
}

// Single block: tiles per item, exclusive scan, total; zero the split/verify counters.
__global__ void __launch_bounds__(1024) schedule_kernel(
    const int32_t *__restrict__ prefix_len, const int32_t *__restrict__ n_nodes,
    const int32_t *__restrict__ req_ok, int B, int Hkv, int chunks, int npc,
    int32_t *__restrict__ item_start, uint32_t *__restrict__ item_cnt,
    uint32_t *__restrict__ verify_cnt, int32_t *__restrict__ status) {
    const int n_items = B * Hkv * chunks;
    const int per = (n_items + blockDim.x - 1) / blockDim.x;
    const int lo = threadIdx.x * per;
    const int hi = min(n_items, lo + per);
    auto tiles_of = [&](int x) -> int {
        const int c = x % chunks;
        const int b = x / (chunks * Hkv);
        if (!req_ok[b]) return 0;
        const int n = n_nodes[b];
        if (c * npc >= n) return 0;
        return (prefix_len[b] + n + kKeyTile - 1) / kKeyTile;
    };
    int local = 0;
    for (int x = lo; x < hi; ++x) local += tiles_of(x);
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
    for (int x = lo; x < hi; ++x) {
        item_start[x] = run;
        run += tiles_of(x);
        item_cnt[x] = 0u;
    }
    if (threadIdx.x == blockDim.x - 1) {
        item_start[n_items] = run;
        status[1] = run;
    }
    for (int b = threadIdx.x; b < B; b += blockDim.x) verify_cnt[b] = 0u;
}

cudaError_t launch_tree_prepare(const specinfer_shape_t &s, const WsLayout &w,
                                const int32_t *parent, const int32_t *depth,
                                const int32_t *prefix_len, const int32_t *n_nodes, char *ws,
                                cudaStream_t stream) {
    int32_t *status = reinterpret_cast<int32_t *>(ws + w.status);
    cudaError_t e = cudaMemsetAsync(status, 0, 64 * 4, stream);
    if (e != cudaSuccess) return e;
    tree_validate_bitsets_kernel<<<s.batch, 256, 0, stream>>>(
        parent, depth, prefix_len, n_nodes, s.max_nodes, s.max_depth, s.max_seq, status,
        reinterpret_cast<int32_t *>(ws + w.req_ok), reinterpret_cast<uint32_t *>(ws + w.anc),
        reinterpret_cast<uint32_t *>(ws + w.desc));
    e = cudaGetLastError();
    if (e != cudaSuccess) return e;
    schedule_kernel<<<1, 1024, 0, stream>>>(
        prefix_len, n_nodes, reinterpret_cast<int32_t *>(ws + w.req_ok), s.batch,
        s.num_kv_heads, w.chunks, w.npc, reinterpret_cast<int32_t *>(ws + w.item_start),
        reinterpret_cast<uint32_t *>(ws + w.item_cnt),
        reinterpret_cast<uint32_t *>(ws + w.verify_cnt), status);
    return cudaGetLastError();
}

}  // namespace specinfer
