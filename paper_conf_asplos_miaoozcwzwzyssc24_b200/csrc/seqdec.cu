// seqdec.cu — NEXT-1: sequence-based parallel decoding, the baseline SpecInfer's tree-based
// parallel decoding replaces (§4.2, Fig. 4 left L682, §6.5).
//
// Sequence-based decoding decomposes the token tree into its root-to-leaf sequences and gives
// every sequence its own KV cache (prefix + its own tokens), so that sequences never conflict;
// each sequence is then an ordinary causal (chain) attention problem.  Two kernels build that
// baseline from a tree batch; the attention itself is specinfer_tree_attention run over the
// sequence batch with chain trees (one launch for all sequences, or one launch per sequence as
// in Fig. 4's "Kernel 1 / 2 / 3").  The prefix is re-read once per leaf instead of once per
// request: that redundant traffic is what the ablation (tools/fig11_ablation.py) measures.
//
//   leaf_paths_kernel     one block per request: leaves in index order (= DFS order for a DFS
//                         linearised tree, Fig. 2), each with its root path
//   sequence_pack_kernel  one block per (sequence, kv-head): copies the request's committed
//                         prefix and the path nodes' K/V rows into the sequence's own cache
//                         (16-byte vector copies), the path nodes' q rows, and writes the chain
//                         tree arrays of the sequence
#include "common.cuh"

namespace specinfer {

__global__ void __launch_bounds__(256) leaf_paths_kernel(const int32_t *__restrict__ parent,
                                                         const int32_t *__restrict__ n_nodes, int Nmax, int Dmax,
                                                         int32_t *__restrict__ paths, int32_t *__restrict__ path_len,
                                                         int32_t *__restrict__ n_leaves, int32_t *__restrict__ status) {
    const int b = blockIdx.x;
    __shared__ int32_t s_par[kMaxNodes];
    __shared__ int32_t s_child[kMaxNodes];
    __shared__ int32_t s_rank[kMaxNodes];
    __shared__ int s_bad;
    const int n = n_nodes[b];
    if (threadIdx.x == 0) s_bad = (n < 1 || n > Nmax) ? 1 : 0;
    for (int i = threadIdx.x; i < Nmax; i += blockDim.x) s_child[i] = 0;
    __syncthreads();
    const bool n_ok = !s_bad;
    for (int i = threadIdx.x; n_ok && i < n; i += blockDim.x) {
        const int p = parent[(size_t)b * Nmax + i];
        s_par[i] = p;
        if (i == 0 ? p != -1 : (p < 0 || p >= i)) atomicOr(&s_bad, 1);
        else if (i > 0) s_child[p] = 1;
    }
    __syncthreads();
    // rank of each leaf among the leaves (exclusive count of leaves with a lower index)
    if (threadIdx.x == 0) {
        int c = 0;
        if (!s_bad)
            for (int i = 0; i < n; ++i) {
                s_rank[i] = c;
                c += s_child[i] ? 0 : 1;
            }
        n_leaves[b] = s_bad ? 0 : c;
        if (s_bad && status) atomicOr(status, kStatusBadTree);
    }
    __syncthreads();
    const int Lp = Dmax + 1;
    for (int i = threadIdx.x; i < Nmax; i += blockDim.x) {
        // clear this request's rows so unused leaf slots read as empty (-1 / 0)
        for (int j = 0; j < Lp; ++j) paths[((size_t)b * Nmax + i) * Lp + j] = -1;
        path_len[(size_t)b * Nmax + i] = 0;
    }
    __syncthreads();
    for (int i = threadIdx.x; !s_bad && i < n; i += blockDim.x) {
        if (s_child[i]) continue;
        int d = 0;
        for (int u = i; u >= 0; u = s_par[u]) ++d;  // path length = depth + 1
        if (d > Lp) {
            atomicOr(&s_bad, 1);
            continue;
        }
        int32_t *row = paths + ((size_t)b * Nmax + s_rank[i]) * Lp;
        int j = d - 1;
        for (int u = i; u >= 0; u = s_par[u]) row[j--] = u;
        path_len[(size_t)b * Nmax + s_rank[i]] = d;
    }
    __syncthreads();
    if (threadIdx.x == 0 && s_bad && n_ok) {
        // depth > Dmax found while writing paths
        n_leaves[b] = 0;
        if (status) atomicOr(status, kStatusBadTree);
    }
}

__global__ void __launch_bounds__(256) sequence_pack_kernel(
    int Nmax, int Dmax, int Hq, int Hkv, int Smax, int seq_smax, const int32_t *__restrict__ seq_map,
    const int32_t *__restrict__ paths, const int32_t *__restrict__ path_len, const int32_t *__restrict__ prefix_len,
    const uint4 *__restrict__ q, const uint4 *__restrict__ k, const uint4 *__restrict__ v, uint4 *__restrict__ q_seq,
    uint4 *__restrict__ k_seq, uint4 *__restrict__ v_seq, int32_t *__restrict__ seq_parent,
    int32_t *__restrict__ seq_depth, int32_t *__restrict__ seq_prefix, int32_t *__restrict__ seq_n) {
    const int s = blockIdx.x, g = blockIdx.y;
    const int b = seq_map[2 * s], leaf = seq_map[2 * s + 1];
    const int Lp = Dmax + 1;
    const int P = prefix_len[b];
    const int len = path_len[(size_t)b * Nmax + leaf];
    const int32_t *path = paths + ((size_t)b * Nmax + leaf) * Lp;
    constexpr int kRowVec = kHeadDim * 2 / 16;  // 16 uint4 per 128-dim bf16 row
    const uint4 *ks = k + ((size_t)b * Hkv + g) * Smax * kRowVec;
    const uint4 *vs = v + ((size_t)b * Hkv + g) * Smax * kRowVec;
    uint4 *kd = k_seq + ((size_t)s * Hkv + g) * seq_smax * kRowVec;
    uint4 *vd = v_seq + ((size_t)s * Hkv + g) * seq_smax * kRowVec;
    // committed prefix (the copy sequence-based decoding keeps per sequence), then the path rows
    const int rows = P + len;
    for (int idx = threadIdx.x; idx < rows * kRowVec; idx += blockDim.x) {
        const int r = idx / kRowVec, c = idx - r * kRowVec;
        const int src = r < P ? r : P + path[r - P];
        kd[(size_t)r * kRowVec + c] = __ldg(ks + (size_t)src * kRowVec + c);
        vd[(size_t)r * kRowVec + c] = __ldg(vs + (size_t)src * kRowVec + c);
    }
    // q rows of the path nodes, heads of this kv-group
    const int G = Hq / Hkv;
    for (int idx = threadIdx.x; idx < len * G * kRowVec; idx += blockDim.x) {
        const int j = idx / (G * kRowVec), rem = idx - j * G * kRowVec;
        const int h = g * G + rem / kRowVec, c = rem % kRowVec;
        q_seq[(((size_t)s * Lp + j) * Hq + h) * kRowVec + c] =
            __ldg(q + (((size_t)b * Nmax + path[j]) * Hq + h) * kRowVec + c);
    }
    if (g == 0) {
        for (int j = threadIdx.x; j < Lp; j += blockDim.x) {
            seq_parent[(size_t)s * Lp + j] = j - 1;  // chain: node j's parent is j - 1
            seq_depth[(size_t)s * Lp + j] = j;
        }
        if (threadIdx.x == 0) {
            seq_prefix[s] = P;
            seq_n[s] = len;
        }
    }
}

cudaError_t launch_leaf_paths(const specinfer_shape_t &s, const int32_t *parent, const int32_t *n_nodes,
                              int32_t *paths, int32_t *path_len, int32_t *n_leaves, int32_t *status,
                              cudaStream_t stream) {
    leaf_paths_kernel<<<s.batch, 256, 0, stream>>>(parent, n_nodes, s.max_nodes, s.max_depth, paths, path_len,
                                                   n_leaves, status);
    return cudaGetLastError();
}

cudaError_t launch_sequence_pack(const specinfer_shape_t &s, int num_seqs, int seq_max_seq, const int32_t *seq_map,
                                 const int32_t *paths, const int32_t *path_len, const int32_t *prefix_len,
                                 const void *q, const void *k, const void *v, void *q_seq, void *k_seq, void *v_seq,
                                 int32_t *seq_parent, int32_t *seq_depth, int32_t *seq_prefix, int32_t *seq_n,
                                 cudaStream_t stream) {
    if (num_seqs == 0) return cudaSuccess;
    sequence_pack_kernel<<<dim3(num_seqs, s.num_kv_heads), 256, 0, stream>>>(
        s.max_nodes, s.max_depth, s.num_q_heads, s.num_kv_heads, s.max_seq, seq_max_seq, seq_map, paths, path_len,
        prefix_len, reinterpret_cast<const uint4 *>(q), reinterpret_cast<const uint4 *>(k),
        reinterpret_cast<const uint4 *>(v), reinterpret_cast<uint4 *>(q_seq), reinterpret_cast<uint4 *>(k_seq),
        reinterpret_cast<uint4 *>(v_seq), seq_parent, seq_depth, seq_prefix, seq_n);
    return cudaGetLastError();
}

}  // namespace specinfer
