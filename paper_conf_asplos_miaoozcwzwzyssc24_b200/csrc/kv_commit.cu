// kv_commit.cu — K6 depth-first KV-cache commit, sm_100a.
//
// SpecInfer keeps ONE KV cache for all sequences of the tree; after
// verification the accepted root path becomes the committed sequence.  With the tree stored
// in topology order at slots P_b + i (L659-661), committing path[0..n-1] means
//     slot P_b + j  <-  slot P_b + path[j]   for j = 0..n-1   (path[0] = root = 0),
// then P_b += n (readings R6, R21).  Because path[] is strictly increasing and path[j] >= j,
// processing j in increasing order never overwrites a row that a later j still has to read,
// so each warp copies its rows in order without staging.  Rows with path[j] == j (the leftmost
// branch, stored in place) are skipped.  One warp per (layer, request, kv-head); lanes 0-15
// move the K row and lanes 16-31 the V row, 16 bytes each (128-bit coalesced).
#include "common.cuh"

namespace specinfer {

// Number of path rows of request b that can be committed: n_acc clamped to the path row length,
// then to the longest prefix of the path that is a valid DFS commit (path[0] = 0, strictly
// increasing, so path[j] >= j, and P + path[j] < Smax).  The verifiers always produce valid paths;
// a caller-built path that breaks the contract is committed only up to its first bad row, by the
// copy and the prefix update alike (include/specinfer.h).
__device__ __forceinline__ int commit_len(const int32_t *path, int n, int P, int Smax, int path_len) {
    n = min(n, path_len);
    if (n <= 0) return 0;
    if (path[0] != 0 || P >= Smax) return 0;
    int j = 1;
    for (; j < n; ++j) {
        const int src = path[j];
        if (src <= path[j - 1] || P + src >= Smax) break;
    }
    return j;
}

// paged KV (NEXT-4): slot s of request b, kv-head g lives at row (page_table[b][s/128] Hkv + g) 128
// + s % 128 of the layer's [num_pages][Hkv][128][128] pages; page_table == nullptr: contiguous.
__global__ void __launch_bounds__(256) kv_commit_copy_kernel(
    __nv_bfloat16 *__restrict__ k_all, __nv_bfloat16 *__restrict__ v_all, const int32_t *__restrict__ prefix_len,
    const int32_t *__restrict__ acc_nodes, const int32_t *__restrict__ n_acc, int L, int B, int Hkv, int Smax,
    long long layer_stride, int path_len, const int32_t *__restrict__ page_table, int max_pages) {
    const long long item = (long long)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
    if (item >= (long long)L * B * Hkv) return;
    const int lane = threadIdx.x & 31;
    const int g = (int)(item % Hkv);
    const int b = (int)((item / Hkv) % B);
    const int l = (int)(item / ((long long)Hkv * B));
    const int P = prefix_len[b];
    const int32_t *path = acc_nodes + (size_t)b * path_len;
    const int n = commit_len(path, n_acc[b], P, Smax, path_len);
    if (n <= 1) return;
    __nv_bfloat16 *layer = (lane < 16 ? k_all : v_all) + (size_t)l * layer_stride;
    const int col = (lane & 15) * 8;  // 8 bf16 = 16 bytes
    auto row = [&](int slot) -> __nv_bfloat16 * {
        if (page_table == nullptr) return layer + (((size_t)b * Hkv + g) * Smax + slot) * kHeadDim + col;
        const int page = page_table[(size_t)b * max_pages + slot / kKeyTile];
        return layer + (((size_t)page * Hkv + g) * kKeyTile + slot % kKeyTile) * kHeadDim + col;
    };
    for (int j = 1; j < n; ++j) {
        const int src = path[j];
        if (src == j) continue;
        const uint4 v = *reinterpret_cast<const uint4 *>(row(P + src));
        *reinterpret_cast<uint4 *>(row(P + j)) = v;
    }
}

__global__ void kv_commit_prefix_kernel(int32_t *__restrict__ prefix_len, const int32_t *__restrict__ acc_nodes,
                                        const int32_t *__restrict__ n_acc, int B, int Smax, int path_len) {
    const int b = blockIdx.x * blockDim.x + threadIdx.x;
    if (b < B) prefix_len[b] += commit_len(acc_nodes + (size_t)b * path_len, n_acc[b], prefix_len[b], Smax, path_len);
}

cudaError_t launch_kv_commit(const specinfer_shape_t &s, void *k_all, void *v_all, int32_t *prefix_len,
                             const int32_t *acc_nodes, const int32_t *n_acc, cudaStream_t stream,
                             const int32_t *page_table, int num_pages) {
    const int max_pages = (s.max_seq + kKeyTile - 1) / kKeyTile;
    const long long layer_stride =
        s.layer_stride > 0 ? s.layer_stride
        : page_table     ? (long long)num_pages * s.num_kv_heads * kKeyTile * kHeadDim
                         : (long long)s.batch * s.num_kv_heads * s.max_seq * kHeadDim;
    const long long items = (long long)s.num_layers * s.batch * s.num_kv_heads;
    if (items > 0) {
        const int warps_per_block = 8;
        const long long blocks = (items + warps_per_block - 1) / warps_per_block;
        kv_commit_copy_kernel<<<(unsigned)blocks, warps_per_block * 32, 0, stream>>>(
            reinterpret_cast<__nv_bfloat16 *>(k_all), reinterpret_cast<__nv_bfloat16 *>(v_all), prefix_len,
            acc_nodes, n_acc, s.num_layers, s.batch, s.num_kv_heads, s.max_seq, layer_stride, s.max_depth + 1,
            page_table, max_pages);
        cudaError_t e = cudaGetLastError();
        if (e != cudaSuccess) return e;
    }
    kv_commit_prefix_kernel<<<(s.batch + 255) / 256, 256, 0, stream>>>(prefix_len, acc_nodes, n_acc, s.batch,
                                                                       s.max_seq, s.max_depth + 1);
    return cudaGetLastError();
}

}  // namespace specinfer
