// rope.cu — NEXT-4: rotary position encoding of the token tree at position P_b + depth[i], sm_100a.
//
// Reading A4 (DESIGN R29): Def. 4.1 defines node u's output as
// Attention(S_u), S_u = committed prefix + root path, where u is token number depth(u) after the
// prefix; a position-encoded model therefore encodes node i of request b at P_b + depth[i] (siblings
// share a position), not at its tree index.  One launch rotates the tree queries q[b][i][h][:]
// (i < n_b) and the tree keys k_cache[b][g][P_b + i][:] in place, so that the committed cache keeps
// the invariant "slot s holds a key encoded at position s" after specinfer_kv_commit (path[j] has
// depth j).  Rotate-half pairing (dims d and d + 64), theta_d = fp32(base^(-2d/128)), angle =
// fp32(pos) * theta_d in fp32 (round to nearest), sin/cos of that angle, rotation in fp32.
//
// HBM-bound and tiny (q + tree keys: ~2 * 256 B per row): one warp per 256-byte row, lane l owns
// pairs d = 2l, 2l + 1 (4-byte loads, 128 B per warp and half).
#include "common.cuh"

namespace specinfer {

__global__ void __launch_bounds__(256) tree_rope_kernel(__nv_bfloat16 *__restrict__ q, __nv_bfloat16 *__restrict__ k,
                                                        const int32_t *__restrict__ prefix_len,
                                                        const int32_t *__restrict__ depth,
                                                        const int32_t *__restrict__ n_nodes, int B, int Nmax, int Hq,
                                                        int Hkv, int Smax, float base) {
    __shared__ float theta[kHeadDim / 2];
    if (threadIdx.x < kHeadDim / 2)
        theta[threadIdx.x] = (float)pow((double)base, -2.0 * (double)threadIdx.x / (double)kHeadDim);
    __syncthreads();
    const long long row = (long long)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
    const long long q_rows = q ? (long long)B * Nmax * Hq : 0;
    const long long k_rows = k ? (long long)B * Hkv * Nmax : 0;
    if (row >= q_rows + k_rows) return;
    const int lane = threadIdx.x & 31;
    int b, i;
    __nv_bfloat16 *x;
    if (row < q_rows) {  // q [B][Nmax][Hq][128]
        b = (int)(row / ((long long)Nmax * Hq));
        i = (int)((row / Hq) % Nmax);
        x = q + (size_t)row * kHeadDim;
    } else {             // k_cache [B][Hkv][Smax][128], tree slot P_b + i
        const long long r = row - q_rows;
        b = (int)(r / ((long long)Hkv * Nmax));
        const int g = (int)((r / Nmax) % Hkv);
        i = (int)(r % Nmax);
        const int P = prefix_len[b];
        x = k + (((size_t)b * Hkv + g) * Smax + (size_t)(P + i)) * kHeadDim;
    }
    const int n = n_nodes[b], P = prefix_len[b];
    if (n < 1 || n > Nmax || P < 0 || P + n > Smax || i >= n) return;  // outside the tree: untouched
    const float pos = (float)(P + depth[(size_t)b * Nmax + i]);
    const int d = 2 * lane;
    __nv_bfloat162 *plo = reinterpret_cast<__nv_bfloat162 *>(x + d);
    __nv_bfloat162 *phi = reinterpret_cast<__nv_bfloat162 *>(x + kHeadDim / 2 + d);
    const float2 lo = __bfloat1622float2(*plo), hi = __bfloat1622float2(*phi);
    float s0, c0, s1, c1;
    sincosf(__fmul_rn(pos, theta[d]), &s0, &c0);
    sincosf(__fmul_rn(pos, theta[d + 1]), &s1, &c1);
    *plo = __floats2bfloat162_rn(fmaf(lo.x, c0, -hi.x * s0), fmaf(lo.y, c1, -hi.y * s1));
    *phi = __floats2bfloat162_rn(fmaf(hi.x, c0, lo.x * s0), fmaf(hi.y, c1, lo.y * s1));
}

cudaError_t launch_tree_rope(const specinfer_shape_t &s, void *q, void *k, const int32_t *prefix_len,
                             const int32_t *depth, const int32_t *n_nodes, float base, cudaStream_t stream) {
    const long long rows = (q ? (long long)s.batch * s.max_nodes * s.num_q_heads : 0) +
                           (k ? (long long)s.batch * s.num_kv_heads * s.max_nodes : 0);
    if (rows == 0) return cudaSuccess;
    const long long blocks = (rows + 7) / 8;
    tree_rope_kernel<<<(unsigned)blocks, 256, 0, stream>>>(
        reinterpret_cast<__nv_bfloat16 *>(q), reinterpret_cast<__nv_bfloat16 *>(k), prefix_len, depth, n_nodes,
        s.batch, s.max_nodes, s.num_q_heads, s.num_kv_heads, s.max_seq, base);
    return cudaGetLastError();
}

}  // namespace specinfer
