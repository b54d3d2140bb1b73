// construct.cu — NEXT-2: token-tree construction on the GPU (§3;
// Fig. 2, Fig. 3), the step that produces the hot path's input trees.
//
//   expansion_topology_kernel  the static expansion <k1..km> (L476-483): step i gives every node
//                              at depth i-1 k_i children.  Node ids in DFS preorder (Fig. 2
//                              "Linearization", L314): with S_d = 1 + k_{d+1} S_{d+1} nodes in a
//                              subtree rooted at depth d, child j of node u (depth d) is
//                              u + 1 + j S_{d+1}; each thread decodes one node id top-down.
//   expand_step_kernel         one expansion step: one CTA per (frontier node, request) reads the
//                              SSM's logits for that node, takes its top-k tokens (descending
//                              logit, lowest token id on ties, reading R7) for the node's k
//                              children in DFS order, and optionally writes q = softmax(l / T)
//                              as the draft distribution of every child (reading R12:
//                              draft_probs[c] = the distribution c was drawn from).
//   tree_merge_kernel          token tree merge (Def. 3.2): the union of the input
//                              trees' sequences S_u as one trie, children in first-appearance
//                              order, relabelled in DFS preorder; one CTA per request (a few
//                              hundred nodes: the build is a short sequential trie insertion by
//                              one thread, the relabel a DFS with an explicit stack).
#include "common.cuh"

namespace specinfer {

constexpr int kMaxExpansion = 16;
struct Expansion {
    int m;
    int k[kMaxExpansion];
    int sub[kMaxExpansion + 1];  // sub[d] = size of a subtree rooted at depth d
};

__global__ void expansion_topology_kernel(Expansion e, int B, int Nmax, int32_t *__restrict__ parent,
                                          int32_t *__restrict__ depth, int32_t *__restrict__ n_nodes) {
    const int n = e.sub[0];
    const long long total = (long long)B * Nmax;
    for (long long idx = (long long)blockIdx.x * blockDim.x + threadIdx.x; idx < total;
         idx += (long long)gridDim.x * blockDim.x) {
        const int b = (int)(idx / Nmax), i = (int)(idx % Nmax);
        int par = -1, d = 0;
        if (i < n) {
            int u = 0;
            while (u != i) {  // descend from the root to the subtree that holds i
                const int j = (i - u - 1) / e.sub[d + 1];
                par = u;
                u = u + 1 + j * e.sub[d + 1];
                ++d;
            }
        }
        parent[idx] = i < n ? par : -1;
        depth[idx] = i < n ? d : 0;
        if (i == 0) n_nodes[b] = n;
    }
}

constexpr int kExpandThreads = 512;
constexpr int kMaxK = 8;  // children per node a single expansion step may create

struct TopEntry {
    float v;
    int i;
};
__device__ __forceinline__ bool better(const TopEntry &a, const TopEntry &b) {
    return a.v > b.v || (a.v == b.v && a.i >= 0 && (b.i < 0 || a.i < b.i));
}

__global__ void __launch_bounds__(kExpandThreads) expand_step_kernel(
    int level, const float *__restrict__ ssm_logits, int F, int V, float invT, const int32_t *__restrict__ parent,
    const int32_t *__restrict__ depth, const int32_t *__restrict__ n_nodes, int Nmax, int32_t *__restrict__ tokens,
    float *__restrict__ draft_probs, int32_t *__restrict__ status) {
    const int f = blockIdx.x, b = blockIdx.y;
    __shared__ int s_u, s_nc, s_child[kMaxK + 1];
    __shared__ TopEntry s_cand[kExpandThreads];
    __shared__ float s_red[32];
    const int n = n_nodes[b];
    if (threadIdx.x == 0) {
        // the f-th node of depth `level` in DFS order, and its children in DFS order
        int u = -1, cnt = 0;
        for (int i = 0; i < n; ++i)
            if (depth[(size_t)b * Nmax + i] == level && cnt++ == f) {
                u = i;
                break;
            }
        int nc = 0;
        if (u >= 0)
            for (int c = u + 1; c < n; ++c)
                if (parent[(size_t)b * Nmax + c] == u) {
                    if (nc < kMaxK) s_child[nc] = c;
                    ++nc;
                }
        if (nc > kMaxK) {
            if (status) atomicOr(status, kStatusBadTree);
            nc = 0;
        }
        s_u = u;
        s_nc = nc;
    }
    __syncthreads();
    const int nc = s_nc;
    if (s_u < 0 || nc == 0) return;
    const float *row = ssm_logits + ((size_t)b * F + f) * V;
    // per-thread top-nc over a strided slice, then nc rounds of block extraction
    TopEntry top[kMaxK];
#pragma unroll
    for (int j = 0; j < kMaxK; ++j) top[j] = TopEntry{-INFINITY, -1};
    float mx = -INFINITY;
    for (int x = threadIdx.x; x < V; x += kExpandThreads) {
        const float v = __ldg(row + x);
        mx = fmaxf(mx, v);
        TopEntry e{v, x};
        if (better(e, top[nc - 1])) {
            // insertion into the sorted list (nc <= 8)
#pragma unroll
            for (int j = kMaxK - 1; j >= 0; --j) {
                if (j >= nc) continue;
                if (j > 0 && better(e, top[j - 1])) {
                    top[j] = top[j - 1];
                } else {
                    top[j] = e;
                    break;
                }
            }
        }
    }
    // block max (for the softmax) and the candidate lists
#pragma unroll
    for (int o = 16; o >= 1; o >>= 1) mx = fmaxf(mx, __shfl_xor_sync(0xffffffffu, mx, o));
    if ((threadIdx.x & 31) == 0) s_red[threadIdx.x >> 5] = mx;
    __syncthreads();
    if (threadIdx.x < 32) {
        float m2 = threadIdx.x < kExpandThreads / 32 ? s_red[threadIdx.x] : -INFINITY;
#pragma unroll
        for (int o = 16; o >= 1; o >>= 1) m2 = fmaxf(m2, __shfl_xor_sync(0xffffffffu, m2, o));
        if (threadIdx.x == 0) s_red[0] = m2;
    }
    __syncthreads();
    const float rmax = s_red[0];
    __syncthreads();
    int head = 0;  // this thread's next unconsumed candidate
    for (int r = 0; r < nc; ++r) {
        TopEntry c{-INFINITY, -1};  // top[head] (unrolled select: top[] stays in registers)
#pragma unroll
        for (int j = 0; j < kMaxK; ++j)
            if (j == head && j < nc) c = top[j];
        s_cand[threadIdx.x] = c;
        __syncthreads();
        for (int s = kExpandThreads / 2; s >= 1; s >>= 1) {
            if (threadIdx.x < s && better(s_cand[threadIdx.x + s], s_cand[threadIdx.x]))
                s_cand[threadIdx.x] = s_cand[threadIdx.x + s];
            __syncthreads();
        }
        const TopEntry w = s_cand[0];
        if (threadIdx.x == 0) tokens[(size_t)b * Nmax + s_child[r]] = w.i;
        if (c.i == w.i && c.i >= 0) ++head;  // the winner came from this thread
        __syncthreads();
    }
    if (draft_probs == nullptr) return;
    // q = softmax(l / T): sum, then the normalised row into every child's draft row
    float z = 0.f;
    for (int x = threadIdx.x; x < V; x += kExpandThreads) z += __expf((__ldg(row + x) - rmax) * invT);
#pragma unroll
    for (int o = 16; o >= 1; o >>= 1) z += __shfl_xor_sync(0xffffffffu, z, o);
    if ((threadIdx.x & 31) == 0) s_red[threadIdx.x >> 5] = z;
    __syncthreads();
    if (threadIdx.x == 0) {
        float t = 0.f;
        for (int w = 0; w < kExpandThreads / 32; ++w) t += s_red[w];
        s_red[0] = t;
    }
    __syncthreads();
    const float invZ = 1.0f / s_red[0];
    for (int x = threadIdx.x; x < V; x += kExpandThreads) {
        const float q = __expf((__ldg(row + x) - rmax) * invT) * invZ;
        for (int j = 0; j < nc; ++j) draft_probs[((size_t)b * Nmax + s_child[j]) * V + x] = q;
    }
}

// Tree merge.  Inputs: T trees per request, each in topological order, [B][T][Nin] parent /
// tokens, n_in[B][T] (0 = absent).  All input roots must carry the same token (the last verified
// token, R6).  Output: the merged tree in DFS preorder (children in first-appearance order), and
// node_map[b][t][i] = merged id of input node i (-1 for i >= n_in).
__global__ void __launch_bounds__(128) tree_merge_kernel(int T, int Nin, const int32_t *__restrict__ in_parent,
                                                         const int32_t *__restrict__ in_tokens,
                                                         const int32_t *__restrict__ in_n, int Nmax, int Dmax,
                                                         int32_t *__restrict__ parent, int32_t *__restrict__ depth,
                                                         int32_t *__restrict__ tokens, int32_t *__restrict__ n_nodes,
                                                         int32_t *__restrict__ node_map, int32_t *__restrict__ status) {
    const int b = blockIdx.x;
    __shared__ int32_t s_tok[kMaxNodes], s_par[kMaxNodes], s_first[kMaxNodes], s_next[kMaxNodes], s_last[kMaxNodes];
    __shared__ int32_t s_dfs[kMaxNodes], s_stack[kMaxNodes];
    __shared__ int s_n, s_bad;
    if (threadIdx.x == 0) {
        int nm = 0, bad = 0;
        for (int t = 0; t < T && !bad; ++t) {
            const int nt = in_n[(size_t)b * T + t];
            if (nt < 0 || nt > Nin) {
                bad = 1;
                break;
            }
            const int32_t *ip = in_parent + ((size_t)b * T + t) * Nin;
            const int32_t *it = in_tokens + ((size_t)b * T + t) * Nin;
            int32_t *map = node_map + ((size_t)b * T + t) * Nin;
            for (int i = 0; i < nt && !bad; ++i) {
                const int p = ip[i], tok = it[i];
                int mp;
                if (i == 0) {
                    if (p != -1) { bad = 1; break; }
                    if (nm == 0) {
                        s_tok[0] = tok;
                        s_par[0] = -1;
                        s_first[0] = s_next[0] = s_last[0] = -1;
                        nm = 1;
                    } else if (s_tok[0] != tok) {
                        bad = 1;
                        break;
                    }
                    map[0] = 0;
                    continue;
                }
                if (p < 0 || p >= i) { bad = 1; break; }
                mp = map[p];
                // find the child of mp with this token, else append it (first-appearance order)
                int c = s_first[mp];
                while (c >= 0 && s_tok[c] != tok) c = s_next[c];
                if (c < 0) {
                    if (nm >= Nmax) { bad = 1; break; }
                    c = nm++;
                    s_tok[c] = tok;
                    s_par[c] = mp;
                    s_first[c] = s_next[c] = s_last[c] = -1;
                    if (s_first[mp] < 0) s_first[mp] = c;
                    else s_next[s_last[mp]] = c;
                    s_last[mp] = c;
                }
                map[i] = c;
            }
            for (int i = nt; i < Nin; ++i) map[i] = -1;
        }
        // DFS preorder relabel
        if (!bad && nm > 0) {
            int sp = 0, k = 0;
            s_stack[sp++] = 0;
            while (sp > 0) {
                const int u = s_stack[--sp];
                s_dfs[u] = k++;
                // push children in reverse so the first child is visited first
                int cnt = 0;
                for (int c = s_first[u]; c >= 0; c = s_next[c]) ++cnt;
                int pos = sp + cnt;
                for (int c = s_first[u]; c >= 0; c = s_next[c]) s_stack[--pos] = c;
                sp += cnt;
            }
        }
        s_n = bad ? 0 : nm;
        s_bad = bad;
    }
    __syncthreads();
    // depths (and the Dmax check) BEFORE any output is written: a merged tree deeper than Dmax is
    // reported like every other bad input (n_nodes 0, padding rows, node_map -1).  s_stack is free.
    const int nm = s_n;
    for (int u = threadIdx.x; u < nm; u += blockDim.x) {
        int dep = 0;
        for (int x = s_par[u]; x >= 0; x = s_par[x]) ++dep;
        s_stack[u] = dep;
        if (dep > Dmax) atomicOr(&s_bad, 1);
    }
    __syncthreads();
    const int nw = s_bad ? 0 : nm;
    for (int i = threadIdx.x; i < Nmax; i += blockDim.x) {
        parent[(size_t)b * Nmax + i] = -1;
        depth[(size_t)b * Nmax + i] = 0;
        tokens[(size_t)b * Nmax + i] = -1;
    }
    __syncthreads();
    for (int u = threadIdx.x; u < nw; u += blockDim.x) {
        const int d = s_dfs[u];
        parent[(size_t)b * Nmax + d] = s_par[u] >= 0 ? s_dfs[s_par[u]] : -1;
        depth[(size_t)b * Nmax + d] = s_stack[u];
        tokens[(size_t)b * Nmax + d] = s_tok[u];
    }
    // node_map: trie ids -> DFS ids
    for (int idx = threadIdx.x; idx < T * Nin; idx += blockDim.x) {
        int32_t *m = node_map + (size_t)b * T * Nin + idx;
        const int v = *m;
        if (!nw) *m = -1;
        else if (v >= 0) *m = s_dfs[v];
    }
    if (threadIdx.x == 0) {
        n_nodes[b] = nw;
        if (s_bad && status) atomicOr(status, kStatusBadTree);
    }
}

cudaError_t launch_expansion_topology(const specinfer_shape_t &s, const int32_t *ks, int m, int32_t *parent,
                                      int32_t *depth, int32_t *n_nodes, cudaStream_t stream) {
    Expansion e{};
    e.m = m;
    for (int i = 0; i < m; ++i) e.k[i] = ks[i];
    e.sub[m] = 1;
    for (int d = m - 1; d >= 0; --d) e.sub[d] = 1 + ks[d] * e.sub[d + 1];
    const long long total = (long long)s.batch * s.max_nodes;
    const int blocks = (int)((total + 255) / 256);
    expansion_topology_kernel<<<blocks, 256, 0, stream>>>(e, s.batch, s.max_nodes, parent, depth, n_nodes);
    return cudaGetLastError();
}

cudaError_t launch_expand_step(const specinfer_shape_t &s, int level, const float *ssm_logits, int F, float temperature,
                               const int32_t *parent, const int32_t *depth, const int32_t *n_nodes, int32_t *tokens,
                               float *draft_probs, int32_t *status, cudaStream_t stream) {
    expand_step_kernel<<<dim3(F, s.batch), kExpandThreads, 0, stream>>>(level, ssm_logits, F, s.vocab,
                                                                         1.0f / temperature, parent, depth, n_nodes,
                                                                         s.max_nodes, tokens, draft_probs, status);
    return cudaGetLastError();
}

cudaError_t launch_tree_merge(const specinfer_shape_t &s, int T, int Nin, const int32_t *in_parent,
                              const int32_t *in_tokens, const int32_t *in_n, int32_t *parent, int32_t *depth,
                              int32_t *tokens, int32_t *n_nodes, int32_t *node_map, int32_t *status,
                              cudaStream_t stream) {
    tree_merge_kernel<<<s.batch, 128, 0, stream>>>(T, Nin, in_parent, in_tokens, in_n, s.max_nodes, s.max_depth,
                                                   parent, depth, tokens, n_nodes, node_map, status);
    return cudaGetLastError();
}

}  // namespace specinfer
