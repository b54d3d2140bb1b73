// verify.cu — K4 verify_greedy and K5 verify_mss, sm_100a.
//
// VerifyGreedy (Alg. 2 lines 16-22, L395-401; §4.3): one CTA per (node, request)
// computes O(u) = argmax_x logits[u][x] with 128-bit loads and a warp-shuffle argmax (lowest
// index on ties, reading R7); the last CTA of a request (counter in the workspace) walks the
// tree from the root.  One launch.
//
// VerifyStochastic = MSS (Alg. 2 lines 24-44, L403-425; Fig. 5): one CTA per request walks at
// most Dmax levels; each level needs one pass over the logits row (softmax statistics), one
// pass per rejected child (residual p <- norm(max(0, p - q)), double-buffered so that an
// all-zero residual keeps p, reading R11) and one pass for the final exponential-race sample.
// The RNG contract (Philox4x32-10, counters from the global request id, node, round, offset;
// readings R9, R15) makes the result independent of batching and GPU count.
#include "common.cuh"

namespace specinfer {

// ------------------------------------------------------------------------------------------
// Philox4x32-10 (Salmon et al., SC'11)
// ------------------------------------------------------------------------------------------
__device__ __forceinline__ uint4 philox4x32_10(uint4 c, uint2 k) {
#pragma unroll
    for (int r = 0; r < 10; ++r) {
        const uint32_t lo0 = 0xD2511F53u * c.x, hi0 = __umulhi(0xD2511F53u, c.x);
        const uint32_t lo1 = 0xCD9E8D57u * c.z, hi1 = __umulhi(0xCD9E8D57u, c.z);
        c = make_uint4(hi1 ^ c.y ^ k.x, lo1, hi0 ^ c.w ^ k.y, lo0);
        k.x += 0x9E3779B9u;
        k.y += 0xBB67AE85u;
    }
    return c;
}

__global__ void philox_debug_kernel(const uint32_t *__restrict__ ck, uint32_t *__restrict__ out, int n) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= n) return;
    const uint32_t *a = ck + (size_t)i * 6;
    const uint4 r = philox4x32_10(make_uint4(a[0], a[1], a[2], a[3]), make_uint2(a[4], a[5]));
    out[(size_t)i * 4 + 0] = r.x;
    out[(size_t)i * 4 + 1] = r.y;
    out[(size_t)i * 4 + 2] = r.z;
    out[(size_t)i * 4 + 3] = r.w;
}

// ------------------------------------------------------------------------------------------
// block reductions
// ------------------------------------------------------------------------------------------
struct ArgMax {
    float v;
    int i;
};

__device__ __forceinline__ ArgMax argmax_merge(ArgMax a, ArgMax b) {
    // larger value wins; equal values -> lower index (R7); index -1 = empty
    if (b.i < 0) return a;
    if (a.i < 0) return b;
    if (b.v > a.v || (b.v == a.v && b.i < a.i)) return b;
    return a;
}

__device__ __forceinline__ ArgMax warp_argmax(ArgMax a) {
#pragma unroll
    for (int o = 16; o >= 1; o >>= 1) {
        ArgMax b;
        b.v = __shfl_xor_sync(0xffffffffu, a.v, o);
        b.i = __shfl_xor_sync(0xffffffffu, a.i, o);
        a = argmax_merge(a, b);
    }
    return a;
}

template <int NTHREADS>
__device__ ArgMax block_argmax(ArgMax a, ArgMax *sh) {
    a = warp_argmax(a);
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    if (lane == 0) sh[wid] = a;
    __syncthreads();
    if (wid == 0) {
        a = (lane < NTHREADS / 32) ? sh[lane] : ArgMax{-INFINITY, -1};
        a = warp_argmax(a);
        if (lane == 0) sh[0] = a;
    }
    __syncthreads();
    a = sh[0];
    __syncthreads();
    return a;
}

template <int NTHREADS>
__device__ float block_sum(float v, float *sh) {
#pragma unroll
    for (int o = 16; o >= 1; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    if (lane == 0) sh[wid] = v;
    __syncthreads();
    if (wid == 0) {
        v = (lane < NTHREADS / 32) ? sh[lane] : 0.f;
#pragma unroll
        for (int o = 16; o >= 1; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
        if (lane == 0) sh[0] = v;
    }
    __syncthreads();
    v = sh[0];
    __syncthreads();
    return v;
}

// ------------------------------------------------------------------------------------------
// K4 verify_greedy
// ------------------------------------------------------------------------------------------
constexpr int kGreedyThreads = 256;

__global__ void __launch_bounds__(kGreedyThreads) verify_greedy_kernel(
    const float *__restrict__ logits, const int32_t *__restrict__ tree_tokens,
    const int32_t *__restrict__ parent, const int32_t *__restrict__ n_nodes,
    const int32_t *__restrict__ req_ok, int32_t *__restrict__ argmax_ws,
    uint32_t *__restrict__ counter, int32_t *__restrict__ acc_nodes, int32_t *__restrict__ acc_tokens,
    int32_t *__restrict__ n_acc, int Nmax, int V, int path_len) {
    const int u = blockIdx.x, b = blockIdx.y;
    const int n = n_nodes[b];
    __shared__ ArgMax sh[32];
    __shared__ int s_last;
    if (!req_ok[b]) {
        if (u == 0) {
            for (int j = threadIdx.x; j < path_len; j += blockDim.x) {
                acc_nodes[(size_t)b * path_len + j] = -1;
                acc_tokens[(size_t)b * path_len + j] = -1;
            }
            if (threadIdx.x == 0) n_acc[b] = 0;
        }
        return;
    }
    if (u >= n) return;
    const float *row = logits + ((size_t)b * Nmax + u) * V;
    ArgMax a{-INFINITY, -1};
    if ((V & 3) == 0) {
        const float4 *row4 = reinterpret_cast<const float4 *>(row);
        const int V4 = V >> 2;
        for (int i = threadIdx.x; i < V4; i += kGreedyThreads) {
            const float4 x = __ldcs(row4 + i);
            const int base = i << 2;
            a = argmax_merge(a, ArgMax{x.x, base});
            a = argmax_merge(a, ArgMax{x.y, base + 1});
            a = argmax_merge(a, ArgMax{x.z, base + 2});
            a = argmax_merge(a, ArgMax{x.w, base + 3});
        }
    } else {
        for (int i = threadIdx.x; i < V; i += kGreedyThreads) a = argmax_merge(a, ArgMax{__ldcs(row + i), i});
    }
    a = block_argmax<kGreedyThreads>(a, sh);
    if (threadIdx.x == 0) {
        argmax_ws[(size_t)b * Nmax + u] = a.i;
        __threadfence();
        const unsigned old = atomicAdd(&counter[b], 1u);
        s_last = (old == (unsigned)(n - 1));
    }
    __syncthreads();
    if (!s_last) return;
    // ---- last CTA of this request: the greedy walk (one warp) ----
    if (threadIdx.x >= 32) return;
    __threadfence();
    const int lane = threadIdx.x;
    const int32_t *par = parent + (size_t)b * Nmax;
    const int32_t *tok = tree_tokens + (size_t)b * Nmax;
    int32_t *an = acc_nodes + (size_t)b * path_len;
    int32_t *at = acc_tokens + (size_t)b * path_len;
    int cur = 0, cnt = 0;
    if (lane == 0) an[0] = 0;
    for (;;) {
        const int o = __ldcg(argmax_ws + (size_t)b * Nmax + cur);
        int next = -1;
        for (int base = cur + 1; base < n && next < 0; base += 32) {
            const int cidx = base + lane;
            const bool hit = cidx < n && par[cidx] == cur && tok[cidx] == o;
            const unsigned m = __ballot_sync(0xffffffffu, hit);
            if (m) next = base + __ffs(m) - 1;
        }
        if (next < 0) {
            if (lane == 0) at[cnt] = o;
            break;
        }
        if (lane == 0) {
            at[cnt] = tok[next];
            an[cnt + 1] = next;
        }
        ++cnt;
        cur = next;
    }
    for (int j = cnt + 1 + lane; j < path_len; j += 32) {
        an[j] = -1;
        at[j] = -1;
    }
    if (lane == 0) {
        n_acc[b] = cnt + 1;
        counter[b] = 0u;  // reusable by the next call on this workspace
    }
}

// ------------------------------------------------------------------------------------------
// K5 verify_mss
// ------------------------------------------------------------------------------------------
constexpr int kMssThreads = 512;

struct MssState {
    int mode;       // 0: p = softmax(logits[u]/T) with stats (mx, invZ); 1: p = buf[cur] * inv
    int cur;        // which residual buffer holds p (mode 1)
    float mx, invZ; // softmax statistics (mode 0)
    float inv;      // 1 / sum of the residual buffer (mode 1)
};

__device__ __forceinline__ float mss_p(const MssState &s, const float *lrow, const float *buf, float invT, int k) {
    return s.mode == 0 ? expf((lrow[k] - s.mx) * invT) * s.invZ : buf[k] * s.inv;
}

__global__ void __launch_bounds__(kMssThreads) verify_mss_kernel(
    const float *__restrict__ logits, const int32_t *__restrict__ tree_tokens,
    const int32_t *__restrict__ parent, const int32_t *__restrict__ n_nodes,
    const float *__restrict__ draft_probs, const int32_t *__restrict__ req_ok, float temperature,
    uint32_t seed_lo, uint32_t seed_hi, uint32_t off, const int32_t *__restrict__ request_ids,
    float *__restrict__ pbuf_all, int32_t *__restrict__ acc_nodes, int32_t *__restrict__ acc_tokens,
    int32_t *__restrict__ n_acc, int Nmax, int V, int path_len) {
    const int b = blockIdx.x;
    const int tid = threadIdx.x;
    int32_t *an = acc_nodes + (size_t)b * path_len;
    int32_t *at = acc_tokens + (size_t)b * path_len;
    for (int j = tid; j < path_len; j += kMssThreads) {
        an[j] = -1;
        at[j] = -1;
    }
    if (!req_ok[b]) {
        if (tid == 0) n_acc[b] = 0;
        return;
    }
    __shared__ int32_t s_par[kMaxNodes], s_tok[kMaxNodes], s_H[kMaxNodes];
    __shared__ float s_red[32];
    __shared__ ArgMax s_am[32];
    __shared__ int s_nh, s_sel;
    __shared__ float s_px;
    const int n = n_nodes[b];
    for (int i = tid; i < n; i += kMssThreads) {
        s_par[i] = parent[(size_t)b * Nmax + i];
        s_tok[i] = tree_tokens[(size_t)b * Nmax + i];
    }
    const uint32_t rid = request_ids ? (uint32_t)request_ids[b] : (uint32_t)b;
    const uint2 key = make_uint2(seed_lo, seed_hi);
    const float invT = 1.0f / temperature;
    float *bufs = pbuf_all + (size_t)b * 2 * V;
    __syncthreads();
    if (tid == 0) an[0] = 0;
    int u = 0, cnt = 0;
    for (;;) {
        const float *lrow = logits + ((size_t)b * Nmax + u) * V;
        // ---- step 1: softmax statistics of logits[u] / T (max, then sum) ----
        float mx = -INFINITY;
        for (int k = tid; k < V; k += kMssThreads) mx = fmaxf(mx, lrow[k]);
#pragma unroll
        for (int o = 16; o >= 1; o >>= 1) mx = fmaxf(mx, __shfl_xor_sync(0xffffffffu, mx, o));
        if ((tid & 31) == 0) s_red[tid >> 5] = mx;
        __syncthreads();
        if (tid < 32) {
            float m2 = tid < kMssThreads / 32 ? s_red[tid] : -INFINITY;
#pragma unroll
            for (int o = 16; o >= 1; o >>= 1) m2 = fmaxf(m2, __shfl_xor_sync(0xffffffffu, m2, o));
            if (tid == 0) s_red[0] = m2;
        }
        __syncthreads();
        mx = s_red[0];
        __syncthreads();
        float z = 0.f;
        for (int k = tid; k < V; k += kMssThreads) z += expf((lrow[k] - mx) * invT);
        z = block_sum<kMssThreads>(z, s_red);
        MssState S{0, 0, mx, 1.0f / z, 0.f};
        uint32_t round = 0;
        // ---- step 2: children of u in ascending order ----
        if (tid == 0) {
            int nh = 0;
            for (int c = u + 1; c < n; ++c)
                if (s_par[c] == u) s_H[nh++] = c;
            s_nh = nh;
        }
        __syncthreads();
        int nh = s_nh;
        int accepted = -1;
        // ---- step 3: try children ----
        while (nh > 0) {
            const uint4 w = philox4x32_10(make_uint4(rid, ((uint32_t)u << 8) | round, 0u, off), key);
            const int idx = (int)(((unsigned long long)(w.x >> 8) * (unsigned long long)nh) >> 24);
            const float r = (float)(w.y >> 8) * (1.0f / 16777216.0f);
            if (tid == 0) s_sel = s_H[idx];
            __syncthreads();
            const int s = s_sel;
            const int x = s_tok[s];
            const float *qrow = draft_probs + ((size_t)b * Nmax + s) * V;
            const float px = mss_p(S, lrow, bufs + (size_t)S.cur * V, invT, x);
            const float rq = r * qrow[x];
            if (px > 0.f && rq <= px) {
                accepted = s;
                break;
            }
            // reject: residual into the other buffer
            const float *src = bufs + (size_t)S.cur * V;
            float *dst = bufs + (size_t)(S.mode == 0 ? 0 : (S.cur ^ 1)) * V;
            float part = 0.f;
            for (int k = tid; k < V; k += kMssThreads) {
                const float pk = mss_p(S, lrow, src, invT, k);
                const float rr = fmaxf(pk - qrow[k], 0.f);
                dst[k] = rr;
                part += rr;
            }
            const float tot = block_sum<kMssThreads>(part, s_red);  // includes __syncthreads
            if (tot > 0.f) {
                S.cur = (S.mode == 0) ? 0 : (S.cur ^ 1);
                S.mode = 1;
                S.inv = 1.0f / tot;
            }
            if (tid == 0) {
                for (int j = idx; j + 1 < nh; ++j) s_H[j] = s_H[j + 1];
            }
            --nh;
            ++round;
            __syncthreads();
        }
        if (accepted >= 0) {
            ++cnt;
            if (tid == 0) {
                an[cnt] = accepted;
                at[cnt - 1] = s_tok[accepted];
            }
            u = accepted;
            __syncthreads();
            continue;
        }
        // ---- step 4: x_next ~ p by an exponential race: argmax_k p_k / E_k ----
        ArgMax best{-INFINITY, -1};
        const float *src = bufs + (size_t)S.cur * V;
        const uint32_t c1 = ((uint32_t)u << 8) | round;
        for (int k4 = tid * 4; k4 < V; k4 += kMssThreads * 4) {
            const uint4 w = philox4x32_10(make_uint4(rid, c1, (2u << 28) | ((uint32_t)k4 >> 2), off), key);
            const uint32_t ws[4] = {w.x, w.y, w.z, w.w};
#pragma unroll
            for (int i = 0; i < 4; ++i) {
                const int k = k4 + i;
                if (k >= V) break;
                const float pk = mss_p(S, lrow, src, invT, k);
                if (!(pk > 0.f)) continue;
                const float U = ((float)(ws[i] >> 9) + 0.5f) * (1.0f / 8388608.0f);
                const float E = -logf(U);
                best = argmax_merge(best, ArgMax{pk / E, k});
            }
        }
        best = block_argmax<kMssThreads>(best, s_am);
        if (tid == 0) at[cnt] = best.i;
        break;
    }
    if (tid == 0) n_acc[b] = cnt + 1;
}

cudaError_t launch_verify_greedy(const specinfer_shape_t &s, const WsLayout &w, const float *logits,
                                 const int32_t *tree_tokens, const int32_t *parent, const int32_t *n_nodes,
                                 int32_t *acc_nodes, int32_t *acc_tokens, int32_t *n_acc, char *ws,
                                 cudaStream_t stream) {
    dim3 grid(s.max_nodes, s.batch);
    verify_greedy_kernel<<<grid, kGreedyThreads, 0, stream>>>(
        logits, tree_tokens, parent, n_nodes, reinterpret_cast<const int32_t *>(ws + w.req_ok),
        reinterpret_cast<int32_t *>(ws + w.argmax), reinterpret_cast<uint32_t *>(ws + w.verify_cnt), acc_nodes,
        acc_tokens, n_acc, s.max_nodes, s.vocab, s.max_depth + 1);
    return cudaGetLastError();
}

cudaError_t launch_verify_mss(const specinfer_shape_t &s, const WsLayout &w, const float *logits,
                              const int32_t *tree_tokens, const int32_t *parent, const int32_t *n_nodes,
                              const float *draft_probs, float temperature, uint64_t seed, uint64_t offset,
                              const int32_t *request_ids, int32_t *acc_nodes, int32_t *acc_tokens,
                              int32_t *n_acc, char *ws, cudaStream_t stream) {
    verify_mss_kernel<<<s.batch, kMssThreads, 0, stream>>>(
        logits, tree_tokens, parent, n_nodes, draft_probs, reinterpret_cast<const int32_t *>(ws + w.req_ok),
        temperature, (uint32_t)seed, (uint32_t)(seed >> 32), (uint32_t)offset, request_ids,
        reinterpret_cast<float *>(ws + w.mss_p), acc_nodes, acc_tokens, n_acc, s.max_nodes, s.vocab,
        s.max_depth + 1);
    return cudaGetLastError();
}

cudaError_t launch_philox_debug(const uint32_t *ck, uint32_t *out, int n, cudaStream_t stream) {
    if (n <= 0) return cudaSuccess;
    philox_debug_kernel<<<(n + 127) / 128, 128, 0, stream>>>(ck, out, n);
    return cudaGetLastError();
}

}  // namespace specinfer
