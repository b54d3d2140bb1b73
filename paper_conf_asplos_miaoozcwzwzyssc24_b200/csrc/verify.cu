// verify.cu — K4 verify_greedy and K5 verify_mss, sm_100a.
//
// VerifyGreedy (Alg. 2 lines 16-22, L395-401; §4.3): one CTA per (node, request)
// computes O(u) = argmax_x logits[u][x] (128-bit loads, 4 in flight per thread, warp-shuffle
// argmax with the lowest index on ties, reading R7); the last CTA of a request (counter in the
// workspace) walks the tree from the root.  One launch.
//
// VerifyStochastic = MSS (Alg. 2 lines 24-44, L403-425; Fig. 5): also one launch.  Phase 1, one
// CTA per (node, request): the softmax statistics (max, sum of exp) of logits[u]/T for every
// node, in parallel.  Phase 2, the last CTA of the request: the sequential walk of Alg. 2.  An
// accept test then costs O(1) (p[x] from the statistics); only a rejection (residual
// p <- norm(max(0, p - q)), double-buffered so that an all-zero residual keeps p, reading R11)
// and the final exponential-race sample stream a V-wide row.  The RNG contract (Philox4x32-10,
// counters from the global request id, node, round, offset; readings R9, R15) makes the result
// independent of batching and GPU count.
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
// reductions
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

// (max, sum exp((x - max) * invT)) pairs, merged exactly as an online softmax
struct MaxSum {
    float m, z;
};

__device__ __forceinline__ MaxSum maxsum_merge(MaxSum a, MaxSum b, float invT) {
    if (b.m == -INFINITY) return a;
    if (a.m == -INFINITY) return b;
    const float m = fmaxf(a.m, b.m);
    return MaxSum{m, a.z * expf((a.m - m) * invT) + b.z * expf((b.m - m) * invT)};
}

template <int NTHREADS>
__device__ MaxSum block_maxsum(MaxSum a, float invT, MaxSum *sh) {
#pragma unroll
    for (int o = 16; o >= 1; o >>= 1) {
        MaxSum b{__shfl_xor_sync(0xffffffffu, a.m, o), __shfl_xor_sync(0xffffffffu, a.z, o)};
        a = maxsum_merge(a, b, invT);
    }
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    if (lane == 0) sh[wid] = a;
    __syncthreads();
    if (wid == 0) {
        a = (lane < NTHREADS / 32) ? sh[lane] : MaxSum{-INFINITY, 0.f};
#pragma unroll
        for (int o = 16; o >= 1; o >>= 1) {
            MaxSum b{__shfl_xor_sync(0xffffffffu, a.m, o), __shfl_xor_sync(0xffffffffu, a.z, o)};
            a = maxsum_merge(a, b, invT);
        }
        if (lane == 0) sh[0] = a;
    }
    __syncthreads();
    a = sh[0];
    __syncthreads();
    return a;
}

// ------------------------------------------------------------------------------------------
// K4 verify_greedy
// ------------------------------------------------------------------------------------------
constexpr int kGreedyThreads = 512;
constexpr int kUnroll = 8;   // 128-bit loads in flight per thread

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
        int i = threadIdx.x;
        for (; i + (kUnroll - 1) * kGreedyThreads < V4; i += kUnroll * kGreedyThreads) {
            float4 x[kUnroll];
#pragma unroll
            for (int j = 0; j < kUnroll; ++j) x[j] = __ldcs(row4 + i + j * kGreedyThreads);
#pragma unroll
            for (int j = 0; j < kUnroll; ++j) {
                const int base = (i + j * kGreedyThreads) << 2;
                a = argmax_merge(a, ArgMax{x[j].x, base});
                a = argmax_merge(a, ArgMax{x[j].y, base + 1});
                a = argmax_merge(a, ArgMax{x[j].z, base + 2});
                a = argmax_merge(a, ArgMax{x[j].w, base + 3});
            }
        }
        for (; i < V4; i += kGreedyThreads) {
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
// Arithmetic: everything V-wide runs on the MUFU fast path in base 2 (ex2/lg2/rcp .approx,
// relative error ~1e-7); the fp64 oracle differs only at decisions whose margin is below that
// (boundary-excused in the parity tests).  p_k = 2^(l_k c - m c) / z with
// c = log2(e) / T.
constexpr int kMssThreads = 512;
constexpr int kMssUnroll = 4;

__device__ __forceinline__ float lg2f(float x) {
    float y;
    asm("lg2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
    return y;
}
__device__ __forceinline__ float rcpf(float x) {
    float y;
    asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
    return y;
}

// E'_k = -log2 U_k = E_k / ln 2 with U_k = ((w >> 9) + 0.5) 2^-23 (c4 step 4); the race argmax of
// p_k / E_k equals that of p_k / E'_k and of log2 p_k - log2 E'_k.
__device__ __forceinline__ float race_E2(uint32_t w) {
    const float U = ((float)(w >> 9) + 0.5f) * (1.0f / 8388608.0f);
    return -lg2f(U);
}

struct MssState {
    int mode;      // 0: p = 2^(l c - mc) * invZ (softmax of node u); 1: p = buf[cur] * inv
    int cur;       // which residual buffer holds p (mode 1)
    float mc;      // max logit * c (mode 0)
    float invZ;    // 1 / sum_k 2^(l_k c - mc) (mode 0)
    float inv;     // 1 / sum of the residual buffer (mode 1)
};

__device__ __forceinline__ float mss_p(const MssState &s, const float *lrow, const float *buf, float c, int k) {
    return s.mode == 0 ? ex2(fmaf(__ldcg(lrow + k), c, -s.mc)) * s.invZ : __ldcg(buf + k) * s.inv;
}

// Loads kMssUnroll float4 groups of a row (k4 = k4b + j * kMssThreads) with all loads in flight.
__device__ __forceinline__ void load_groups(const float *row, int k4b, int nk4, int V, float (&v)[kMssUnroll][4],
                                            bool streaming) {
#pragma unroll
    for (int j = 0; j < kMssUnroll; ++j) {
        const int k4 = k4b + j * kMssThreads;
        if (k4 >= nk4) continue;
        if ((V & 3) == 0) {
            const float4 x = streaming ? __ldcs(reinterpret_cast<const float4 *>(row) + k4)
                                       : __ldcg(reinterpret_cast<const float4 *>(row) + k4);
            v[j][0] = x.x;
            v[j][1] = x.y;
            v[j][2] = x.z;
            v[j][3] = x.w;
        } else {
#pragma unroll
            for (int i = 0; i < 4; ++i) v[j][i] = (4 * k4 + i < V) ? __ldcg(row + 4 * k4 + i) : -INFINITY;
        }
    }
}

// One V-wide pass of the walk: residual r = max(0, p - q) into dst (returns sum r); when
// `race` is set also the exponential race over r (the sample that follows the last rejection).
__device__ void mss_residual_pass(const MssState &S, const float *lrow, const float *src, const float *qrow,
                                  float *dst, float c, int V, bool race, uint32_t rid, uint32_t c1, uint32_t off,
                                  uint2 key, float *tot_out, ArgMax *best_out, float *s_red, ArgMax *s_am) {
    const int tid = threadIdx.x;
    float part = 0.f;
    ArgMax best{-INFINITY, -1};
    const int nk4 = (V + 3) >> 2;
    for (int k4b = tid; k4b < nk4; k4b += kMssUnroll * kMssThreads) {
        float pv[kMssUnroll][4], qv[kMssUnroll][4];
        load_groups(qrow, k4b, nk4, V, qv, true);
        load_groups(S.mode == 0 ? lrow : src, k4b, nk4, V, pv, false);
#pragma unroll
        for (int j = 0; j < kMssUnroll; ++j) {
            const int k4 = k4b + j * kMssThreads;
            if (k4 >= nk4) continue;
            uint4 w = make_uint4(0, 0, 0, 0);
            if (race) w = philox4x32_10(make_uint4(rid, c1, (2u << 28) | (uint32_t)k4, off), key);
            const uint32_t ws[4] = {w.x, w.y, w.z, w.w};
            float rr[4];
#pragma unroll
            for (int i = 0; i < 4; ++i) {
                const float pk = S.mode == 0 ? ex2(fmaf(pv[j][i], c, -S.mc)) * S.invZ : pv[j][i] * S.inv;
                rr[i] = (4 * k4 + i < V) ? fmaxf(pk - qv[j][i], 0.f) : 0.f;
                part += rr[i];
                if (race && rr[i] > 0.f) best = argmax_merge(best, ArgMax{rr[i] * rcpf(race_E2(ws[i])), 4 * k4 + i});
            }
            if ((V & 3) == 0) {
                __stcg(reinterpret_cast<float4 *>(dst) + k4, make_float4(rr[0], rr[1], rr[2], rr[3]));
            } else {
#pragma unroll
                for (int i = 0; i < 4; ++i)
                    if (4 * k4 + i < V) __stcg(dst + 4 * k4 + i, rr[i]);
            }
        }
    }
    *tot_out = block_sum<kMssThreads>(part, s_red);
    if (race) *best_out = block_argmax<kMssThreads>(best, s_am);
}

// The race over the current p (fallback for an all-zero residual, reading R11).
__device__ ArgMax mss_race_pass(const MssState &S, const float *lrow, const float *src, float c, int V,
                                uint32_t rid, uint32_t c1, uint32_t off, uint2 key, ArgMax *s_am) {
    ArgMax best{-INFINITY, -1};
    for (int k4 = threadIdx.x; 4 * k4 < V; k4 += kMssThreads) {
        const uint4 w = philox4x32_10(make_uint4(rid, c1, (2u << 28) | (uint32_t)k4, off), key);
        const uint32_t ws[4] = {w.x, w.y, w.z, w.w};
#pragma unroll
        for (int i = 0; i < 4; ++i) {
            const int k = 4 * k4 + i;
            if (k >= V) continue;
            const float pk = mss_p(S, lrow, src, c, k);
            if (pk > 0.f) best = argmax_merge(best, ArgMax{pk * rcpf(race_E2(ws[i])), k});
        }
    }
    return block_argmax<kMssThreads>(best, s_am);
}

__global__ void __launch_bounds__(kMssThreads, 2) verify_mss_kernel(
    const float *__restrict__ logits, const int32_t *__restrict__ tree_tokens,
    const int32_t *__restrict__ parent, const int32_t *__restrict__ n_nodes,
    const float *__restrict__ draft_probs, const int32_t *__restrict__ req_ok, float temperature,
    uint32_t seed_lo, uint32_t seed_hi, uint32_t off, const int32_t *__restrict__ request_ids,
    float2 *__restrict__ stats, int32_t *__restrict__ leaf_sample, uint32_t *__restrict__ counter,
    float *__restrict__ pbuf_all, int32_t *__restrict__ acc_nodes, int32_t *__restrict__ acc_tokens,
    int32_t *__restrict__ n_acc, int Nmax, int V, int path_len, unsigned long long *__restrict__ trace) {
    const int u0 = blockIdx.x, b = blockIdx.y;
    const int tid = threadIdx.x;
    const int n = n_nodes[b];
    const float c = 1.4426950408889634f / temperature;
    int tev = 0;
    auto TR = [&](int ev) {
        if (trace != nullptr && tid == 0 && b < 16 && ev < 64) {
            unsigned long long t;
            asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
            trace[b * 64 + ev] = t;
        }
    };
    if (u0 == 0) TR(0);
    __shared__ float s_red[32];
    __shared__ ArgMax s_am[32];
    __shared__ int32_t s_par[kMaxNodes], s_tok[kMaxNodes], s_H[kMaxNodes];
    __shared__ int s_last, s_nh;
    if (!req_ok[b]) {
        if (u0 == 0) {
            for (int j = tid; j < path_len; j += kMssThreads) {
                acc_nodes[(size_t)b * path_len + j] = -1;
                acc_tokens[(size_t)b * path_len + j] = -1;
            }
            if (tid == 0) n_acc[b] = 0;
        }
        return;
    }
    if (u0 >= n) return;
    const uint32_t rid = request_ids ? (uint32_t)request_ids[b] : (uint32_t)b;
    const uint2 key = make_uint2(seed_lo, seed_hi);
    const int nk4 = (V + 3) >> 2;
    // ---------------- phase 1 (one CTA per node): softmax statistics of node u0, and for a
    // leaf its final sample (c4 step 4 at round 0 on p = softmax(logits[u0]/T)) ----------------
    {
        bool has_child = false;
        for (int ch = u0 + 1 + tid; ch < n; ch += kMssThreads) has_child |= (parent[(size_t)b * Nmax + ch] == u0);
        const bool leaf = !__syncthreads_or(has_child);
        const float *lrow = logits + ((size_t)b * Nmax + u0) * V;
        // pass A: row max (and, for a leaf, the race in log2 domain: l c - log2 E')
        float mx = -INFINITY;
        ArgMax best{-INFINITY, -1};
        const uint32_t c1 = (uint32_t)u0 << 8;  // round 0
        for (int k4b = tid; k4b < nk4; k4b += kMssUnroll * kMssThreads) {
            float xv[kMssUnroll][4];
            load_groups(lrow, k4b, nk4, V, xv, false);
#pragma unroll
            for (int j = 0; j < kMssUnroll; ++j) {
                const int k4 = k4b + j * kMssThreads;
                if (k4 >= nk4) continue;
#pragma unroll
                for (int i = 0; i < 4; ++i) mx = fmaxf(mx, xv[j][i]);
                if (leaf) {
                    const uint4 w = philox4x32_10(make_uint4(rid, c1, (2u << 28) | (uint32_t)k4, off), key);
                    const uint32_t ws[4] = {w.x, w.y, w.z, w.w};
#pragma unroll
                    for (int i = 0; i < 4; ++i)
                        if (4 * k4 + i < V) best = argmax_merge(best, ArgMax{xv[j][i] * c - lg2f(race_E2(ws[i])), 4 * k4 + i});
                }
            }
        }
        // block max
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
        const float mc = s_red[0] * c;
        __syncthreads();
        if (leaf) best = block_argmax<kMssThreads>(best, s_am);
        // pass B: z = sum 2^(l c - m c)  (the row is L2-resident after pass A)
        float z = 0.f;
        for (int k4b = tid; k4b < nk4; k4b += kMssUnroll * kMssThreads) {
            float xv[kMssUnroll][4];
            load_groups(lrow, k4b, nk4, V, xv, false);
#pragma unroll
            for (int j = 0; j < kMssUnroll; ++j)
#pragma unroll
                for (int i = 0; i < 4; ++i) z += (k4b + j * kMssThreads < nk4) ? ex2(fmaf(xv[j][i], c, -mc)) : 0.f;
        }
        z = block_sum<kMssThreads>(z, s_red);
        if (tid == 0) {
            stats[(size_t)b * Nmax + u0] = make_float2(mc, z);
            leaf_sample[(size_t)b * Nmax + u0] = leaf ? best.i : -1;
            __threadfence();
            const unsigned old = atomicAdd(&counter[b], 1u);
            s_last = (old == (unsigned)(n - 1));
        }
        __syncthreads();
        if (!s_last) return;
        __threadfence();
    }
    TR(1);
    tev = 2;
    // ---------------- phase 2 (last CTA of the request): the walk of Alg. 2 ----------------
    int32_t *an = acc_nodes + (size_t)b * path_len;
    int32_t *at = acc_tokens + (size_t)b * path_len;
    for (int j = tid; j < path_len; j += kMssThreads) {
        an[j] = -1;
        at[j] = -1;
    }
    for (int i = tid; i < n; i += kMssThreads) {
        s_par[i] = parent[(size_t)b * Nmax + i];
        s_tok[i] = tree_tokens[(size_t)b * Nmax + i];
    }
    float *bufs = pbuf_all + (size_t)b * 2 * V;
    __syncthreads();
    if (tid == 0) {
        an[0] = 0;
        counter[b] = 0u;  // reusable by the next call on this workspace
    }
    int u = 0, cnt = 0;
    for (;;) {
        const float *lrow = logits + ((size_t)b * Nmax + u) * V;
        // step 1: p = softmax(logits[u] / T), implicit through the phase-1 statistics
        const float2 su = __ldcg(stats + (size_t)b * Nmax + u);
        MssState S{0, 0, su.x, 1.0f / su.y, 0.f};
        uint32_t round = 0;
        // step 2: children of u in ascending order
        if (tid == 0) {
            int nh = 0;
            for (int ch = u + 1; ch < n; ++ch)
                if (s_par[ch] == u) s_H[nh++] = ch;
            s_nh = nh;
        }
        __syncthreads();
        int nh = s_nh;
        if (nh == 0) {
            // a leaf: its round-0 sample was drawn in phase 1
            if (tid == 0) at[cnt] = __ldcg(leaf_sample + (size_t)b * Nmax + u);
            break;
        }
        int accepted = -1;
        int final_tok = -1;
        // step 3: try children in Philox-uniform order
        while (nh > 0) {
            const uint4 w = philox4x32_10(make_uint4(rid, ((uint32_t)u << 8) | round, 0u, off), key);
            const int idx = (int)(((unsigned long long)(w.x >> 8) * (unsigned long long)nh) >> 24);
            const float r = (float)(w.y >> 8) * (1.0f / 16777216.0f);
            const int s = s_H[idx];
            const int x = s_tok[s];
            const float *qrow = draft_probs + ((size_t)b * Nmax + s) * V;
            const float px = mss_p(S, lrow, bufs + (size_t)S.cur * V, c, x);
            const float rq = r * __ldg(qrow + x);
            if (px > 0.f && rq <= px) {
                accepted = s;
                break;
            }
            // reject: residual max(0, p - q) into the other buffer (and, after the last child,
            // the exponential race over it with the next round's counters)
            const bool last = (nh == 1);
            const int dsti = (S.mode == 0) ? 0 : (S.cur ^ 1);
            float tot;
            ArgMax best;
            mss_residual_pass(S, lrow, bufs + (size_t)S.cur * V, qrow, bufs + (size_t)dsti * V, c, V, last, rid,
                              ((uint32_t)u << 8) | (round + 1), off, key, &tot, &best, s_red, s_am);
            if (tot > 0.f) {
                S.cur = dsti;
                S.mode = 1;
                S.inv = 1.0f / tot;
                if (last) final_tok = best.i;
            } else if (last) {
                // R11: the residual is all zero, p is kept; sample from it
                final_tok = mss_race_pass(S, lrow, bufs + (size_t)S.cur * V, c, V, rid,
                                          ((uint32_t)u << 8) | (round + 1), off, key, s_am).i;
            }
            if (tid == 0) {
                for (int j = idx; j + 1 < nh; ++j) s_H[j] = s_H[j + 1];
            }
            --nh;
            ++round;
            __syncthreads();
            TR(tev++);
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
        // step 4: every child was rejected; x_next was drawn during the last residual pass
        if (tid == 0) at[cnt] = final_tok;
        break;
    }
    if (tid == 0) n_acc[b] = cnt + 1;
    TR(63);
}

unsigned long long *g_mss_trace = nullptr;  // debug only (specinfer_debug_set_trace with SPECINFER_TRACE_MSS)

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
    dim3 grid(s.max_nodes, s.batch);
    verify_mss_kernel<<<grid, kMssThreads, 0, stream>>>(
        logits, tree_tokens, parent, n_nodes, draft_probs, reinterpret_cast<const int32_t *>(ws + w.req_ok),
        temperature, (uint32_t)seed, (uint32_t)(seed >> 32), (uint32_t)offset, request_ids,
        reinterpret_cast<float2 *>(ws + w.mss_stats), reinterpret_cast<int32_t *>(ws + w.mss_leaf),
        reinterpret_cast<uint32_t *>(ws + w.verify_cnt) + s.batch,
        reinterpret_cast<float *>(ws + w.mss_p), acc_nodes, acc_tokens, n_acc, s.max_nodes, s.vocab,
        s.max_depth + 1, g_mss_trace);
    return cudaGetLastError();
}

cudaError_t launch_philox_debug(const uint32_t *ck, uint32_t *out, int n, cudaStream_t stream) {
    if (n <= 0) return cudaSuccess;
    philox_debug_kernel<<<(n + 127) / 128, 128, 0, stream>>>(ck, out, n);
    return cudaGetLastError();
}

}  // namespace specinfer
