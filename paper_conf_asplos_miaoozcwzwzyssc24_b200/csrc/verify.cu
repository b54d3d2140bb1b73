// verify.cu — K4 verify_greedy and K5 verify_mss, sm_100a.
//
// VerifyGreedy (Alg. 2 lines 16-22, L395-401; §4.3): one CTA per (node, request)
// computes O(u) = argmax_x logits[u][x] (128-bit loads, 8 in flight per thread, warp-shuffle
// argmax with the lowest index on ties, reading R7); the last CTA of a request (counter in the
// workspace) stages parents, tokens and O(u) in shared memory and walks the tree from the root
// there.  One launch.
//
// Naive sampling (NEXT-3, L747-753, the baseline of Theorem 4.3) reuses the K4 kernel: the
// per-node key is the exponential-race key of x ~ softmax(l / T) instead of the logit, and the
// walk follows the child whose token equals that sample.
//
// VerifyStochastic = MSS (Alg. 2 lines 24-44, L403-425; Fig. 5): also one launch, one 8-CTA
// thread-block cluster per request walking Alg. 2 sequentially.  At every visited node the
// cluster computes the softmax statistics of logits[u]/T (a V-wide pass split over the 8 CTAs and
// reduced through distributed shared memory); an accept test is then O(1); a rejection streams one
// V-wide residual pass p <- norm(max(0, p - q)) (double-buffered so that an all-zero residual
// keeps p, reading R11) split the same way, and the exponential race of the final sample is fused
// into the last pass.  The RNG contract (Philox4x32-10, counters from the global request id, node,
// round, offset; readings R9, R15) makes the result independent of batching and GPU count.
// NEXT-4a: with a gather descriptor, the finishing warp of every request also stores its packed
// row into every rank's receive table (gather.cuh).
#include "common.cuh"
#include "gather.cuh"

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

__device__ __forceinline__ float lg2f(float x) {
    float y;
    asm("lg2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
    return y;
}
// E'_k = -log2 U_k = E_k / ln 2 with U_k = ((w >> 9) + 0.5) 2^-23 (c4 step 4); the race argmax of
// p_k / E_k equals that of p_k / E'_k and of log2 p_k - log2 E'_k.
__device__ __forceinline__ float race_E2(uint32_t w) {
    const float U = ((float)(w >> 9) + 0.5f) * (1.0f / 8388608.0f);
    return -lg2f(U);
}

// Per-node key of the "argmax then walk" verifiers.  Greedy (K4): the logit itself.  Naive
// sampling (NEXT-3, L747-753): the exponential-race key of x ~ softmax(l / T) at round 0 with the
// counters of c4 step 4 (rid, u<<8, (2<<28) | (k>>2), offset), in the log2 domain:
// l_k c - log2 E'_k with c = log2(e) / T (same draw as MSS's leaf sample).
struct NsParams {
    float c;
    uint32_t seed_lo, seed_hi, off;
    const int32_t *request_ids;
};

template <bool kNS>
__device__ __forceinline__ void key4(ArgMax &a, float4 x, int k4, uint32_t rid, uint32_t u, const NsParams &ns) {
    const int base = k4 << 2;
    if (kNS) {
        const uint4 w = philox4x32_10(make_uint4(rid, u << 8, (2u << 28) | (uint32_t)k4, ns.off),
                                      make_uint2(ns.seed_lo, ns.seed_hi));
        a = argmax_merge(a, ArgMax{x.x * ns.c - lg2f(race_E2(w.x)), base});
        a = argmax_merge(a, ArgMax{x.y * ns.c - lg2f(race_E2(w.y)), base + 1});
        a = argmax_merge(a, ArgMax{x.z * ns.c - lg2f(race_E2(w.z)), base + 2});
        a = argmax_merge(a, ArgMax{x.w * ns.c - lg2f(race_E2(w.w)), base + 3});
    } else {
        a = argmax_merge(a, ArgMax{x.x, base});
        a = argmax_merge(a, ArgMax{x.y, base + 1});
        a = argmax_merge(a, ArgMax{x.z, base + 2});
        a = argmax_merge(a, ArgMax{x.w, base + 3});
    }
}

template <bool kNS>
__global__ void __launch_bounds__(kGreedyThreads) verify_greedy_kernel(
    const float *__restrict__ logits, const int32_t *__restrict__ tree_tokens,
    const int32_t *__restrict__ parent, const int32_t *__restrict__ n_nodes,
    const int32_t *__restrict__ req_ok, int32_t *__restrict__ argmax_ws,
    uint32_t *__restrict__ counter, int32_t *__restrict__ acc_nodes, int32_t *__restrict__ acc_tokens,
    int32_t *__restrict__ n_acc, int Nmax, int V, int path_len, NsParams ns, GatherDev g) {
    const int u = blockIdx.x, b = blockIdx.y;
    const int n = n_nodes[b];
    __shared__ ArgMax sh[32];
    __shared__ int s_last;
    __shared__ int32_t s_par[kMaxNodes], s_tok[kMaxNodes], s_o[kMaxNodes];
    if (!req_ok[b]) {
        if (u == 0) {
            for (int j = threadIdx.x; j < path_len; j += blockDim.x) {
                acc_nodes[(size_t)b * path_len + j] = -1;
                acc_tokens[(size_t)b * path_len + j] = -1;
            }
            if (threadIdx.x == 0) n_acc[b] = 0;
            __syncthreads();
            if (threadIdx.x < 32)   // an invalid request still publishes its (empty) row
                gather_publish(g, b, 0, acc_nodes + (size_t)b * path_len, acc_tokens + (size_t)b * path_len, path_len);
        }
        return;
    }
    if (u >= n) return;
    const uint32_t rid = kNS ? (ns.request_ids ? (uint32_t)ns.request_ids[b] : (uint32_t)b) : 0u;
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
            for (int j = 0; j < kUnroll; ++j) key4<kNS>(a, x[j], i + j * kGreedyThreads, rid, u, ns);
        }
        for (; i < V4; i += kGreedyThreads) key4<kNS>(a, __ldcs(row4 + i), i, rid, u, ns);
    } else {
        for (int i = threadIdx.x; i < V; i += kGreedyThreads) {
            float key = __ldcs(row + i);
            if (kNS) {
                const uint4 w = philox4x32_10(make_uint4(rid, (uint32_t)u << 8, (2u << 28) | (uint32_t)(i >> 2), ns.off),
                                              make_uint2(ns.seed_lo, ns.seed_hi));
                const uint32_t ws[4] = {w.x, w.y, w.z, w.w};
                key = key * ns.c - lg2f(race_E2(ws[i & 3]));
            }
            a = argmax_merge(a, ArgMax{key, i});
        }
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
    // parents, tokens and every node's O(u) are staged in shared memory with one round of
    // parallel loads (one L2 round trip), so the walk itself is dependent shared-memory reads only
    if (threadIdx.x >= 32) return;
    __threadfence();
    const int lane = threadIdx.x;
    const int32_t *par = parent + (size_t)b * Nmax;
    const int32_t *tok = tree_tokens + (size_t)b * Nmax;
    for (int j = lane; j < n; j += 32) {
        s_par[j] = par[j];
        s_tok[j] = tok[j];
        s_o[j] = __ldcg(argmax_ws + (size_t)b * Nmax + j);
    }
    __syncwarp();
    int32_t *an = acc_nodes + (size_t)b * path_len;
    int32_t *at = acc_tokens + (size_t)b * path_len;
    int cur = 0, cnt = 0;
    if (lane == 0) an[0] = 0;
    for (;;) {
        const int o = s_o[cur];
        int next = -1;
        for (int base = cur + 1; base < n && next < 0; base += 32) {
            const int cidx = base + lane;
            const bool hit = cidx < n && s_par[cidx] == cur && s_tok[cidx] == o;
            const unsigned m = __ballot_sync(0xffffffffu, hit);
            if (m) next = base + __ffs(m) - 1;
        }
        if (next < 0) {
            if (lane == 0) at[cnt] = o;
            break;
        }
        if (lane == 0) {
            at[cnt] = s_tok[next];
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
    __syncwarp();
    gather_publish(g, b, cnt + 1, an, at, path_len);   // NEXT-4a (no-op without a gather)
}

// ------------------------------------------------------------------------------------------
// K5 verify_mss: one thread-block cluster per request walks Alg. 2; every V-wide pass (softmax
// statistics, residual, exponential race) is split over the cluster's CTAs and reduced through
// distributed shared memory, so a pass costs ~1/CS of a single SM's time.
// Arithmetic: V-wide work runs on the MUFU fast path in base 2 (ex2/lg2/rcp .approx, relative
// error ~1e-7); the fp64 oracle differs only at decisions whose margin is below that
// (boundary-excused in the parity tests).  p_k = 2^(l_k c - m c) / z, c = log2(e)/T.
// ------------------------------------------------------------------------------------------
constexpr int kMssThreads = 256;
constexpr int kMssUnroll = 4;
constexpr int kMssCluster = 8;

__device__ __forceinline__ float rcpf(float x) {
    float y;
    asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
    return y;
}
__device__ __forceinline__ uint32_t cluster_ctarank() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
}
__device__ __forceinline__ uint32_t cluster_nctarank() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_nctarank;" : "=r"(r));
    return r;
}
__device__ __forceinline__ void cluster_sync_all() {
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
__device__ __forceinline__ uint32_t map_to_rank(const void *p, uint32_t rank) {
    uint32_t r;
    asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(smem_u32(p)), "r"(rank));
    return r;
}
__device__ __forceinline__ float ld_dsmem_f32(uint32_t a) {
    float v;
    asm volatile("ld.shared::cluster.f32 %0, [%1];" : "=f"(v) : "r"(a) : "memory");
    return v;
}
__device__ __forceinline__ int ld_dsmem_s32(uint32_t a) {
    int v;
    asm volatile("ld.shared::cluster.s32 %0, [%1];" : "=r"(v) : "r"(a) : "memory");
    return v;
}

// Per-CTA partial results exchanged through DSMEM (double-buffered by reduction parity).
struct MssPart {
    float a, b;  // (max, sum) pair or (sum, -)
    float v;     // race key
    int i;       // race index
};

struct MssCluster {
    MssPart *slot;    // smem [2], this CTA's contribution per reduction parity
    MssPart *result;  // smem [1], the merged value broadcast to the CTA
    uint32_t rank, size;
    int parity;
    // every CTA contributes `mine` (already reduced over the block); returns the merged result
    // identically on every CTA.  Warp 0 gathers the cluster's slots through DSMEM.
    template <class Merge>
    __device__ MssPart reduce(const MssPart &mine, Merge merge) {
        if (threadIdx.x == 0) slot[parity] = mine;
        cluster_sync_all();
        if (threadIdx.x < 32) {
            const int lane = threadIdx.x;
            MssPart o = mine;
            bool have = false;
            if (lane < (int)size) {
                const uint32_t base = map_to_rank(&slot[parity], lane);
                o.a = ld_dsmem_f32(base);
                o.b = ld_dsmem_f32(base + 4);
                o.v = ld_dsmem_f32(base + 8);
                o.i = ld_dsmem_s32(base + 12);
                have = true;
            }
#pragma unroll
            for (int off = 16; off >= 1; off >>= 1) {
                MssPart t;
                t.a = __shfl_xor_sync(0xffffffffu, o.a, off);
                t.b = __shfl_xor_sync(0xffffffffu, o.b, off);
                t.v = __shfl_xor_sync(0xffffffffu, o.v, off);
                t.i = __shfl_xor_sync(0xffffffffu, o.i, off);
                const bool th = __shfl_xor_sync(0xffffffffu, have, off);
                if (th) o = have ? merge(o, t) : t;
                have = have || th;
            }
            if (lane == 0) *result = o;
        }
        __syncthreads();
        const MssPart r = *result;
        __syncthreads();
        parity ^= 1;
        return r;
    }
};

__device__ __forceinline__ MssPart merge_maxsum(MssPart x, MssPart y) {
    // (max, sum 2^(l c - max c)) in the log2 domain: a = max*c, b = sum
    if (y.a == -INFINITY) return x;
    if (x.a == -INFINITY) return y;
    const float m = fmaxf(x.a, y.a);
    MssPart r = x;
    r.a = m;
    r.b = x.b * ex2(x.a - m) + y.b * ex2(y.a - m);
    return r;
}
__device__ __forceinline__ MssPart merge_sum_race(MssPart x, MssPart y) {
    MssPart r;
    r.a = x.a + y.a;
    r.b = 0.f;
    const ArgMax m = argmax_merge(ArgMax{x.v, x.i}, ArgMax{y.v, y.i});
    r.v = m.v;
    r.i = m.i;
    return r;
}

// Loads kMssUnroll float4 groups of a row slice (k4 = k4b + j * kMssThreads < k4end).
__device__ __forceinline__ void load_groups(const float *row, int k4b, int k4end, int V, float (&v)[kMssUnroll][4],
                                            bool streaming) {
#pragma unroll
    for (int j = 0; j < kMssUnroll; ++j) {
        const int k4 = k4b + j * kMssThreads;
        if (k4 >= k4end) continue;
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

__global__ void __launch_bounds__(kMssThreads) verify_mss_kernel(
    const float *__restrict__ logits, const int32_t *__restrict__ tree_tokens,
    const int32_t *__restrict__ parent, const int32_t *__restrict__ n_nodes,
    const float *__restrict__ draft_probs, const int32_t *__restrict__ req_ok, float temperature,
    uint32_t seed_lo, uint32_t seed_hi, uint32_t off, const int32_t *__restrict__ request_ids,
    float *__restrict__ pbuf_all, int32_t *__restrict__ acc_nodes, int32_t *__restrict__ acc_tokens,
    int32_t *__restrict__ n_acc, int Nmax, int V, int path_len, unsigned long long *__restrict__ trace,
    GatherDev g) {
    const int b = blockIdx.y;
    const int tid = threadIdx.x;
    __shared__ MssPart s_slot[2], s_result;
    __shared__ float s_red[32];
    __shared__ ArgMax s_am[32];
    __shared__ int32_t s_par[kMaxNodes], s_tok[kMaxNodes], s_H[kMaxNodes];
    __shared__ int s_nh;
    MssCluster cl{s_slot, &s_result, cluster_ctarank(), cluster_nctarank(), 0};
    const bool leader = (cl.rank == 0);
    int tev = 0;
    auto TR = [&](int ev) {
        if (trace != nullptr && tid == 0 && leader && b < 16 && ev < 64) {
            unsigned long long t;
            asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
            trace[b * 64 + ev] = t;
        }
    };
    TR(tev++);
    int32_t *an = acc_nodes + (size_t)b * path_len;
    int32_t *at = acc_tokens + (size_t)b * path_len;
    if (leader)
        for (int j = tid; j < path_len; j += kMssThreads) {
            an[j] = -1;
            at[j] = -1;
        }
    if (!req_ok[b]) {  // uniform over the cluster
        if (leader) {
            if (tid == 0) n_acc[b] = 0;
            __syncthreads();
            if (tid < 32) gather_publish(g, b, 0, an, at, path_len);   // its (empty) row
        }
        return;
    }
    const int n = n_nodes[b];
    for (int i = tid; i < n; i += kMssThreads) {
        s_par[i] = parent[(size_t)b * Nmax + i];
        s_tok[i] = tree_tokens[(size_t)b * Nmax + i];
    }
    const float c = 1.4426950408889634f / temperature;
    const uint32_t rid = request_ids ? (uint32_t)request_ids[b] : (uint32_t)b;
    const uint2 key = make_uint2(seed_lo, seed_hi);
    // this CTA's slice of the vocabulary, in float4 groups
    const int nk4 = (V + 3) >> 2;
    const int k4lo = (int)((long long)nk4 * cl.rank / cl.size);
    const int k4hi = (int)((long long)nk4 * (cl.rank + 1) / cl.size);
    float *bufs = pbuf_all + (size_t)b * 2 * V;
    __syncthreads();
    if (leader && tid == 0) an[0] = 0;

    int u = 0, cnt = 0;
    for (;;) {
        const float *lrow = logits + ((size_t)b * Nmax + u) * V;
        // children of u in ascending order (step 2)
        if (tid == 0) {
            int nh = 0;
            for (int ch = u + 1; ch < n; ++ch)
                if (s_par[ch] == u) s_H[nh++] = ch;
            s_nh = nh;
        }
        __syncthreads();
        int nh = s_nh;
        if (nh == 0) {
            // a leaf: x_next ~ softmax(logits[u]/T) at round 0 (steps 1 and 4); race in log2 domain
            ArgMax best{-INFINITY, -1};
            const uint32_t c1 = (uint32_t)u << 8;
            for (int k4b = k4lo + tid; k4b < k4hi; k4b += kMssUnroll * kMssThreads) {
                float xv[kMssUnroll][4];
                load_groups(lrow, k4b, k4hi, V, xv, true);
#pragma unroll
                for (int j = 0; j < kMssUnroll; ++j) {
                    const int k4 = k4b + j * kMssThreads;
                    if (k4 >= k4hi) continue;
                    const uint4 w = philox4x32_10(make_uint4(rid, c1, (2u << 28) | (uint32_t)k4, off), key);
                    const uint32_t ws[4] = {w.x, w.y, w.z, w.w};
#pragma unroll
                    for (int i = 0; i < 4; ++i)
                        if (4 * k4 + i < V) best = argmax_merge(best, ArgMax{xv[j][i] * c - lg2f(race_E2(ws[i])), 4 * k4 + i});
                }
            }
            best = block_argmax<kMssThreads>(best, s_am);
            const MssPart r = cl.reduce(MssPart{0.f, 0.f, best.v, best.i}, merge_sum_race);
            if (leader && tid == 0) at[cnt] = r.i;
            break;
        }
        // step 1: softmax statistics of logits[u] / T (one pass, online max/sum)
        float mc = -INFINITY, z = 0.f;
        for (int k4b = k4lo + tid; k4b < k4hi; k4b += kMssUnroll * kMssThreads) {
            float xv[kMssUnroll][4];
            load_groups(lrow, k4b, k4hi, V, xv, false);
#pragma unroll
            for (int j = 0; j < kMssUnroll; ++j) {
                if (k4b + j * kMssThreads >= k4hi) continue;
                float lm = -INFINITY;
#pragma unroll
                for (int i = 0; i < 4; ++i) lm = fmaxf(lm, xv[j][i] * c);
                if (lm > mc) {
                    z = (mc == -INFINITY) ? 0.f : z * ex2(mc - lm);
                    mc = lm;
                }
#pragma unroll
                for (int i = 0; i < 4; ++i) z += ex2(fmaf(xv[j][i], c, -mc));
            }
        }
        {
            // block merge of (mc, z)
#pragma unroll
            for (int o = 16; o >= 1; o >>= 1) {
                const float om = __shfl_xor_sync(0xffffffffu, mc, o), oz = __shfl_xor_sync(0xffffffffu, z, o);
                const MssPart m = merge_maxsum(MssPart{mc, z, 0.f, 0}, MssPart{om, oz, 0.f, 0});
                mc = m.a;
                z = m.b;
            }
            __shared__ float s_m[32], s_z[32];
            if ((tid & 31) == 0) {
                s_m[tid >> 5] = mc;
                s_z[tid >> 5] = z;
            }
            __syncthreads();
            MssPart acc{-INFINITY, 0.f, 0.f, 0};
            for (int w = 0; w < kMssThreads / 32; ++w) acc = merge_maxsum(acc, MssPart{s_m[w], s_z[w], 0.f, 0});
            __syncthreads();
            const MssPart r = cl.reduce(acc, merge_maxsum);
            mc = r.a;
            z = r.b;
        }
        int mode = 0, cur = 0;    // p = 2^(l c - mc)/z (mode 0) or buf[cur] * inv (mode 1)
        const float invZ = 1.0f / z;
        float inv = 0.f;
        uint32_t round = 0;
        int accepted = -1, final_tok = -1;
        // step 3: try children in Philox-uniform order
        while (nh > 0) {
            const uint4 w = philox4x32_10(make_uint4(rid, ((uint32_t)u << 8) | round, 0u, off), key);
            const int idx = (int)(((unsigned long long)(w.x >> 8) * (unsigned long long)nh) >> 24);
            const float r = (float)(w.y >> 8) * (1.0f / 16777216.0f);
            const int s = s_H[idx];
            const int x = s_tok[s];
            const float *qrow = draft_probs + ((size_t)b * Nmax + s) * V;
            const float px = mode == 0 ? ex2(fmaf(__ldcg(lrow + x), c, -mc)) * invZ
                                       : __ldcg(bufs + (size_t)cur * V + x) * inv;
            const float rq = r * __ldg(qrow + x);
            if (px > 0.f && rq <= px) {
                accepted = s;
                break;
            }
            // reject: residual max(0, p - q) of this CTA's slice into the other buffer, and after
            // the last child the exponential race over it (next round's counters)
            const bool last = (nh == 1);
            const int dsti = (mode == 0) ? 0 : (cur ^ 1);
            const float *src = mode == 0 ? lrow : bufs + (size_t)cur * V;
            float *dst = bufs + (size_t)dsti * V;
            const uint32_t c1 = ((uint32_t)u << 8) | (round + 1);
            float part = 0.f;
            ArgMax best{-INFINITY, -1};
            for (int k4b = k4lo + tid; k4b < k4hi; k4b += kMssUnroll * kMssThreads) {
                float pv[kMssUnroll][4], qv[kMssUnroll][4];
                load_groups(qrow, k4b, k4hi, V, qv, true);
                load_groups(src, k4b, k4hi, V, pv, false);
#pragma unroll
                for (int j = 0; j < kMssUnroll; ++j) {
                    const int k4 = k4b + j * kMssThreads;
                    if (k4 >= k4hi) continue;
                    uint4 wr = make_uint4(0, 0, 0, 0);
                    if (last) wr = philox4x32_10(make_uint4(rid, c1, (2u << 28) | (uint32_t)k4, off), key);
                    const uint32_t ws[4] = {wr.x, wr.y, wr.z, wr.w};
                    float rr[4];
#pragma unroll
                    for (int i = 0; i < 4; ++i) {
                        const float pk = mode == 0 ? ex2(fmaf(pv[j][i], c, -mc)) * invZ : pv[j][i] * inv;
                        rr[i] = (4 * k4 + i < V) ? fmaxf(pk - qv[j][i], 0.f) : 0.f;
                        part += rr[i];
                        if (last && rr[i] > 0.f) best = argmax_merge(best, ArgMax{rr[i] * rcpf(race_E2(ws[i])), 4 * k4 + i});
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
            part = block_sum<kMssThreads>(part, s_red);
            if (last) best = block_argmax<kMssThreads>(best, s_am);
            // the reduction's cluster barrier also publishes this CTA's residual slice
            const MssPart red = cl.reduce(MssPart{part, 0.f, best.v, best.i}, merge_sum_race);
            if (red.a > 0.f) {
                mode = 1;
                cur = dsti;
                inv = 1.0f / red.a;
                if (last) final_tok = red.i;
            } else if (last) {
                // R11: the residual is all zero, p is kept; sample from it with the same counters
                ArgMax b2{-INFINITY, -1};
                const float *src2 = mode == 0 ? lrow : bufs + (size_t)cur * V;
                for (int k4 = k4lo + tid; k4 < k4hi; k4 += kMssThreads) {
                    const uint4 w2 = philox4x32_10(make_uint4(rid, c1, (2u << 28) | (uint32_t)k4, off), key);
                    const uint32_t ws[4] = {w2.x, w2.y, w2.z, w2.w};
#pragma unroll
                    for (int i = 0; i < 4; ++i) {
                        const int k = 4 * k4 + i;
                        if (k >= V) continue;
                        const float pk = mode == 0 ? ex2(fmaf(__ldcg(src2 + k), c, -mc)) * invZ : __ldcg(src2 + k) * inv;
                        if (pk > 0.f) b2 = argmax_merge(b2, ArgMax{pk * rcpf(race_E2(ws[i])), k});
                    }
                }
                b2 = block_argmax<kMssThreads>(b2, s_am);
                final_tok = cl.reduce(MssPart{0.f, 0.f, b2.v, b2.i}, merge_sum_race).i;
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
            if (leader && tid == 0) {
                an[cnt] = accepted;
                at[cnt - 1] = s_tok[accepted];
            }
            u = accepted;
            __syncthreads();
            continue;
        }
        // step 4: every child was rejected; x_next was drawn during the last residual pass
        if (leader && tid == 0) at[cnt] = final_tok;
        break;
    }
    if (leader && tid == 0) n_acc[b] = cnt + 1;
    TR(63);
    if (leader) {
        __syncthreads();
        if (tid < 32) gather_publish(g, b, cnt + 1, an, at, path_len);   // NEXT-4a (no-op without a gather)
    }
    cluster_sync_all();  // no CTA leaves while others may still read its DSMEM slots
}

#ifdef SPECINFER_DEBUG_HOOKS
unsigned long long *g_mss_trace = nullptr;  // debug build only (specinfer_debug_set_trace + SPECINFER_TRACE_MSS)
#else
static unsigned long long *const g_mss_trace = nullptr;  // production: no MSS timestamps
#endif

cudaError_t launch_verify_greedy(const specinfer_shape_t &s, const WsLayout &w, const float *logits,
                                 const int32_t *tree_tokens, const int32_t *parent, const int32_t *n_nodes,
                                 int32_t *acc_nodes, int32_t *acc_tokens, int32_t *n_acc, char *ws,
                                 cudaStream_t stream, const GatherDev *gather) {
    dim3 grid(s.max_nodes, s.batch);
    verify_greedy_kernel<false><<<grid, kGreedyThreads, 0, stream>>>(
        logits, tree_tokens, parent, n_nodes, reinterpret_cast<const int32_t *>(ws + w.req_ok),
        reinterpret_cast<int32_t *>(ws + w.argmax), reinterpret_cast<uint32_t *>(ws + w.verify_cnt), acc_nodes,
        acc_tokens, n_acc, s.max_nodes, s.vocab, s.max_depth + 1, NsParams{}, gather ? *gather : GatherDev{});
    return cudaGetLastError();
}

cudaError_t launch_verify_ns(const specinfer_shape_t &s, const WsLayout &w, const float *logits,
                             const int32_t *tree_tokens, const int32_t *parent, const int32_t *n_nodes,
                             float temperature, uint64_t seed, uint64_t offset, const int32_t *request_ids,
                             int32_t *acc_nodes, int32_t *acc_tokens, int32_t *n_acc, char *ws, cudaStream_t stream) {
    dim3 grid(s.max_nodes, s.batch);
    const NsParams ns{1.4426950408889634f / temperature, (uint32_t)seed, (uint32_t)(seed >> 32), (uint32_t)offset,
                      request_ids};
    verify_greedy_kernel<true><<<grid, kGreedyThreads, 0, stream>>>(
        logits, tree_tokens, parent, n_nodes, reinterpret_cast<const int32_t *>(ws + w.req_ok),
        reinterpret_cast<int32_t *>(ws + w.argmax), reinterpret_cast<uint32_t *>(ws + w.verify_cnt), acc_nodes,
        acc_tokens, n_acc, s.max_nodes, s.vocab, s.max_depth + 1, ns, GatherDev{});
    return cudaGetLastError();
}

cudaError_t launch_verify_mss(const specinfer_shape_t &s, const WsLayout &w, const float *logits,
                              const int32_t *tree_tokens, const int32_t *parent, const int32_t *n_nodes,
                              const float *draft_probs, float temperature, uint64_t seed, uint64_t offset,
                              const int32_t *request_ids, int32_t *acc_nodes, int32_t *acc_tokens,
                              int32_t *n_acc, char *ws, cudaStream_t stream, const GatherDev *gather) {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(kMssCluster, s.batch);
    cfg.blockDim = dim3(kMssThreads);
    cfg.dynamicSmemBytes = 0;
    cfg.stream = stream;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = kMssCluster;
    attr[0].val.clusterDim.y = 1;
    attr[0].val.clusterDim.z = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, verify_mss_kernel, logits, tree_tokens, parent, n_nodes, draft_probs,
                              reinterpret_cast<const int32_t *>(ws + w.req_ok), temperature, (uint32_t)seed,
                              (uint32_t)(seed >> 32), (uint32_t)offset, request_ids,
                              reinterpret_cast<float *>(ws + w.mss_p), acc_nodes, acc_tokens, n_acc, s.max_nodes,
                              s.vocab, s.max_depth + 1, g_mss_trace, gather ? *gather : GatherDev{});
}

// NEXT-4a: waits until every rank published this epoch's rows here, copies the table to table_out
// (a fixed address for the consumers: the buffer alternates by epoch parity) and advances the epoch
__global__ void __launch_bounds__(256) gather_wait_kernel(GatherDev g, int32_t *__restrict__ table_out) {
    const uint32_t e = ld_volatile_u32(g.state) + 1u;
    if ((int)threadIdx.x < g.world) {
        const uint32_t *f = g.flags[g.rank] + threadIdx.x;
        if (ld_acquire_sys(f) < e) {
            const long long t0 = clock64();
            while (ld_acquire_sys(f) < e) {
                if (clock64() - t0 > SPECINFER_WATCHDOG_CYCLES) {
                    printf("specinfer: gather_wait timeout rank %d waiting for rank %d epoch %u\n", g.rank,
                           (int)threadIdx.x, e);
                    __trap();
                }
            }
        }
    }
    __syncthreads();
    __threadfence_system();
    const size_t n = (size_t)g.world * g.rows_per_rank * g.row_len;
    const int32_t *src = g.recv[g.rank] + (size_t)((e - 1u) & 1u) * n;
    if (table_out != nullptr)
        for (size_t i = threadIdx.x; i < n; i += blockDim.x) table_out[i] = __ldcv(src + i);
    __syncthreads();
    if (threadIdx.x == 0) g.state[0] = e;
}

cudaError_t launch_gather_wait(const GatherDev &g, int32_t *table_out, cudaStream_t stream) {
    gather_wait_kernel<<<1, 256, 0, stream>>>(g, table_out);
    return cudaGetLastError();
}

cudaError_t launch_philox_debug(const uint32_t *ck, uint32_t *out, int n, cudaStream_t stream) {
    if (n <= 0) return cudaSuccess;
    philox_debug_kernel<<<(n + 127) / 128, 128, 0, stream>>>(ck, out, n);
    return cudaGetLastError();
}

}  // namespace specinfer
