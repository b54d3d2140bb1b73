// api.cu — the extern "C" boundary of libspecinfer.so (include/specinfer.h).
//
// Host-side argument validation, per-device capability cache (sm_100 check, SM count, max
// dynamic shared memory), workspace layout, and the launches of the K1..K6 kernels.
#include <math.h>
#include <stdlib.h>
#include <string.h>

#include <mutex>

#include "common.cuh"
#include "gather.cuh"

namespace specinfer {
cudaError_t launch_tree_prepare(const specinfer_shape_t &s, const WsLayout &w, const int32_t *parent,
                                const int32_t *depth, const int32_t *prefix_len, const int32_t *n_nodes,
                                char *ws, int num_ctas, cudaStream_t stream);
cudaError_t launch_tree_attention(const specinfer_shape_t &s, const WsLayout &w, const void *q, const void *k,
                                  const void *v, const int32_t *prefix_len, const int32_t *n_nodes, void *out,
                                  char *ws, int num_sms, size_t max_smem, cudaStream_t stream,
                                  const int32_t *page_table = nullptr, int num_pages = 0, uint32_t flags = 0);
cudaError_t launch_verify_greedy(const specinfer_shape_t &s, const WsLayout &w, const float *logits,
                                 const int32_t *tree_tokens, const int32_t *parent, const int32_t *n_nodes,
                                 int32_t *acc_nodes, int32_t *acc_tokens, int32_t *n_acc, char *ws,
                                 cudaStream_t stream, const GatherDev *gather);
cudaError_t launch_gather_wait(const GatherDev &g, int32_t *table_out, cudaStream_t stream);
cudaError_t launch_verify_mss(const specinfer_shape_t &s, const WsLayout &w, const float *logits,
                              const int32_t *tree_tokens, const int32_t *parent, const int32_t *n_nodes,
                              const float *draft_probs, float temperature, uint64_t seed, uint64_t offset,
                              const int32_t *request_ids, int32_t *acc_nodes, int32_t *acc_tokens,
                              int32_t *n_acc, char *ws, cudaStream_t stream, const GatherDev *gather);
cudaError_t launch_verify_ns(const specinfer_shape_t &s, const WsLayout &w, const float *logits,
                             const int32_t *tree_tokens, const int32_t *parent, const int32_t *n_nodes,
                             float temperature, uint64_t seed, uint64_t offset, const int32_t *request_ids,
                             int32_t *acc_nodes, int32_t *acc_tokens, int32_t *n_acc, char *ws, cudaStream_t stream);
cudaError_t launch_kv_commit(const specinfer_shape_t &s, void *k_all, void *v_all, int32_t *prefix_len,
                             const int32_t *acc_nodes, const int32_t *n_acc, cudaStream_t stream,
                             const int32_t *page_table = nullptr, int num_pages = 0);
cudaError_t launch_leaf_paths(const specinfer_shape_t &s, const int32_t *parent, const int32_t *n_nodes,
                              int32_t *paths, int32_t *path_len, int32_t *n_leaves, int32_t *status,
                              cudaStream_t stream);
cudaError_t launch_sequence_pack(const specinfer_shape_t &s, int num_seqs, int seq_max_seq, const int32_t *seq_map,
                                 const int32_t *paths, const int32_t *path_len, const int32_t *prefix_len,
                                 const void *q, const void *k, const void *v, void *q_seq, void *k_seq, void *v_seq,
                                 int32_t *seq_parent, int32_t *seq_depth, int32_t *seq_prefix, int32_t *seq_n,
                                 cudaStream_t stream);
cudaError_t launch_expansion_topology(const specinfer_shape_t &s, const int32_t *ks, int m, int32_t *parent,
                                      int32_t *depth, int32_t *n_nodes, cudaStream_t stream);
cudaError_t launch_expand_step(const specinfer_shape_t &s, int level, const float *ssm_logits, int F, float temperature,
                               const int32_t *parent, const int32_t *depth, const int32_t *n_nodes, int32_t *tokens,
                               float *draft_probs, int32_t *status, cudaStream_t stream);
cudaError_t launch_tree_merge(const specinfer_shape_t &s, int T, int Nin, const int32_t *in_parent,
                              const int32_t *in_tokens, const int32_t *in_n, int32_t *parent, int32_t *depth,
                              int32_t *tokens, int32_t *n_nodes, int32_t *node_map, int32_t *status,
                              cudaStream_t stream);
cudaError_t launch_tree_rope(const specinfer_shape_t &s, void *q, void *k, const int32_t *prefix_len,
                             const int32_t *depth, const int32_t *n_nodes, float base, cudaStream_t stream);
cudaError_t launch_philox_debug(const uint32_t *ck, uint32_t *out, int n, cudaStream_t stream);
cudaError_t launch_hbm_read_probe(const void *src, size_t bytes, int num_sms, cudaStream_t stream);
#ifdef SPECINFER_DEBUG_HOOKS
extern unsigned long long *g_attn_trace;
extern int g_attn_debug_flags;
extern unsigned long long *g_mss_trace;
#endif
}  // namespace specinfer

using namespace specinfer;

namespace {

struct DeviceInfo {
    bool valid = false;
    bool sm100 = false;
    int num_sms = 0;
    size_t max_smem = 0;
};

DeviceInfo g_dev[64];
std::mutex g_mu;

bool device_info(DeviceInfo *out) {
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) return false;
    std::lock_guard<std::mutex> lk(g_mu);
    DeviceInfo &d = g_dev[dev];
    if (!d.valid) {
        int major = 0, minor = 0, sms = 0, smem = 0;
        if (cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, dev) != cudaSuccess) return false;
        cudaDeviceGetAttribute(&minor, cudaDevAttrComputeCapabilityMinor, dev);
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        cudaDeviceGetAttribute(&smem, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
        d.sm100 = (major == 10 && minor == 0);
        d.num_sms = sms;
        d.max_smem = (size_t)smem;
        d.valid = true;
    }
    *out = d;
    return true;
}

// the workspace layout / attention schedule of a shape on this device (the debug build can switch
// the split-KV cluster mode off: experiment flag 64)
WsLayout layout(const specinfer_shape_t &s, int num_sms) {
#ifdef SPECINFER_DEBUG_HOOKS
    WsLayout w = ws_layout(s, num_sms, !(g_attn_debug_flags & 64));
    if (const char *gs = getenv("SPECINFER_DEBUG_GRID")) {   // experiment: persistent grid of N CTAs
        const int g = atoi(gs);
        if (g > 0 && g <= w.max_ctas && w.lanes == 1) {
            w.splitk = 1;
            w.grid = g;
        }
    }
    return w;
#else
    return ws_layout(s, num_sms);
#endif
}

specinfer_status_t check_shape(const specinfer_shape_t *s) {
    if (!s) return SPECINFER_ERR_INVALID_ARG;
    if (s->batch < 1 || s->max_nodes < 1 || s->num_q_heads < 1 || s->num_kv_heads < 1 || s->max_seq < 1 ||
        s->max_depth < 0)
        return SPECINFER_ERR_INVALID_ARG;
    if (s->head_dim != kHeadDim) return SPECINFER_ERR_UNSUPPORTED;
    if (s->max_nodes > kMaxNodes) return SPECINFER_ERR_UNSUPPORTED;
    if (s->num_q_heads % s->num_kv_heads != 0) return SPECINFER_ERR_UNSUPPORTED;
    if (s->num_q_heads / s->num_kv_heads > 64) return SPECINFER_ERR_UNSUPPORTED;
    if ((long long)s->batch * s->num_kv_heads * s->max_seq > (1ll << 31) - 1) return SPECINFER_ERR_UNSUPPORTED;
    return SPECINFER_OK;
}

specinfer_status_t check_device(DeviceInfo *d) {
    if (!device_info(d)) return SPECINFER_ERR_CUDA;
    if (!d->sm100) return SPECINFER_ERR_UNSUPPORTED;
    return SPECINFER_OK;
}

specinfer_status_t check_ws(const void *ws) {
    if (!ws || (reinterpret_cast<uintptr_t>(ws) & 255u) != 0) return SPECINFER_ERR_WORKSPACE;
    return SPECINFER_OK;
}

// the verifiers read logits / draft rows with 128-bit loads: the row bases must be 16-byte aligned
bool misaligned16(const void *a, const void *b = nullptr) {
    return ((reinterpret_cast<uintptr_t>(a) | reinterpret_cast<uintptr_t>(b)) & 15u) != 0;
}

// host validation of a gather descriptor (NEXT-4a) against the verify shape
specinfer_status_t gather_dev(const specinfer_gather_t *g, const specinfer_shape_t &s, GatherDev *out) {
    if (g->world < 1 || g->world > SPECINFER_MAX_PEERS || g->rank < 0 || g->rank >= g->world) return SPECINFER_ERR_INVALID_ARG;
    if (g->rows_per_rank < s.batch || g->row_len != 2 * (s.max_depth + 1) + 1 || !g->state)
        return SPECINFER_ERR_INVALID_ARG;
    GatherDev d{};
    for (int r = 0; r < g->world; ++r) {
        if (!g->recv[r] || !g->flags[r]) return SPECINFER_ERR_INVALID_ARG;
        d.recv[r] = g->recv[r];
        d.flags[r] = g->flags[r];
    }
    d.state = g->state;
    d.world = g->world;
    d.rank = g->rank;
    d.rows_per_rank = g->rows_per_rank;
    d.row_len = g->row_len;
    d.nreq = s.batch;
    *out = d;
    return SPECINFER_OK;
}

specinfer_status_t from_cuda(cudaError_t e) { return e == cudaSuccess ? SPECINFER_OK : SPECINFER_ERR_CUDA; }

#define SPI_TRY(x)                                 \
    do {                                           \
        specinfer_status_t _s = (x);               \
        if (_s != SPECINFER_OK) return _s;         \
    } while (0)

}  // namespace

extern "C" {

size_t specinfer_workspace_size(const specinfer_shape_t *shape) {
    if (check_shape(shape) != SPECINFER_OK) return 0;
    DeviceInfo d;
    const int sms = device_info(&d) ? d.num_sms : 148;
    return layout(*shape, sms > 0 ? sms : 148).total;
}

specinfer_status_t specinfer_tree_prepare(const specinfer_shape_t *shape, const int32_t *parent,
                                          const int32_t *depth, const int32_t *prefix_len, const int32_t *n_nodes,
                                          void *workspace, specinfer_stream_t stream) {
    SPI_TRY(check_shape(shape));
    if (!parent || !depth || !prefix_len || !n_nodes) return SPECINFER_ERR_INVALID_ARG;
    SPI_TRY(check_ws(workspace));
    DeviceInfo d;
    SPI_TRY(check_device(&d));
    const WsLayout w = layout(*shape, d.num_sms);
    return from_cuda(launch_tree_prepare(*shape, w, parent, depth, prefix_len, n_nodes,
                                         reinterpret_cast<char *>(workspace), w.grid,
                                         (cudaStream_t)stream));
}

specinfer_status_t specinfer_tree_attention_ex(const specinfer_shape_t *shape, const void *q, const void *k_cache,
                                               const void *v_cache, const int32_t *parent, const int32_t *depth,
                                               const int32_t *prefix_len, const int32_t *n_nodes, void *out,
                                               void *workspace, uint32_t flags, specinfer_stream_t stream) {
    SPI_TRY(check_shape(shape));
    if (!q || !k_cache || !v_cache || !parent || !depth || !prefix_len || !n_nodes || !out)
        return SPECINFER_ERR_INVALID_ARG;
    if ((reinterpret_cast<uintptr_t>(q) | reinterpret_cast<uintptr_t>(k_cache) |
         reinterpret_cast<uintptr_t>(v_cache) | reinterpret_cast<uintptr_t>(out)) & 15u)
        return SPECINFER_ERR_INVALID_ARG;
    if (flags & ~(uint32_t)SPECINFER_ATTN_EARLY_PREFIX) return SPECINFER_ERR_INVALID_ARG;
    SPI_TRY(check_ws(workspace));
    DeviceInfo d;
    SPI_TRY(check_device(&d));
    const WsLayout w = layout(*shape, d.num_sms);
    return from_cuda(launch_tree_attention(*shape, w, q, k_cache, v_cache, prefix_len, n_nodes, out,
                                           reinterpret_cast<char *>(workspace), w.grid, d.max_smem,
                                           (cudaStream_t)stream, nullptr, 0, flags));
}

specinfer_status_t specinfer_tree_attention(const specinfer_shape_t *shape, const void *q, const void *k_cache,
                                            const void *v_cache, const int32_t *parent, const int32_t *depth,
                                            const int32_t *prefix_len, const int32_t *n_nodes, void *out,
                                            void *workspace, specinfer_stream_t stream) {
    return specinfer_tree_attention_ex(shape, q, k_cache, v_cache, parent, depth, prefix_len, n_nodes, out, workspace,
                                       0u, stream);
}

specinfer_status_t specinfer_tree_attention_paged(const specinfer_shape_t *shape, const void *q, const void *k_pages,
                                                  const void *v_pages, int32_t num_pages, const int32_t *page_table,
                                                  const int32_t *parent, const int32_t *depth,
                                                  const int32_t *prefix_len, const int32_t *n_nodes, void *out,
                                                  void *workspace, specinfer_stream_t stream) {
    SPI_TRY(check_shape(shape));
    if (!q || !k_pages || !v_pages || !page_table || num_pages < 1 || !parent || !depth || !prefix_len ||
        !n_nodes || !out)
        return SPECINFER_ERR_INVALID_ARG;
    if ((long long)num_pages * shape->num_kv_heads * kKeyTile > (1ll << 31) - 1) return SPECINFER_ERR_UNSUPPORTED;
    if ((reinterpret_cast<uintptr_t>(q) | reinterpret_cast<uintptr_t>(k_pages) |
         reinterpret_cast<uintptr_t>(v_pages) | reinterpret_cast<uintptr_t>(out)) & 15u)
        return SPECINFER_ERR_INVALID_ARG;
    SPI_TRY(check_ws(workspace));
    DeviceInfo d;
    SPI_TRY(check_device(&d));
    const WsLayout w = layout(*shape, d.num_sms);
    return from_cuda(launch_tree_attention(*shape, w, q, k_pages, v_pages, prefix_len, n_nodes, out,
                                           reinterpret_cast<char *>(workspace), w.grid, d.max_smem,
                                           (cudaStream_t)stream, page_table, num_pages));
}

specinfer_status_t specinfer_kv_commit_paged(const specinfer_shape_t *shape, void *k_pages_all, void *v_pages_all,
                                             int32_t num_pages, const int32_t *page_table, int32_t *prefix_len,
                                             const int32_t *accepted_nodes, const int32_t *n_accepted,
                                             specinfer_stream_t stream) {
    SPI_TRY(check_shape(shape));
    if (shape->num_layers < 1 || num_pages < 1) return SPECINFER_ERR_INVALID_ARG;
    if (!k_pages_all || !v_pages_all || !page_table || !prefix_len || !accepted_nodes || !n_accepted)
        return SPECINFER_ERR_INVALID_ARG;
    if ((reinterpret_cast<uintptr_t>(k_pages_all) | reinterpret_cast<uintptr_t>(v_pages_all)) & 15u)
        return SPECINFER_ERR_INVALID_ARG;
    DeviceInfo d;
    SPI_TRY(check_device(&d));
    return from_cuda(launch_kv_commit(*shape, k_pages_all, v_pages_all, prefix_len, accepted_nodes, n_accepted,
                                      (cudaStream_t)stream, page_table, num_pages));
}

specinfer_status_t specinfer_tree_rope(const specinfer_shape_t *shape, void *q, void *k_cache,
                                      const int32_t *prefix_len, const int32_t *depth, const int32_t *n_nodes,
                                      float rope_base, specinfer_stream_t stream) {
    SPI_TRY(check_shape(shape));
    if ((!q && !k_cache) || !prefix_len || !depth || !n_nodes || !(rope_base > 1.0f)) return SPECINFER_ERR_INVALID_ARG;
    if ((reinterpret_cast<uintptr_t>(q) | reinterpret_cast<uintptr_t>(k_cache)) & 3u) return SPECINFER_ERR_INVALID_ARG;
    DeviceInfo d;
    SPI_TRY(check_device(&d));
    return from_cuda(launch_tree_rope(*shape, q, k_cache, prefix_len, depth, n_nodes, rope_base, (cudaStream_t)stream));
}

specinfer_status_t specinfer_verify_greedy_ex(const specinfer_shape_t *shape, const float *logits,
                                              const int32_t *tree_tokens, const int32_t *parent,
                                              const int32_t *n_nodes, int32_t *accepted_nodes,
                                              int32_t *accepted_tokens, int32_t *n_accepted, void *workspace,
                                              const specinfer_gather_t *gather, specinfer_stream_t stream) {
    SPI_TRY(check_shape(shape));
    if (shape->vocab < 1) return SPECINFER_ERR_INVALID_ARG;
    if (!logits || !tree_tokens || !parent || !n_nodes || !accepted_nodes || !accepted_tokens || !n_accepted)
        return SPECINFER_ERR_INVALID_ARG;
    if (misaligned16(logits)) return SPECINFER_ERR_INVALID_ARG;
    GatherDev g{};
    if (gather) SPI_TRY(gather_dev(gather, *shape, &g));
    SPI_TRY(check_ws(workspace));
    DeviceInfo d;
    SPI_TRY(check_device(&d));
    const WsLayout w = layout(*shape, d.num_sms);
    return from_cuda(launch_verify_greedy(*shape, w, logits, tree_tokens, parent, n_nodes, accepted_nodes,
                                          accepted_tokens, n_accepted, reinterpret_cast<char *>(workspace),
                                          (cudaStream_t)stream, gather ? &g : nullptr));
}

specinfer_status_t specinfer_verify_greedy(const specinfer_shape_t *shape, const float *logits,
                                           const int32_t *tree_tokens, const int32_t *parent, const int32_t *n_nodes,
                                           int32_t *accepted_nodes, int32_t *accepted_tokens, int32_t *n_accepted,
                                           void *workspace, specinfer_stream_t stream) {
    return specinfer_verify_greedy_ex(shape, logits, tree_tokens, parent, n_nodes, accepted_nodes, accepted_tokens,
                                      n_accepted, workspace, nullptr, stream);
}

specinfer_status_t specinfer_verify_mss_ex(const specinfer_shape_t *shape, const float *logits,
                                           const int32_t *tree_tokens, const int32_t *parent, const int32_t *n_nodes,
                                           const float *draft_probs, float temperature, uint64_t seed, uint64_t offset,
                                           const int32_t *request_ids, int32_t *accepted_nodes,
                                           int32_t *accepted_tokens, int32_t *n_accepted, void *workspace,
                                           const specinfer_gather_t *gather, specinfer_stream_t stream) {
    SPI_TRY(check_shape(shape));
    if (shape->vocab < 1 || !(temperature > 0.f) || !isfinite(temperature)) return SPECINFER_ERR_INVALID_ARG;
    if (!logits || !tree_tokens || !parent || !n_nodes || !draft_probs || !accepted_nodes || !accepted_tokens ||
        !n_accepted)
        return SPECINFER_ERR_INVALID_ARG;
    if (misaligned16(logits, draft_probs)) return SPECINFER_ERR_INVALID_ARG;
    GatherDev g{};
    if (gather) SPI_TRY(gather_dev(gather, *shape, &g));
    SPI_TRY(check_ws(workspace));
    DeviceInfo d;
    SPI_TRY(check_device(&d));
    const WsLayout w = layout(*shape, d.num_sms);
    return from_cuda(launch_verify_mss(*shape, w, logits, tree_tokens, parent, n_nodes, draft_probs, temperature,
                                       seed, offset, request_ids, accepted_nodes, accepted_tokens, n_accepted,
                                       reinterpret_cast<char *>(workspace), (cudaStream_t)stream,
                                       gather ? &g : nullptr));
}

specinfer_status_t specinfer_verify_mss(const specinfer_shape_t *shape, const float *logits,
                                        const int32_t *tree_tokens, const int32_t *parent, const int32_t *n_nodes,
                                        const float *draft_probs, float temperature, uint64_t seed, uint64_t offset,
                                        const int32_t *request_ids, int32_t *accepted_nodes,
                                        int32_t *accepted_tokens, int32_t *n_accepted, void *workspace,
                                        specinfer_stream_t stream) {
    return specinfer_verify_mss_ex(shape, logits, tree_tokens, parent, n_nodes, draft_probs, temperature, seed, offset,
                                   request_ids, accepted_nodes, accepted_tokens, n_accepted, workspace, nullptr,
                                   stream);
}

specinfer_status_t specinfer_gather_wait(const specinfer_gather_t *gather, int32_t *table_out,
                                         specinfer_stream_t stream) {
    if (!gather) return SPECINFER_ERR_INVALID_ARG;
    specinfer_shape_t s{};
    s.batch = 1;
    s.max_depth = (gather->row_len - 3) / 2;
    GatherDev g{};
    SPI_TRY(gather_dev(gather, s, &g));
    DeviceInfo d;
    SPI_TRY(check_device(&d));
    return from_cuda(launch_gather_wait(g, table_out, (cudaStream_t)stream));
}

specinfer_status_t specinfer_verify_ns(const specinfer_shape_t *shape, const float *logits,
                                       const int32_t *tree_tokens, const int32_t *parent, const int32_t *n_nodes,
                                       float temperature, uint64_t seed, uint64_t offset,
                                       const int32_t *request_ids, int32_t *accepted_nodes,
                                       int32_t *accepted_tokens, int32_t *n_accepted, void *workspace,
                                       specinfer_stream_t stream) {
    SPI_TRY(check_shape(shape));
    if (shape->vocab < 1 || !(temperature > 0.f) || !isfinite(temperature)) return SPECINFER_ERR_INVALID_ARG;
    if (!logits || !tree_tokens || !parent || !n_nodes || !accepted_nodes || !accepted_tokens || !n_accepted)
        return SPECINFER_ERR_INVALID_ARG;
    if (misaligned16(logits)) return SPECINFER_ERR_INVALID_ARG;
    SPI_TRY(check_ws(workspace));
    DeviceInfo d;
    SPI_TRY(check_device(&d));
    const WsLayout w = layout(*shape, d.num_sms);
    return from_cuda(launch_verify_ns(*shape, w, logits, tree_tokens, parent, n_nodes, temperature, seed, offset,
                                      request_ids, accepted_nodes, accepted_tokens, n_accepted,
                                      reinterpret_cast<char *>(workspace), (cudaStream_t)stream));
}

specinfer_status_t specinfer_kv_commit(const specinfer_shape_t *shape, void *k_cache_all, void *v_cache_all,
                                       int32_t *prefix_len, const int32_t *accepted_nodes, const int32_t *n_accepted,
                                       specinfer_stream_t stream) {
    SPI_TRY(check_shape(shape));
    if (shape->num_layers < 1) return SPECINFER_ERR_INVALID_ARG;
    if (!k_cache_all || !v_cache_all || !prefix_len || !accepted_nodes || !n_accepted)
        return SPECINFER_ERR_INVALID_ARG;
    if ((reinterpret_cast<uintptr_t>(k_cache_all) | reinterpret_cast<uintptr_t>(v_cache_all)) & 15u)
        return SPECINFER_ERR_INVALID_ARG;
    DeviceInfo d;
    SPI_TRY(check_device(&d));
    return from_cuda(launch_kv_commit(*shape, k_cache_all, v_cache_all, prefix_len, accepted_nodes, n_accepted,
                                      (cudaStream_t)stream));
}

specinfer_status_t specinfer_leaf_paths(const specinfer_shape_t *shape, const int32_t *parent,
                                        const int32_t *n_nodes, int32_t *paths, int32_t *path_len,
                                        int32_t *n_leaves, void *workspace, specinfer_stream_t stream) {
    SPI_TRY(check_shape(shape));
    if (!parent || !n_nodes || !paths || !path_len || !n_leaves) return SPECINFER_ERR_INVALID_ARG;
    if (workspace) SPI_TRY(check_ws(workspace));
    DeviceInfo d;
    SPI_TRY(check_device(&d));
    return from_cuda(launch_leaf_paths(*shape, parent, n_nodes, paths, path_len, n_leaves,
                                       reinterpret_cast<int32_t *>(workspace), (cudaStream_t)stream));
}

specinfer_status_t specinfer_sequence_pack(const specinfer_shape_t *shape, int32_t num_seqs, int32_t seq_max_seq,
                                           const int32_t *seq_map, const int32_t *paths, const int32_t *path_len,
                                           const int32_t *prefix_len, const void *q, const void *k_cache,
                                           const void *v_cache, void *q_seq, void *k_seq, void *v_seq,
                                           int32_t *seq_parent, int32_t *seq_depth, int32_t *seq_prefix_len,
                                           int32_t *seq_n_nodes, specinfer_stream_t stream) {
    SPI_TRY(check_shape(shape));
    if (num_seqs < 0 || seq_max_seq < 1) return SPECINFER_ERR_INVALID_ARG;
    if (num_seqs > 0 && (!seq_map || !paths || !path_len || !prefix_len || !q || !k_cache || !v_cache || !q_seq ||
                         !k_seq || !v_seq || !seq_parent || !seq_depth || !seq_prefix_len || !seq_n_nodes))
        return SPECINFER_ERR_INVALID_ARG;
    if ((reinterpret_cast<uintptr_t>(q) | reinterpret_cast<uintptr_t>(k_cache) | reinterpret_cast<uintptr_t>(v_cache) |
         reinterpret_cast<uintptr_t>(q_seq) | reinterpret_cast<uintptr_t>(k_seq) | reinterpret_cast<uintptr_t>(v_seq)) &
        15u)
        return SPECINFER_ERR_INVALID_ARG;
    DeviceInfo d;
    SPI_TRY(check_device(&d));
    return from_cuda(launch_sequence_pack(*shape, num_seqs, seq_max_seq, seq_map, paths, path_len, prefix_len, q,
                                          k_cache, v_cache, q_seq, k_seq, v_seq, seq_parent, seq_depth,
                                          seq_prefix_len, seq_n_nodes, (cudaStream_t)stream));
}

specinfer_status_t specinfer_expansion_topology(const specinfer_shape_t *shape, const int32_t *expansion,
                                                int32_t m, int32_t *parent, int32_t *depth, int32_t *n_nodes,
                                                specinfer_stream_t stream) {
    SPI_TRY(check_shape(shape));
    if (!expansion || m < 0 || m > 16 || m > shape->max_depth || !parent || !depth || !n_nodes)
        return SPECINFER_ERR_INVALID_ARG;
    long long n = 1, level = 1;
    for (int i = 0; i < m; ++i) {
        if (expansion[i] < 1 || expansion[i] > 8) return SPECINFER_ERR_INVALID_ARG;
        level *= expansion[i];
        n += level;
        if (n > shape->max_nodes) return SPECINFER_ERR_INVALID_ARG;
    }
    DeviceInfo d;
    SPI_TRY(check_device(&d));
    return from_cuda(launch_expansion_topology(*shape, expansion, m, parent, depth, n_nodes, (cudaStream_t)stream));
}

specinfer_status_t specinfer_expand_step(const specinfer_shape_t *shape, int32_t level, int32_t num_frontier,
                                         const float *ssm_logits, float temperature, const int32_t *parent,
                                         const int32_t *depth, const int32_t *n_nodes, int32_t *tree_tokens,
                                         float *draft_probs, void *workspace, specinfer_stream_t stream) {
    SPI_TRY(check_shape(shape));
    if (shape->vocab < 1 || level < 0 || num_frontier < 0 || !(temperature > 0.f) || !isfinite(temperature))
        return SPECINFER_ERR_INVALID_ARG;
    if (!ssm_logits || !parent || !depth || !n_nodes || !tree_tokens) return SPECINFER_ERR_INVALID_ARG;
    if (workspace) SPI_TRY(check_ws(workspace));
    DeviceInfo d;
    SPI_TRY(check_device(&d));
    if (num_frontier == 0) return SPECINFER_OK;
    return from_cuda(launch_expand_step(*shape, level, ssm_logits, num_frontier, temperature, parent, depth, n_nodes,
                                        tree_tokens, draft_probs, reinterpret_cast<int32_t *>(workspace),
                                        (cudaStream_t)stream));
}

specinfer_status_t specinfer_tree_merge(const specinfer_shape_t *shape, int32_t num_inputs, int32_t input_nodes,
                                        const int32_t *in_parent, const int32_t *in_tokens, const int32_t *in_n,
                                        int32_t *parent, int32_t *depth, int32_t *tree_tokens, int32_t *n_nodes,
                                        int32_t *node_map, void *workspace, specinfer_stream_t stream) {
    SPI_TRY(check_shape(shape));
    if (num_inputs < 1 || input_nodes < 1 || input_nodes > kMaxNodes) return SPECINFER_ERR_INVALID_ARG;
    if (!in_parent || !in_tokens || !in_n || !parent || !depth || !tree_tokens || !n_nodes || !node_map)
        return SPECINFER_ERR_INVALID_ARG;
    if (workspace) SPI_TRY(check_ws(workspace));
    DeviceInfo d;
    SPI_TRY(check_device(&d));
    return from_cuda(launch_tree_merge(*shape, num_inputs, input_nodes, in_parent, in_tokens, in_n, parent, depth,
                                       tree_tokens, n_nodes, node_map, reinterpret_cast<int32_t *>(workspace),
                                       (cudaStream_t)stream));
}

specinfer_status_t specinfer_read_device_status(const void *workspace, specinfer_stream_t stream,
                                                int32_t *status_bits_out) {
    SPI_TRY(check_ws(workspace));
    int32_t bits = 0;
    // the status word sits at offset 0 of every workspace layout
    cudaError_t e = cudaMemcpyAsync(&bits, workspace, sizeof(bits), cudaMemcpyDeviceToHost, (cudaStream_t)stream);
    if (e == cudaSuccess) e = cudaStreamSynchronize((cudaStream_t)stream);
    if (e != cudaSuccess) return SPECINFER_ERR_CUDA;
    if (status_bits_out) *status_bits_out = bits;
    return (bits & kStatusBadTree) ? SPECINFER_ERR_BAD_TREE : SPECINFER_OK;
}

specinfer_status_t specinfer_philox_debug(const uint32_t *ctr_key, uint32_t *out, int32_t n,
                                          specinfer_stream_t stream) {
    if (n < 0 || (n > 0 && (!ctr_key || !out))) return SPECINFER_ERR_INVALID_ARG;
    DeviceInfo d;
    SPI_TRY(check_device(&d));
    return from_cuda(launch_philox_debug(ctr_key, out, n, (cudaStream_t)stream));
}

specinfer_status_t specinfer_hbm_read_probe(const void *src, size_t bytes, specinfer_stream_t stream) {
    if (bytes > 0 && !src) return SPECINFER_ERR_INVALID_ARG;
    if ((reinterpret_cast<uintptr_t>(src) | bytes) & 15u) return SPECINFER_ERR_INVALID_ARG;
    DeviceInfo d;
    SPI_TRY(check_device(&d));
    return from_cuda(launch_hbm_read_probe(src, bytes, d.num_sms, (cudaStream_t)stream));
}

void specinfer_debug_set_trace(void *trace) {
#ifdef SPECINFER_DEBUG_HOOKS
    // development build only (libspecinfer_debug.so): pipeline timestamps and experiment switches
    // (flags 1/2/4/8 make results invalid); the production library compiles all of it out
    g_attn_trace = reinterpret_cast<unsigned long long *>(trace);
    g_mss_trace = getenv("SPECINFER_TRACE_MSS") ? reinterpret_cast<unsigned long long *>(trace) : nullptr;
    if (g_mss_trace) g_attn_trace = nullptr;
    const char *f = getenv("SPECINFER_DEBUG_FLAGS");
    g_attn_debug_flags = f ? atoi(f) : 0;
#else
    (void)trace;
#endif
}

int32_t specinfer_debug_hooks_enabled(void) {
#ifdef SPECINFER_DEBUG_HOOKS
    return 1;
#else
    return 0;
#endif
}

int32_t specinfer_launches_per_call(const char *name) {
    if (!name) return -1;
    if (!strcmp(name, "tree_prepare")) return 2;     // validate+bitsets, schedule+status
    if (!strcmp(name, "tree_attention")) return 1;   // split combine fused (last piece merges)
    if (!strcmp(name, "tree_attention_ex")) return 1;
    if (!strcmp(name, "verify_greedy")) return 1;    // argmax + walk fused (last CTA walks)
    if (!strcmp(name, "verify_mss")) return 1;
    if (!strcmp(name, "verify_greedy_ex") || !strcmp(name, "verify_mss_ex")) return 1;  // gather fused
    if (!strcmp(name, "gather_wait")) return 1;
    if (!strcmp(name, "kv_commit")) return 2;        // copy, prefix update
    if (!strcmp(name, "leaf_paths")) return 1;
    if (!strcmp(name, "verify_ns")) return 1;
    if (!strcmp(name, "expansion_topology")) return 1;
    if (!strcmp(name, "tree_attention_paged")) return 1;
    if (!strcmp(name, "kv_commit_paged")) return 2;
    if (!strcmp(name, "expand_step")) return 1;
    if (!strcmp(name, "tree_merge")) return 1;         // race-argmax + walk fused (last CTA walks)
    if (!strcmp(name, "sequence_pack")) return 1;
    if (!strcmp(name, "tree_rope")) return 1;
    if (!strcmp(name, "hbm_read_probe")) return 1;
    return -1;
}

const char *specinfer_status_string(specinfer_status_t s) {
    switch (s) {
        case SPECINFER_OK: return "ok";
        case SPECINFER_ERR_INVALID_ARG: return "invalid argument";
        case SPECINFER_ERR_UNSUPPORTED: return "unsupported shape or device (needs sm_100, head_dim 128, Nmax <= 256)";
        case SPECINFER_ERR_CUDA: return "CUDA error";
        case SPECINFER_ERR_BAD_TREE: return "invalid token tree in at least one request";
        case SPECINFER_ERR_WORKSPACE: return "workspace NULL or not 256-byte aligned";
    }
    return "unknown status";
}

}  // extern "C"
