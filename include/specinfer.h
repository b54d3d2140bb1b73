/*
 * specinfer.h — C ABI of libspecinfer.so: the data-parallel hot path of SpecInfer's token-tree
 * verification (SpecInfer, ASPLOS'24), hand-written CUDA for B200 (sm_100a).
 *
 * PAPER.md passages the calls implement (line numbers of /root/reference/PAPER.md):
 *   specinfer_tree_prepare    Def. 3.1 L450-454 (token tree, S_u); L657-674 (topology-aware mask)
 *   specinfer_tree_attention  Alg. 2 line 6 TreeParallelDecode L385; Def. 4.1;
 *                             Eq. 1-4; footnote L627-628; L645-674 (one fused kernel)
 *   specinfer_verify_greedy   Alg. 2 VerifyGreedy L395-401; §4.3
 *   specinfer_verify_mss      Alg. 2 VerifyStochastic L403-425; Fig. 5; Thm 4.2
 *   specinfer_kv_commit       depth-first KV-cache update L635-644; tree-topology KV layout L659-661
 *   specinfer_expansion_topology, specinfer_expand_step, specinfer_tree_merge
 *                             NEXT-2: token-tree construction (§3)
 *   specinfer_tree_rope       NEXT-4: position encoding at P_b + depth[i] (Def. 4.1, A4)
 *   specinfer_tree_attention_paged, specinfer_kv_commit_paged
 *                             NEXT-4: paged KV cache (tree layout L659-661 over 128-slot pages)
 *   specinfer_verify_ns       NEXT-3: naive sampling, the baseline of Theorem 4.3 (L747-765)
 *   specinfer_leaf_paths,     NEXT-1 baseline: sequence-based parallel decoding (§4.2,
 *   specinfer_sequence_pack   Fig. 4 left L682, §6.5)
 * Readings of the paper where it is silent or garbled are numbered R1..R23 in DESIGN.md.
 *
 * General conventions
 *   - Every data pointer is a DEVICE pointer unless stated otherwise; the caller owns every
 *     buffer (allocation, lifetime, freeing).  The library never allocates device memory and
 *     keeps no global mutable state except a per-device capability cache (sm_100 check, SM
 *     count, shared-memory limit, and which kernels already carry their shared-memory
 *     attribute on that device; thread-safe).  The production build has no debug hooks.
 *   - Every call is asynchronous and stream-ordered on `stream` (a cudaStream_t; NULL = the
 *     legacy default stream).  Calls are CUDA-graph capturable.
 *   - Host-checkable errors (NULL pointer, unsupported shape, non-sm_100 device) are returned
 *     synchronously before any launch: SPECINFER_ERR_INVALID_ARG / SPECINFER_ERR_UNSUPPORTED.
 *     Launch failures return SPECINFER_ERR_CUDA (from cudaGetLastError).
 *   - Tree defects are only visible on the device; kernels record them in a sticky status word
 *     inside the workspace, skip the offending request (no attention output, n_accepted = 0)
 *     and continue.  Read it with specinfer_read_device_status (the CUDA async-error model).
 *   - Nothing throws across the ABI.
 *
 * Shapes and layouts (row-major, innermost last; B = batch, Nmax = max_nodes, Hq/Hkv = q/kv
 * heads, D = head_dim = 128, Smax = max_seq, L = num_layers, V = vocab, Dmax = max_depth):
 *   parent, depth, tree_tokens   int32 [B][Nmax]  node 0 is the root (parent -1, depth 0);
 *                                 nodes in topological order: 0 <= parent[i] < i (R5)
 *   prefix_len                   int32 [B]  committed KV length P_b, excluding the root (R18)
 *   n_nodes                      int32 [B]  1 <= n_b <= Nmax; rows i >= n_b are padding
 *   q, out                       bf16  [B][Nmax][Hq][D]
 *   k_cache, v_cache (one layer) bf16  [B][Hkv][Smax][D]; committed keys at slots [0, P_b),
 *                                 tree node i's key at slot P_b + i ("tree topology", L659-661)
 *   logits, draft_probs          fp32  [B][Nmax][V]
 *   accepted_nodes/tokens        int32 [B][Dmax+1]; n_accepted int32 [B]
 */
#ifndef SPECINFER_H_
#define SPECINFER_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct CUstream_st *specinfer_stream_t; /* == cudaStream_t */

typedef enum {
    SPECINFER_OK = 0,
    SPECINFER_ERR_INVALID_ARG = 1, /* NULL pointer or inconsistent shape */
    SPECINFER_ERR_UNSUPPORTED = 2, /* head_dim != 128, Nmax > 256, Hq % Hkv != 0, G > 64, device not sm_100 */
    SPECINFER_ERR_CUDA = 3,        /* a CUDA launch/runtime call failed */
    SPECINFER_ERR_BAD_TREE = 4,    /* (device status) at least one request's tree was invalid */
    SPECINFER_ERR_WORKSPACE = 5    /* workspace NULL or misaligned (needs 256-byte alignment) */
} specinfer_status_t;

typedef struct {
    int32_t batch;        /* B */
    int32_t max_nodes;    /* Nmax, 1..256 */
    int32_t num_q_heads;  /* Hq */
    int32_t num_kv_heads; /* Hkv; Hq % Hkv == 0, G = Hq/Hkv <= 64 */
    int32_t head_dim;     /* D, must be 128 */
    int32_t max_seq;      /* Smax; every request needs P_b + n_b <= Smax */
    int32_t num_layers;   /* L (kv_commit only) */
    int32_t vocab;        /* V (verify only) */
    int32_t max_depth;    /* Dmax; every node needs depth <= Dmax; path buffers hold Dmax+1 */
    float sm_scale;       /* 0 => 1/sqrt(head_dim) (R1: A = QK^T / sqrt(d)) */
    int64_t layer_stride; /* elements between consecutive layers' caches (kv_commit);
                             0 => B*Hkv*Smax*D (caches laid out [L][B][Hkv][Smax][D]) */
} specinfer_shape_t;

/* Bytes of device workspace the calls below need for `shape` (host call, no CUDA work other
 * than a device-attribute query).  One workspace holds one stream's state: it must not be
 * shared by calls in flight on different streams. */
size_t specinfer_workspace_size(const specinfer_shape_t *shape);

/* a0 (K1).  Validates every request's tree (parent/depth/n_nodes/prefix_len against Smax and
 * Dmax), builds the ancestor-or-self and descendant bitsets of the topology-aware mask
 * (L657-674) and the tree-attention work schedule, resets the status word and counters.
 * Must be called once per iteration (per tree) before the other calls that take `workspace`;
 * its results stay valid for every layer of that iteration.
 * workspace: device, >= specinfer_workspace_size bytes, 256-byte aligned. */
specinfer_status_t specinfer_tree_prepare(const specinfer_shape_t *shape, const int32_t *parent,
                                          const int32_t *depth, const int32_t *prefix_len,
                                          const int32_t *n_nodes, void *workspace,
                                          specinfer_stream_t stream);

/* a1-a3 (K2).  Tree attention for ONE layer (Def. 4.1): for each request b, q-head h
 * (kv-head g = h / (Hq/Hkv)) and node i < n_b,
 *   out[b][i][h] = sum_j softmax_j(sm_scale q.k_j) v_j  over key slots j in
 *                  [0, P_b) U { P_b + a : a ancestor-or-self of i }          (R2, L657-674)
 * computed in fp32 from bf16 inputs (tcgen05 tensor cores, TMA-staged K/V tiles shared by all
 * G*n_b query rows of a kv-head), rounded to bf16.  Masked keys get exactly zero weight.
 * Cache slots >= P_b + n_b are never used (may hold anything, NaN included).
 * parent/depth are accepted for the record of the call (the mask comes from `workspace`,
 * which tree_prepare built from the same arrays).  Rows i >= n_b, and all rows of an invalid
 * request, are left untouched.  k_cache/v_cache must be 16-byte aligned.
 * Work distribution: with enough (request, kv-head, row-block) items per SM the CTAs claim whole
 * items from a ticket counter in `workspace` (reset by tree_prepare; each call draws exactly one
 * ticket per item), so calls on one workspace must not overlap in time (one stream, as above) and
 * at most 2^32 / items calls may follow one tree_prepare.  Results do not depend on the order. */
specinfer_status_t specinfer_tree_attention(const specinfer_shape_t *shape, const void *q,
                                            const void *k_cache, const void *v_cache,
                                            const int32_t *parent, const int32_t *depth,
                                            const int32_t *prefix_len, const int32_t *n_nodes,
                                            void *out, void *workspace, specinfer_stream_t stream);

/* specinfer_tree_attention with launch flags (0 = specinfer_tree_attention exactly).
 * SPECINFER_ATTN_EARLY_PREFIX: the kernel's producers may read the attention schedule in
 * `workspace` and stage committed-prefix K/V tiles (slots < P_b) BEFORE the programmatic
 * dependency on the preceding kernel of `stream` resolves (programmatic dependent launch: that
 * kernel may still be running).  Valid only when the immediately preceding kernel on `stream` wrote
 * neither those cache slots nor the workspace schedule, i.e. it was not tree_prepare or kv_commit
 * for this state; the tree slots, q and everything else are still read after the dependency.
 * Consecutive layers' attention launches qualify (the bench passes it for every layer but the
 * first).  Unknown flag bits: SPECINFER_ERR_INVALID_ARG.  Results are identical either way. */
#define SPECINFER_ATTN_EARLY_PREFIX 1u
specinfer_status_t specinfer_tree_attention_ex(const specinfer_shape_t *shape, const void *q,
                                               const void *k_cache, const void *v_cache,
                                               const int32_t *parent, const int32_t *depth,
                                               const int32_t *prefix_len, const int32_t *n_nodes,
                                               void *out, void *workspace, uint32_t flags,
                                               specinfer_stream_t stream);

/* a4 (K4).  VerifyGreedy (Alg. 2): O(u) = lowest token id attaining max logits[u];
 * from the root, repeatedly move to the lowest-index child whose token equals O(u) (R7);
 * finally emit O(u).  Writes accepted_nodes[b] = [0, v1..vL], accepted_tokens[b] =
 * [t_v1..t_vL, O(vL)], n_accepted[b] = L + 1; unused entries -1.  Invalid trees: n_accepted 0.
 * Needs the workspace of tree_prepare for the same tree.  `logits` must be 16-byte aligned
 * (rows are read with 128-bit loads when V % 4 == 0), else SPECINFER_ERR_INVALID_ARG. */
specinfer_status_t specinfer_verify_greedy(const specinfer_shape_t *shape, const float *logits,
                                           const int32_t *tree_tokens, const int32_t *parent,
                                           const int32_t *n_nodes, int32_t *accepted_nodes,
                                           int32_t *accepted_tokens, int32_t *n_accepted,
                                           void *workspace, specinfer_stream_t stream);

/* a5 (K5).  VerifyStochastic / multi-step speculative sampling (Alg. 2) with the RNG
 * contract of DESIGN.md R9/R15 (Philox4x32-10, key = seed, counters from the global request
 * id request_ids[b] (NULL => b), the node, the rejection round and `offset` (low 32 bits)):
 * p = softmax(logits[u]/temperature); children tried in Philox-uniform order; accept child s
 * with token x iff p[x] > 0 and r*q_s[x] <= p[x] (q_s = draft_probs[s], the distribution s was
 * drawn from, R12); on reject p <- norm(max(0, p - q_s)) (kept if all zero, R11); after the
 * last rejection (or at a leaf) sample x_next ~ p by an exponential race.  Outputs as for
 * verify_greedy.  temperature > 0.  Needs the workspace of tree_prepare for the same tree.
 * `logits` and `draft_probs` must be 16-byte aligned, else SPECINFER_ERR_INVALID_ARG. */
specinfer_status_t specinfer_verify_mss(const specinfer_shape_t *shape, const float *logits,
                                        const int32_t *tree_tokens, const int32_t *parent,
                                        const int32_t *n_nodes, const float *draft_probs,
                                        float temperature, uint64_t seed, uint64_t offset,
                                        const int32_t *request_ids, int32_t *accepted_nodes,
                                        int32_t *accepted_tokens, int32_t *n_accepted,
                                        void *workspace, specinfer_stream_t stream);

/* NEXT-4a: the tokens-only exchange after verification (a7) fused into the
 * verifier.  Every rank r of `world` allocates (device memory, zero-initialised, owned by the
 * caller) a receive table recv_r int32 [2][world * rows_per_rank][row_len] (double-buffered by
 * step parity), arrival flags flags_r uint32 [world] and a local state uint32 [2]; the descriptor
 * holds EVERY rank's recv / flags pointers as mapped in this process (CUDA IPC / peer access over
 * NVLink; recv[rank] / flags[rank] are this rank's own) and this rank's state.  row_len =
 * 2 (Dmax + 1) + 1: a row is [n_accepted | accepted_tokens | accepted_nodes] of one request; request
 * b of rank r goes to row r * rows_per_rank + b (rows_per_rank >= every rank's batch; rows of absent
 * requests stay as the caller initialised them, zero = nothing accepted).
 * specinfer_verify_greedy_ex / specinfer_verify_mss_ex (gather NULL = the plain call): the CTA
 * that finishes a request stores its row into every rank's table (peer stores), the last request
 * of the rank releases the step's epoch on every rank's flag (system scope).
 * specinfer_gather_wait: waits (acquire) until every rank released this step's epoch to us, copies
 * the step's table to table_out int32 [world * rows_per_rank][row_len] (device, may be NULL) and
 * advances the local epoch.  Calls of one rank must alternate verify_*_ex, gather_wait on one stream
 * (graph-capturable: the epoch lives in `state`).  A rank that never publishes makes the others'
 * gather_wait trap after a watchdog timeout (launch failure).  Errors: INVALID_ARG for world
 * outside [1, SPECINFER_MAX_PEERS], rank >= world, rows_per_rank < batch, wrong row_len, NULL
 * pointers. */
#define SPECINFER_MAX_PEERS 8
typedef struct {
    int32_t world, rank, rows_per_rank, row_len;
    int32_t *recv[SPECINFER_MAX_PEERS];
    uint32_t *flags[SPECINFER_MAX_PEERS];
    uint32_t *state;
} specinfer_gather_t;
specinfer_status_t specinfer_verify_greedy_ex(const specinfer_shape_t *shape, const float *logits,
                                              const int32_t *tree_tokens, const int32_t *parent,
                                              const int32_t *n_nodes, int32_t *accepted_nodes,
                                              int32_t *accepted_tokens, int32_t *n_accepted,
                                              void *workspace, const specinfer_gather_t *gather,
                                              specinfer_stream_t stream);
specinfer_status_t specinfer_verify_mss_ex(const specinfer_shape_t *shape, const float *logits,
                                           const int32_t *tree_tokens, const int32_t *parent,
                                           const int32_t *n_nodes, const float *draft_probs,
                                           float temperature, uint64_t seed, uint64_t offset,
                                           const int32_t *request_ids, int32_t *accepted_nodes,
                                           int32_t *accepted_tokens, int32_t *n_accepted,
                                           void *workspace, const specinfer_gather_t *gather,
                                           specinfer_stream_t stream);
specinfer_status_t specinfer_gather_wait(const specinfer_gather_t *gather, int32_t *table_out,
                                         specinfer_stream_t stream);

/* NEXT-4: rotary position encoding of the tree (reading A4: node i of request b is token number
 * depth[i] after the committed prefix of S_u, Def. 4.1, so it is encoded at position
 * P_b + depth[i]; siblings share a position).  In place, one launch:
 *   q       bf16 [B][Nmax][Hq][128], rows i < n_b rotated (NULL: keys only);
 *   k_cache bf16 [B][Hkv][Smax][128], ONE layer, tree slots P_b + i (i < n_b) rotated (NULL:
 *           queries only); committed slots are assumed already encoded at their own positions.
 * Rotate-half pairs (d, d + 64), theta_d = fp32(rope_base^(-2d/128)), angle = fp32(pos) * theta_d
 * in fp32, rotation in fp32, rounded to bf16.  rope_base > 1 (LLaMA: 10000).  depth[] must be the
 * node depths (tree_prepare validates them); requests with n_b outside [1, Nmax] or
 * P_b + n_b > Smax are left untouched.  After kv_commit, committed slot P + j holds a key encoded at
 * P + j (path[j] has depth j).  Errors: INVALID_ARG (both q and k_cache NULL, NULL tree arrays,
 * rope_base <= 1, misaligned pointers), UNSUPPORTED / ERR_CUDA as elsewhere. */
specinfer_status_t specinfer_tree_rope(const specinfer_shape_t *shape, void *q, void *k_cache,
                                      const int32_t *prefix_len, const int32_t *depth,
                                      const int32_t *n_nodes, float rope_base, specinfer_stream_t stream);

/* NEXT-4: paged KV cache (for serving; same computation as tree_attention / kv_commit).
 * Keys of request b live in pages of 128 slots: slot s is row s % 128 of page
 * page_table[b][s / 128] (int32 [B][ceil(Smax / 128)], entries in [0, num_pages); pages covering
 * [0, P_b + n_b) must be valid and the pages of different requests distinct).  A page holds every
 * kv-head: k_pages / v_pages bf16 [num_pages][Hkv][128][128] for one layer (attention) or
 * [L][...] `layer_stride` apart (0 => num_pages*Hkv*128*128) for the commit.  Tree node i is at
 * slot P_b + i as in the contiguous layout.  Results are bit-identical to the contiguous calls on
 * the same data (same tiles, same schedule). */
specinfer_status_t specinfer_tree_attention_paged(const specinfer_shape_t *shape, const void *q,
                                                  const void *k_pages, const void *v_pages,
                                                  int32_t num_pages, const int32_t *page_table,
                                                  const int32_t *parent, const int32_t *depth,
                                                  const int32_t *prefix_len, const int32_t *n_nodes,
                                                  void *out, void *workspace, specinfer_stream_t stream);
specinfer_status_t specinfer_kv_commit_paged(const specinfer_shape_t *shape, void *k_pages_all,
                                             void *v_pages_all, int32_t num_pages,
                                             const int32_t *page_table, int32_t *prefix_len,
                                             const int32_t *accepted_nodes, const int32_t *n_accepted,
                                             specinfer_stream_t stream);

/* NEXT-3: naive sampling (NS), the verifier Theorem 4.3 compares MSS with (L747-765): at each
 * node u on the walk draw x ~ softmax(logits[u]/temperature) by the exponential race of
 * verify_mss step 4 at round 0 (same Philox counters, so a leaf draws the same token under both
 * verifiers); if a child of u carries token x (lowest index, R7) append it and continue, else
 * emit x and stop.  Outputs, workspace, alignment and error behaviour as verify_greedy. */
specinfer_status_t specinfer_verify_ns(const specinfer_shape_t *shape, const float *logits,
                                       const int32_t *tree_tokens, const int32_t *parent,
                                       const int32_t *n_nodes, float temperature, uint64_t seed,
                                       uint64_t offset, const int32_t *request_ids,
                                       int32_t *accepted_nodes, int32_t *accepted_tokens,
                                       int32_t *n_accepted, void *workspace,
                                       specinfer_stream_t stream);

/* NEXT-2: token-tree construction on the GPU (§3; Fig. 2, Fig. 3).
 *
 * specinfer_expansion_topology: the static expansion <k_1..k_m> (L476-483; `expansion` is a
 * HOST array of m ints, 1 <= k_i <= 8, m <= min(16, Dmax), 1 + sum_i prod_{j<=i} k_j <= Nmax):
 * every request gets the same tree, node ids in DFS preorder (Fig. 2 "Linearization", L314),
 * children of a node ordered by SSM rank (child j carries the node's (j+1)-th best token).
 * Writes parent/depth int32 [B][Nmax] (padding: -1 / 0) and n_nodes int32 [B].
 *
 * specinfer_expand_step: expansion step `level` (0-based): the frontier = the nodes of depth
 * `level` in DFS order, num_frontier of them; ssm_logits fp32 [B][num_frontier][V] holds the
 * SSM's next-token logits for each frontier node (row f for the f-th frontier node).  Every
 * frontier node's children (from parent[], in index order, at most 8) get its top tokens
 * (descending logit, lowest token id on ties, R7) in tree_tokens [B][Nmax].  If draft_probs
 * (fp32 [B][Nmax][V]) is not NULL, each child's row receives q = softmax(logits / temperature)
 * of its parent (R12, the distribution the child was drawn from).  More than 8 children: the
 * step writes nothing for that node and sets BAD_TREE in `workspace` (if not NULL).
 *
 * specinfer_tree_merge: token tree merge (Def. 3.2).  Inputs: num_inputs trees per
 * request, in_parent / in_tokens int32 [B][num_inputs][input_nodes] (topological order, roots
 * carrying the same token), in_n int32 [B][num_inputs] (0 = no tree).  Output: the tree whose
 * sequences S_v are exactly the union of the inputs' S_u, node ids in DFS preorder with
 * children in first-appearance order (inputs in order, nodes in index order): parent, depth,
 * tree_tokens [B][Nmax], n_nodes [B]; node_map [B][num_inputs][input_nodes] = merged id of each
 * input node (-1 beyond in_n).  Invalid input, differing roots, more than Nmax merged nodes or
 * depth > Dmax: n_nodes[b] = 0, node_map -1, BAD_TREE set in `workspace` (if not NULL). */
specinfer_status_t specinfer_expansion_topology(const specinfer_shape_t *shape,
                                                const int32_t *expansion, int32_t m,
                                                int32_t *parent, int32_t *depth, int32_t *n_nodes,
                                                specinfer_stream_t stream);
specinfer_status_t specinfer_expand_step(const specinfer_shape_t *shape, int32_t level,
                                         int32_t num_frontier, const float *ssm_logits,
                                         float temperature, const int32_t *parent,
                                         const int32_t *depth, const int32_t *n_nodes,
                                         int32_t *tree_tokens, float *draft_probs, void *workspace,
                                         specinfer_stream_t stream);
specinfer_status_t specinfer_tree_merge(const specinfer_shape_t *shape, int32_t num_inputs,
                                        int32_t input_nodes, const int32_t *in_parent,
                                        const int32_t *in_tokens, const int32_t *in_n,
                                        int32_t *parent, int32_t *depth, int32_t *tree_tokens,
                                        int32_t *n_nodes, int32_t *node_map, void *workspace,
                                        specinfer_stream_t stream);

/* NEXT-1: sequence-based parallel decoding, the baseline tree-based decoding replaces (§4.2
 * L622-632, Fig. 4 left L682, §6.5).  Not part of the hot path; used by the Fig. 11
 * ablation and by the tests that check tree attention == per-sequence causal attention.
 *
 * specinfer_leaf_paths: for each request, its leaves in node-index order (= DFS order for a
 * DFS-linearised tree) and their root paths: paths[b][r][0..len-1] = root..leaf node ids of
 * the r-th leaf (-1 padded), path_len[b][r] = depth(leaf) + 1 (0 for r >= n_leaves[b]).
 * Layouts: paths int32 [B][Nmax][Dmax+1], path_len int32 [B][Nmax], n_leaves int32 [B].
 * Invalid trees (bad parent / n_nodes, depth > Dmax): n_leaves[b] = 0 and, when `workspace`
 * is not NULL, the sticky BAD_TREE bit is set in it.  No other state is used. */
specinfer_status_t specinfer_leaf_paths(const specinfer_shape_t *shape, const int32_t *parent,
                                        const int32_t *n_nodes, int32_t *paths, int32_t *path_len,
                                        int32_t *n_leaves, void *workspace, specinfer_stream_t stream);

/* specinfer_sequence_pack: builds the sequence batch of sequence-based decoding for ONE layer.
 * Sequence s (0 <= s < num_seqs) is leaf seq_map[s][1] of request seq_map[s][0] (int32 [S][2],
 * host-chosen, e.g. all (b, r) with r < n_leaves[b]).  Writes, for every kv-head g:
 *   k_seq/v_seq [S][Hkv][seq_max_seq][128]: slots [0, P_b) = the request's committed prefix,
 *       slot P_b + j = the tree slot P_b + path[j] (its own cache, "a different key-value cache
 *       for each sequence", L627-628); seq_max_seq >= P_b + path_len;
 *   q_seq [S][Dmax+1][Hq][128]: row j = q of node path[j];
 *   seq_parent/seq_depth int32 [S][Dmax+1]: the chain j-1 / j; seq_prefix_len, seq_n_nodes
 *       int32 [S]: P_b and path_len.
 * The result is a valid input of specinfer_tree_prepare / specinfer_tree_attention with
 * shape {batch = S, max_nodes = Dmax+1, max_seq = seq_max_seq, heads as `shape`}. */
specinfer_status_t specinfer_sequence_pack(const specinfer_shape_t *shape, int32_t num_seqs,
                                           int32_t seq_max_seq, const int32_t *seq_map,
                                           const int32_t *paths, const int32_t *path_len,
                                           const int32_t *prefix_len, const void *q,
                                           const void *k_cache, const void *v_cache, void *q_seq,
                                           void *k_seq, void *v_seq, int32_t *seq_parent,
                                           int32_t *seq_depth, int32_t *seq_prefix_len,
                                           int32_t *seq_n_nodes, specinfer_stream_t stream);

/* a6 (K6).  Depth-first KV-cache commit (L635-644): for every layer l < L, request b with
 * n = n_accepted[b] > 0 and kv-head g: slot P_b + j <- old slot P_b + accepted_nodes[b][j]
 * for j < n (bit copy of K and V rows), then prefix_len[b] += n (device, in/out).
 * k_cache_all/v_cache_all: [L] caches `layer_stride` elements apart (0 = contiguous layers),
 * 16-byte aligned.  accepted_nodes rows have Dmax+1 entries (the verifiers' output).
 * Path contract (always met by the verifiers' output): path[0] = 0 (the root), strictly
 * increasing (hence path[j] >= j, which makes the in-place order safe), P_b + path[j] < Smax.
 * A caller-built path is committed only up to its first row that breaks the contract, and
 * n is clamped to Dmax+1: the copy and the prefix_len update use the same clamped count, so the
 * cache stays consistent (no status is reported: kv_commit takes no workspace). */
specinfer_status_t specinfer_kv_commit(const specinfer_shape_t *shape, void *k_cache_all,
                                       void *v_cache_all, int32_t *prefix_len,
                                       const int32_t *accepted_nodes, const int32_t *n_accepted,
                                       specinfer_stream_t stream);

/* Synchronises `stream` and returns SPECINFER_OK or SPECINFER_ERR_BAD_TREE from the sticky
 * device status word; *bad_request_mask_out (host, may be NULL) receives the status bits. */
specinfer_status_t specinfer_read_device_status(const void *workspace, specinfer_stream_t stream,
                                                int32_t *status_bits_out);

/* Debug/KAT entry: out[i][0..4) = Philox4x32-10(ctr = ctr_key[i][0..4), key = ctr_key[i][4..6))
 * computed by the device implementation used in verify_mss.  ctr_key/out are device pointers. */
specinfer_status_t specinfer_philox_debug(const uint32_t *ctr_key, uint32_t *out, int32_t n,
                                          specinfer_stream_t stream);

/* Development build only (libspecinfer_debug.so, compiled with -DSPECINFER_DEBUG_HOOKS by
 * `build_lib.py --debug-hooks`; the production libspecinfer.so compiles every hook out and this
 * call does nothing there): when `trace` (device, >= 8*64*12 + 4*1024 uint64) is non-NULL,
 * subsequent tree_attention launches record per-tile clock64() timestamps of CTAs 0-7 and
 * per-CTA entry / exit / first-load times; the environment variable SPECINFER_DEBUG_FLAGS is
 * read here (pipeline experiments that invalidate results).  Not thread-safe; process-global. */
void specinfer_debug_set_trace(void *trace);

/* 1 in the development build (debug hooks compiled in), 0 in the production library. */
int32_t specinfer_debug_hooks_enabled(void);

/* Measurement only: reads `bytes` (16-byte aligned, multiple of 16) of device memory
 * at `src` the way tree_attention streams its K/V tiles (32 KB bulk async copies into a 6-deep
 * shared-memory ring, one CTA per SM, no compute) and discards them: the practical HBM read
 * ceiling the attention kernel's bandwidth is compared with.  No output. */
specinfer_status_t specinfer_hbm_read_probe(const void *src, size_t bytes, specinfer_stream_t stream);

/* Number of kernel launches each call issues (for launch accounting in benchmarks). */
int32_t specinfer_launches_per_call(const char *call_name);

const char *specinfer_status_string(specinfer_status_t status);

#ifdef __cplusplus
}
#endif

#endif /* SPECINFER_H_ */
