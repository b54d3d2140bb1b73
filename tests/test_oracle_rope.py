"""Pins for the oracle's rotary position encoding of the token tree (NEXT-4; reading A4 / DESIGN R29:
node i sits at position P_b + depth[i], Def. 4.1 L594-598 places u at index depth(u) of S_u after the
committed prefix).

Independent of the oracle's code: the complex-number form of a rotation (textbook), closed-form
angles, invariants (identity at 0, norm, relative position), and brute-force causal decoding of
the explicit sequence S_u with ordinary sequence positions 0, 1, 2, ...
"""
import numpy as np
import pytest
import torch

import oracle
import workloads as W

D = 128


def test_rope_position_zero_is_identity():
    x = np.random.default_rng(1).standard_normal((5, D))
    assert np.array_equal(oracle.rope_rotate(x, np.zeros(5, np.int64)), x)


def test_rope_matches_complex_multiplication():
    """(x_i + j x_{i+D/2}) * exp(j a_i) with a_i = fp32(pos) * fp32(base^(-2i/D))."""
    rng = np.random.default_rng(2)
    x = rng.standard_normal((7, D))
    pos = np.array([1, 2, 17, 300, 2048, 4103, 8447])
    theta = np.array([np.float32(10000.0 ** (-2.0 * i / D)) for i in range(D // 2)], np.float32)
    ang = np.array([[float(np.float32(np.float32(p) * t)) for t in theta] for p in pos])
    z = (x[:, :D // 2] + 1j * x[:, D // 2:]) * np.exp(1j * ang)
    want = np.concatenate([z.real, z.imag], axis=1)
    got = oracle.rope_rotate(x, pos)
    assert np.abs(got - want).max() < 1e-12


def test_rope_closed_form_unit_vectors():
    """Position 1, pair 0: theta_0 = 1 -> rotation by exactly one radian; pair D/2-1 at position
    p rotates by p * 10000^(-(D-2)/D)."""
    x = np.zeros(D)
    x[0] = 1.0
    y = oracle.rope_rotate(x, 1)
    assert abs(y[0] - np.cos(1.0)) < 1e-15 and abs(y[D // 2] - np.sin(1.0)) < 1e-15
    x = np.zeros(D)
    x[D // 2 - 1] = 1.0
    a = float(np.float32(np.float32(1000.0) * np.float32(10000.0 ** (-(D - 2) / D))))
    y = oracle.rope_rotate(x, 1000)
    assert abs(y[D // 2 - 1] - np.cos(a)) < 1e-15 and abs(y[D - 1] - np.sin(a)) < 1e-15


def test_rope_preserves_pair_norms():
    rng = np.random.default_rng(3)
    x = rng.standard_normal((4, D))
    y = oracle.rope_rotate(x, np.array([5, 77, 1024, 8191]))
    nx = x[:, :D // 2] ** 2 + x[:, D // 2:] ** 2
    ny = y[:, :D // 2] ** 2 + y[:, D // 2:] ** 2
    assert np.abs(nx - ny).max() < 1e-12


def test_rope_scores_depend_on_relative_position_only():
    """<R(p) q, R(p') k> = <R(p + s) q, R(p' + s) k> (small positions: fp32 angles exact enough)."""
    rng = np.random.default_rng(4)
    q, k = rng.standard_normal(D), rng.standard_normal(D)
    for p, pp, s in ((3, 1, 5), (10, 10, 7), (20, 4, 31)):
        a = oracle.rope_rotate(q, p) @ oracle.rope_rotate(k, pp)
        b = oracle.rope_rotate(q, p + s) @ oracle.rope_rotate(k, pp + s)
        assert abs(a - b) < 1e-4 * (1 + abs(a))


def test_tree_rope_positions_are_prefix_plus_depth():
    """Fig. 4 tree (L682): siblings share a position, a chain gets P, P+1, ... (= incremental
    decoding); rows / slots outside the tree are untouched."""
    parent = np.array([-1, 0, 1, 2, 2, 4, 1, 6])
    depth = np.array([0, 1, 2, 3, 3, 4, 2, 3])
    B, N, H, P, Smax = 1, 10, 2, 5, 20
    rng = np.random.default_rng(5)
    q = rng.standard_normal((B, N, H, D))
    k = rng.standard_normal((B, H, Smax, D))
    qr, kr = oracle.tree_rope(q, k, [P], depth[None], [8])
    for i in range(8):
        assert np.abs(qr[0, i] - oracle.rope_rotate(q[0, i], np.full(H, P + depth[i]))).max() == 0
        assert np.abs(kr[0, :, P + i] - oracle.rope_rotate(k[0, :, P + i], np.full(H, P + depth[i]))).max() == 0
    assert np.array_equal(qr[0, 8:], q[0, 8:])
    assert np.array_equal(kr[0, :, :P], k[0, :, :P]) and np.array_equal(kr[0, :, P + 8:], k[0, :, P + 8:])
    # siblings 3 and 4 (both depth 3) get identical rotations
    assert np.array_equal(oracle.rope_rotate(q[0, 3], np.full(H, P + 3)),
                          oracle.rope_rotate(q[0, 3], np.full(H, P + depth[4])))


@pytest.mark.parametrize("seed", [0, 1])
def test_tree_rope_attention_equals_sequence_decoding(seed):
    """End to end: tree attention over the position-encoded tree (oracle.tree_rope +
    oracle.tree_attention) gives, for every node u, the output of ordinary causal decoding of the
    explicit sequence S_u = prefix + root path whose token at sequence index j is encoded at
    position j (brute-force softmax here)."""
    rng = np.random.default_rng(10 + seed)
    parent, depth = W.random_tree(12, 5, 3, rng)
    n = len(parent)
    P, H, Smax = 9, 2, 9 + 12 + 1
    q = rng.standard_normal((1, 12, H, D))
    k_raw = rng.standard_normal((1, H, Smax, D))
    v = rng.standard_normal((1, H, Smax, D))
    # the committed prefix is stored encoded at its own positions 0..P-1; tree slots raw
    k = k_raw.copy()
    for j in range(P):
        k[0, :, j] = oracle.rope_rotate(k_raw[0, :, j], np.full(H, j))
    par = np.full((1, 12), -1, np.int64)
    dep = np.zeros((1, 12), np.int64)
    par[0, :n], dep[0, :n] = parent, depth
    qr, kr = oracle.tree_rope(q, k, [P], dep, [n])
    bf = lambda a: torch.as_tensor(np.asarray(a, np.float32)).to(torch.bfloat16)
    f64 = lambda a: bf(a).to(torch.float64).numpy()
    out = oracle.tree_attention(bf(qr), bf(kr), bf(v), par.astype(np.int32), dep.astype(np.int32),
                                np.array([P], np.int32), np.array([n], np.int32))
    scale = 1.0 / np.sqrt(D)
    for u in range(n):
        path = [u]
        while parent[path[-1]] != -1:
            path.append(parent[path[-1]])
        path = path[::-1]
        for h in range(H):
            # sequence S_u: prefix tokens 0..P-1 then the path; token at index j encoded at position j
            keys = [oracle.rope_rotate(k_raw[0, h, j], j) for j in range(P)]
            keys += [oracle.rope_rotate(k_raw[0, h, P + c], P + jj) for jj, c in enumerate(path)]
            vals = [v[0, h, j] for j in range(P)] + [v[0, h, P + c] for c in path]
            qq = f64(oracle.rope_rotate(q[0, u, h], P + len(path) - 1))
            s_ = f64(np.array(keys)) @ qq * scale
            w = np.exp(s_ - s_.max())
            want = (w[:, None] * f64(np.array(vals))).sum(0) / w.sum()
            assert np.abs(out[0, u, h] - want).max() < 1e-9, (u, h)
