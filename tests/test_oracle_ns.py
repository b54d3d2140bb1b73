"""Pins for the oracle's naive-sampling verifier (NEXT-3: "directly sampling
the next token x ~ P(u_i | U; LLM) and examining whether x is a child node"), the baseline of
Theorem 4.3 (L754-765).

Independent of the oracle's code: the closed-form distribution of NS (every emitted token is an
exact sample of the LLM distribution at its node, so the first token ~ p(root) and the walk
accepts at node u with probability sum_{x in child tokens(u)} p(x)); the greedy special case
(a one-hot p makes NS walk exactly the greedy path of Alg. 2 VerifyGreedy); Theorem 4.3 as an
inequality between MSS's empirical rejection and NS's; fixed seeds, chi-square p >= 1e-3.
"""
import numpy as np
from scipy import stats

import oracle
from tests.test_oracle_mss import ALPHA, _batch, _chi2_ok, _logp, _norm


def test_first_token_is_an_exact_sample_of_p():
    """Root-only tree: NS is plain sampling from p (L747-749): chi-square against p."""
    V, R = 9, 60000
    rng = np.random.default_rng(21)
    p = _norm(rng.uniform(0.01, 1, V))
    par, nn = _batch(R, [-1], V)
    logits = np.tile(_logp(p)[None, None], (R, 1, 1))
    toks = np.zeros((R, 1), np.int32)
    an, at, na, _ = oracle.verify_ns(logits, toks, par, nn, seed=5)
    assert np.all(na == 1) and np.all(an[:, 0] == 0)
    assert _chi2_ok(np.bincount(at[:, 0], minlength=V), p) >= ALPHA


def test_acceptance_probability_closed_form_and_output_distribution():
    """A root with children carrying tokens {0, 2}: NS accepts with probability p(0) + p(2)
    (binomial test); the emitted first token is ~ p regardless of the tree (chi-square); after
    accepting child c the second token is ~ p(. | c) (chi-square)."""
    V, R = 5, 80000
    rng = np.random.default_rng(22)
    p_root = _norm(rng.uniform(0.05, 1, V))
    p_c1 = _norm(rng.uniform(0.05, 1, V))
    p_c2 = _norm(rng.uniform(0.05, 1, V))
    parent = [-1, 0, 0]
    par, nn = _batch(R, parent, V)
    logits = np.stack([_logp(p_root), _logp(p_c1), _logp(p_c2)])[None].repeat(R, 0)
    toks = np.tile(np.array([0, 0, 2], np.int32), (R, 1))
    an, at, na, _ = oracle.verify_ns(logits, toks, par, nn, seed=6)
    acc = (na == 2)
    assert stats.binomtest(int(acc.sum()), R, p_root[0] + p_root[2]).pvalue >= ALPHA
    assert _chi2_ok(np.bincount(at[:, 0], minlength=V), p_root) >= ALPHA
    # accepted child follows the token: node 1 for token 0, node 2 for token 2
    assert np.all(an[acc, 1] == np.where(at[acc, 0] == 0, 1, 2))
    sel = acc & (an[:, 1] == 1)
    assert _chi2_ok(np.bincount(at[sel, 1], minlength=V), p_c1) >= ALPHA


def test_one_hot_llm_reduces_to_greedy():
    """With a one-hot LLM distribution (all other logits -inf) the only possible sample is the
    argmax, so NS follows exactly the greedy path (Alg. 2 VerifyGreedy, L395-401)."""
    rng = np.random.default_rng(23)
    V, n, R = 12, 10, 50
    parent = np.array([-1, 0, 0, 1, 1, 2, 3, 3, 6, 0], np.int32)
    par, nn = _batch(R, parent, V)
    logits = np.full((R, n, V), -np.inf, np.float32)
    arg = rng.integers(0, 4, (R, n))
    for b in range(R):
        logits[b, np.arange(n), arg[b]] = 0.0
    toks = rng.integers(0, 4, (R, n)).astype(np.int32)
    ns = oracle.verify_ns(logits, toks, par, nn, seed=7)
    gr = oracle.verify_greedy(np.where(np.isinf(logits), -1e30, logits).astype(np.float32), toks, par, nn,
                              path_len=ns[0].shape[1])
    for x, y in zip(ns[:3], gr):
        assert np.array_equal(x, y)


def test_theorem_4_3_mss_rejects_no_more_than_ns():
    """Theorem 4.3 (L754-765), in expectation over the drafts (R22): empirical rejection rate at
    the root of MSS <= that of NS, on the same trees, both from the oracle."""
    V = 6
    rng = np.random.default_rng(24)
    for trial in range(3):
        p = _norm(rng.uniform(0.05, 1, V))
        q = _norm(rng.uniform(0.05, 1, V))
        k = 3
        parent = np.array([-1] + [0] * k, np.int32)
        R = 60000
        par, nn = _batch(R, parent, V)
        logits = np.tile(_logp(p)[None, None], (R, k + 1, 1))
        draft = np.tile(q.astype(np.float32)[None, None], (R, k + 1, 1))
        toks = np.zeros((R, k + 1), np.int32)
        toks[:, 1:] = rng.choice(V, size=(R, k), p=q)
        _, _, na_m, _ = oracle.verify_mss(logits, toks, par, nn, draft, seed=30 + trial)
        _, _, na_n, _ = oracle.verify_ns(logits, toks, par, nn, seed=40 + trial)
        rm, rn = (na_m == 1).mean(), (na_n == 1).mean()
        sigma = np.sqrt(rm * (1 - rm) / R + rn * (1 - rn) / R)
        assert rm <= rn + 4 * sigma, (trial, rm, rn)


def test_leaf_sample_matches_mss_leaf_sample():
    """At a leaf both verifiers draw x_next from p with the same counters (round 0), so a
    root-only tree gives identical outputs under NS and MSS (RNG contract R15)."""
    V, R = 50, 200
    rng = np.random.default_rng(25)
    logits = (2 * rng.standard_normal((R, 1, V))).astype(np.float32)
    par, nn = _batch(R, [-1], V)
    toks = np.zeros((R, 1), np.int32)
    a = oracle.verify_ns(logits, toks, par, nn, seed=8, offset=2)
    b = oracle.verify_mss(logits, toks, par, nn, np.zeros_like(logits), seed=8, offset=2)
    for x, y in zip(a[:3], b[:3]):
        assert np.array_equal(x, y)
