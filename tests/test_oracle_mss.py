"""Pins for the oracle's multi-step speculative sampling (c4, Alg. 2).

The statistical tests use fixed seeds and fixed request ids, so pass/fail is deterministic; the
acceptance threshold for every chi-square test is p-value >= 1e-3.
"""
from fractions import Fraction

import numpy as np
import pytest
from scipy import stats

import oracle
from tests.conftest import load_golden

ALPHA = 1e-3


def test_philox_known_answers():
    """Philox4x32-10 known-answer vectors (Random123)."""
    g = load_golden("philox_kat.json")
    for vec in g["vectors"]:
        ctr = [int(x, 16) for x in vec["ctr"]]
        key = [int(x, 16) for x in vec["key"]]
        out = oracle.philox4x32_10(ctr, key)
        assert [f"{int(x):08x}" for x in out] == vec["out"]


def _batch(n_req, parent, V):
    Nmax = len(parent)
    par = np.tile(np.asarray(parent, np.int32), (n_req, 1))
    return par, np.full(n_req, Nmax, np.int32)


def _logp(p):
    p = np.asarray(p, np.float64)
    with np.errstate(divide="ignore"):
        lg = np.where(p > 0, np.log(p), -1e30)
    return lg.astype(np.float32)


def _norm(x):
    x = np.asarray(x, np.float64)
    return x / x.sum()


def _chi2_ok(counts, probs):
    counts = np.asarray(counts, np.float64)
    exp = np.asarray(probs, np.float64) * counts.sum()
    keep = exp > 0
    assert counts[~keep].sum() == 0, "outcome with zero probability observed"
    return stats.chisquare(counts[keep], exp[keep]).pvalue


def test_q_equals_p_always_accepts():
    """q = p => r q[x] <= p[x] for every r < 1: the first tried child is accepted (L409)."""
    V, n = 7, 6
    rng = np.random.default_rng(0)
    parent = np.arange(-1, n - 1, dtype=np.int32)
    R = 500
    par, nn = _batch(R, parent, V)
    p = rng.dirichlet(np.ones(V), size=n)
    logits = np.tile(_logp(p)[None], (R, 1, 1))
    draft = np.zeros_like(logits)
    toks = np.zeros((R, n), np.int32)
    for c in range(1, n):
        draft[:, c] = p[c - 1]
        toks[:, c] = rng.choice(V, size=R, p=p[c - 1])
    an, at, na, _ = oracle.verify_mss(logits, toks, par, nn, draft, seed=1)
    assert np.all(na == n)
    assert np.all(an[:, :n] == np.arange(n))


def test_disjoint_support_never_accepts_and_samples_p():
    """Disjoint supports: p[x] = 0 for every drafted x => every child is rejected, the residual
    max(0, p - q) = p, and x_next ~ p (L409, L416-423)."""
    V = 6
    p = _norm([0.1, 0.3, 0.6, 0, 0, 0])
    q = _norm([0, 0, 0, 0.2, 0.3, 0.5])
    parent = np.array([-1, 0, 0], np.int32)
    R = 60000
    rng = np.random.default_rng(1)
    par, nn = _batch(R, parent, V)
    logits = np.tile(_logp(p)[None, None], (R, 3, 1))
    draft = np.tile(q.astype(np.float32)[None, None], (R, 3, 1))
    toks = np.zeros((R, 3), np.int32)
    toks[:, 1:] = rng.choice(V, size=(R, 2), p=q)
    an, at, na, _ = oracle.verify_mss(logits, toks, par, nn, draft, seed=2)
    assert np.all(na == 1)
    counts = np.bincount(at[:, 0], minlength=V)
    assert _chi2_ok(counts, p) >= ALPHA


def test_single_child_is_classic_speculative_sampling():
    """One child = single-step speculative sampling ([5, 25], L766-769): acceptance rate
    sum_x min(p(x), q(x)), and the first emitted token ~ p (Theorem 4.2 with one SSM)."""
    V = 5
    p = _norm([0.05, 0.15, 0.4, 0.3, 0.1])
    q = _norm([0.3, 0.3, 0.1, 0.2, 0.1])
    parent = np.array([-1, 0], np.int32)
    R = 200000
    rng = np.random.default_rng(3)
    par, nn = _batch(R, parent, V)
    logits = np.tile(_logp(p)[None, None], (R, 2, 1))
    draft = np.tile(q.astype(np.float32)[None, None], (R, 2, 1))
    toks = np.zeros((R, 2), np.int32)
    toks[:, 1] = rng.choice(V, size=R, p=q)
    an, at, na, _ = oracle.verify_mss(logits, toks, par, nn, draft, seed=3)
    acc = (na == 2).mean()
    expect = np.minimum(p, q).sum()
    sigma = np.sqrt(expect * (1 - expect) / R)
    assert abs(acc - expect) < 4 * sigma
    counts = np.bincount(at[:, 0], minlength=V)
    assert _chi2_ok(counts, p) >= ALPHA


def test_theorem_4_2_two_levels_multiple_ssms():
    """Theorem 4.2 (L732-746): with children drawn i.i.d. from their SSM's q, the emitted tokens
    follow the LLM.  Toy LLM p(x1), p(x2 | x1) over V = 5; root has three children from three
    different SSMs; each child has two grandchildren.  The first two emitted tokens (taking the
    second from a simulated next iteration when only one was emitted) ~ p(x1) p(x2 | x1)."""
    V = 5
    rng = np.random.default_rng(4)
    p1 = _norm(rng.uniform(0.5, 1.5, V))
    p2 = np.stack([_norm(rng.uniform(0.2, 1.8, V)) for _ in range(V)])
    q_root = [_norm(rng.uniform(0.1, 2, V)) for _ in range(3)]
    q_next = np.stack([_norm(rng.uniform(0.1, 2, V)) for _ in range(V)])
    # tree: 0 -> {1 -> {2, 3}, 4 -> {5, 6}, 7 -> {8, 9}}  (DFS preorder)
    parent = np.array([-1, 0, 1, 1, 0, 4, 4, 0, 7, 7], np.int32)
    kids_of_root = [1, 4, 7]
    R = 200000
    par, nn = _batch(R, parent, V)
    n = len(parent)
    toks = np.zeros((R, n), np.int32)
    logits = np.zeros((R, n, V), np.float32)
    draft = np.zeros((R, n, V), np.float32)
    logits[:, 0] = _logp(p1)
    for si, c in enumerate(kids_of_root):
        toks[:, c] = rng.choice(V, size=R, p=q_root[si])
        draft[:, c] = q_root[si]
        logits[:, c] = _logp(p2)[toks[:, c]]
        for gc in (c + 1, c + 2):
            # grandchildren drafted from the SSM's next-step distribution given the child token
            u = rng.random(R)
            cdf = np.cumsum(q_next[toks[:, c]], axis=1)
            toks[:, gc] = np.minimum((u[:, None] > cdf).sum(1), V - 1)
            draft[:, gc] = q_next[toks[:, c]]
            logits[:, gc] = 0.0   # leaves: never entered except for final sampling
            logits[:, gc] = _logp(p2)[toks[:, gc]]  # (unused for x2)
    an, at, na, _ = oracle.verify_mss(logits, toks, par, nn, draft, seed=5, offset=0)
    x1 = at[:, 0].copy()
    x2 = np.where(na >= 2, at[:, 1], -1)
    # second iteration for requests that emitted a single token: root context x1,
    # two fresh children i.i.d. from q_next[x1]
    need = np.nonzero(na == 1)[0]
    m = len(need)
    par2 = np.tile(np.array([-1, 0, 0], np.int32), (m, 1))
    lg2 = np.zeros((m, 3, V), np.float32)
    lg2[:, 0] = _logp(p2)[x1[need]]
    dr2 = np.zeros((m, 3, V), np.float32)
    t2 = np.zeros((m, 3), np.int32)
    for c in (1, 2):
        u = rng.random(m)
        cdf = np.cumsum(q_next[x1[need]], axis=1)
        t2[:, c] = np.minimum((u[:, None] > cdf).sum(1), V - 1)
        dr2[:, c] = q_next[x1[need]]
    _, at2, na2, _ = oracle.verify_mss(lg2, t2, par2, np.full(m, 3, np.int32), dr2, seed=5,
                                       offset=1, request_ids=need.astype(np.int32))
    x2[need] = at2[:, 0]
    assert np.all(x2 >= 0)
    counts = np.bincount(x1 * V + x2, minlength=V * V)
    expect = (p1[:, None] * p2).reshape(-1)
    assert _chi2_ok(counts, expect) >= ALPHA


def _enumerate_mss(p, children, p_child):
    """Exact outcome distribution of Alg. 2 (L403-425) at a root whose children (token, q) are
    leaves, in rational arithmetic.  Outcome = tuple of emitted tokens."""
    out = {}

    def add(key, w):
        out[key] = out.get(key, Fraction(0)) + w

    def rec(p, H, w):
        if not H:
            for y, py in enumerate(p):
                if py > 0:
                    add((y,), w * py)
            return
        for s in H:
            ws = w / len(H)
            tok, q = children[s]
            if p[tok] > 0:
                acc = Fraction(1) if q[tok] == 0 else min(Fraction(1), p[tok] / q[tok])
            else:
                acc = Fraction(0)
            if acc > 0:
                for y, py in enumerate(p_child[s]):
                    if py > 0:
                        add((tok, y), ws * acc * py)
            if acc < 1:
                res = [max(Fraction(0), a - b) for a, b in zip(p, q)]
                S = sum(res)
                p2 = [r / S for r in res] if S > 0 else p
                rec(p2, [h for h in H if h != s], ws * (1 - acc))

    rec(list(p), list(range(len(children))), Fraction(1))
    return out


def test_exact_enumeration_fixed_drafts():
    """Brute force: enumerate Alg. 2's pick orders and accept/reject branches exactly (in
    rationals) for a fixed 3-child tree (duplicate tokens included); the oracle's empirical
    outcome frequencies over 2e5 request ids must match (chi-square)."""
    V = 4
    P = [Fraction(1, 10), Fraction(2, 10), Fraction(3, 10), Fraction(4, 10)]
    Qa = [Fraction(1, 2), Fraction(1, 4), Fraction(1, 8), Fraction(1, 8)]
    Qb = [Fraction(1, 8), Fraction(1, 8), Fraction(1, 4), Fraction(1, 2)]
    children = [(0, Qa), (0, Qa), (3, Qb)]            # two siblings carry token 0 (R13)
    PC = [[Fraction(1, 4)] * 4, [Fraction(1, 2), Fraction(1, 2), 0, 0], [0, 0, Fraction(1, 3), Fraction(2, 3)]]
    exact = _enumerate_mss(P, children, PC)
    assert sum(exact.values()) == 1
    parent = np.array([-1, 0, 0, 0], np.int32)
    R = 200000
    par, nn = _batch(R, parent, V)
    f = lambda fr: np.asarray([float(x) for x in fr])
    logits = np.zeros((R, 4, V), np.float32)
    logits[:, 0] = _logp(f(P))
    draft = np.zeros((R, 4, V), np.float32)
    toks = np.zeros((R, 4), np.int32)
    for c, (tok, q) in enumerate(children, start=1):
        toks[:, c] = tok
        draft[:, c] = f(q)
        logits[:, c] = _logp(f(PC[c - 1]))
    an, at, na, _ = oracle.verify_mss(logits, toks, par, nn, draft, seed=7)
    keys = sorted(exact)
    idx = {k: i for i, k in enumerate(keys)}
    counts = np.zeros(len(keys))
    for r in range(R):
        counts[idx[tuple(at[r, :na[r]].tolist())]] += 1
    assert _chi2_ok(counts, [float(exact[k]) for k in keys]) >= ALPHA


def test_theorem_4_3_in_expectation():
    """Theorem 4.3 (L754-765), read in expectation over the drafts (reading R22): MSS rejects
    no more often than naive sampling, whose rejection given the drafts is
    1 - sum_{distinct child tokens} p(x)."""
    V = 6
    rng = np.random.default_rng(8)
    for trial in range(3):
        p = _norm(rng.uniform(0.05, 1, V))
        q = _norm(rng.uniform(0.05, 1, V))
        k = 3
        parent = np.array([-1] + [0] * k, np.int32)
        R = 100000
        par, nn = _batch(R, parent, V)
        logits = np.tile(_logp(p)[None, None], (R, k + 1, 1))
        draft = np.tile(q.astype(np.float32)[None, None], (R, k + 1, 1))
        toks = np.zeros((R, k + 1), np.int32)
        toks[:, 1:] = rng.choice(V, size=(R, k), p=q)
        _, _, na, _ = oracle.verify_mss(logits, toks, par, nn, draft, seed=9 + trial)
        mss_rej = (na == 1).mean()
        covered = np.zeros(R)
        for x in range(V):
            covered += p[x] * (toks[:, 1:] == x).any(1)
        ns_rej = 1 - covered.mean()
        sigma = np.sqrt(mss_rej * (1 - mss_rej) / R) + np.sqrt(np.var(1 - covered) / R)
        assert mss_rej <= ns_rej + 4 * sigma


def test_temperature_and_request_id_invariances():
    """softmax(l / T) (R14): halving the logits at T = 1 equals T = 2 on the original logits.
    Results depend on the global request id, not on the batch position (R9; multi-GPU
    sharding invariance)."""
    V, n = 32, 9
    rng = np.random.default_rng(10)
    parent = np.array([-1, 0, 0, 1, 1, 2, 0, 6, 6], np.int32)
    R = 64
    par, nn = _batch(R, parent, V)
    logits = (3 * rng.standard_normal((R, n, V))).astype(np.float32)
    draft = rng.dirichlet(np.ones(V), size=(R, n)).astype(np.float32)
    toks = rng.integers(0, V, (R, n)).astype(np.int32)
    a = oracle.verify_mss(logits, toks, par, nn, draft, temperature=2.0, seed=11, offset=3)
    b = oracle.verify_mss(logits * 0.5, toks, par, nn, draft, temperature=1.0, seed=11, offset=3)
    for x, y in zip(a[:3], b[:3]):
        assert np.array_equal(x, y)
    perm = rng.permutation(R)
    c = oracle.verify_mss(logits[perm], toks[perm], par[perm], nn[perm], draft[perm],
                          temperature=2.0, seed=11, offset=3, request_ids=perm.astype(np.int32))
    for x, y in zip(a[:3], c[:3]):
        assert np.array_equal(x[perm], y)
    # a different offset changes the draws for at least one request
    d = oracle.verify_mss(logits, toks, par, nn, draft, temperature=2.0, seed=11, offset=4)
    assert not all(np.array_equal(x, y) for x, y in zip(a[:3], d[:3]))
