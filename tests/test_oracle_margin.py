"""Pins for the oracle's per-decision margins and decision log (c4 MSS, NEXT-3 NS), which decide
whether a GPU/oracle mismatch may be boundary-excused (tests/mss_compare.py).

Each pin constructs a decision whose distance to its boundary is known by construction, from the
RNG contract alone (Philox4x32-10, pinned by the Random123 KATs in test_oracle_mss.py; counters of
DESIGN.md R9/R10/R15), and checks the oracle's outcome AND its reported margin:
  * accept test (Alg. 2, reading R10): accept iff r q[x] <= p[x]; we set q[x] so that
    r q[x] = p[x] (1 -/+ eps) and expect accept / reject with margin eps (relative);
  * final race (L423, R15): key_k = p_k / E_k; we set p0 / p1 = (1 +/- eps) E0 / E1 and expect the
    winner 0 / 1 with margin eps.
A margin formula with a dropped factor (q instead of r q), an absolute instead of relative gap, or
the wrong pair in the race fails these by orders of magnitude.
"""
import numpy as np
import pytest

import oracle
from tests.mss_compare import compare_sampled, first_divergent_decision

SEED = 0x1234_5678_9ABC
OFF = 3


def _words(rid, w1, w2):
    return [int(x) for x in oracle.philox4x32_10([rid, w1, w2, OFF], [SEED & 0xFFFFFFFF, SEED >> 32])]


def _softmax64(logits):
    x = np.asarray(logits, np.float64)
    e = np.exp(x - x.max())
    return e / e.sum()


@pytest.mark.parametrize("eps", [1e-3, 1e-4, 3e-5])
@pytest.mark.parametrize("side", [-1, +1])
def test_accept_margin_near_tie(eps, side):
    """Root with one child carrying token 0 (V = 2).  r = (w1 >> 8) 2^-24 from the round-0 counter
    of node 0; q[0] is chosen so that r q[0] = p[0] (1 + side eps): side -1 accepts, +1 rejects,
    and the reported margin is eps (relative to max(p, r q))."""
    # pick a request id whose round-0 uniform r is large enough that q[0] = p0 (1 +/- eps) / r <= 1
    for rid in range(1000):
        w = _words(rid, 0 << 8, 0)
        r = (w[1] >> 8) * 2.0 ** -24
        if r > 0.5:
            break
    logits = np.array([[[0.0, np.log(3.0)], [0.0, 0.0]]], np.float32)   # p = (1/4, 3/4)
    p0 = _softmax64(logits[0, 0])[0]
    q0 = np.float32(p0 * (1 + side * eps) / r)
    draft = np.zeros((1, 2, 2), np.float32)
    draft[0, 1] = [q0, 1 - q0]
    toks = np.array([[0, 0]], np.int32)
    par = np.array([[-1, 0]], np.int32)
    res = oracle.verify_mss(logits, toks, par, np.array([2], np.int32), draft, seed=SEED, offset=OFF,
                            request_ids=np.array([rid], np.int32))
    dec = res.decisions[0]
    assert dec[0][:2] == (0, 1)
    accepted = dec[0][2] == 1
    assert accepted == (side < 0)
    rq = r * float(q0)
    # the exact gap of the constructed (fp32-rounded) inputs, and the construction's eps
    assert dec[0][3] == pytest.approx(abs(p0 - rq) / max(p0, rq), rel=1e-9)
    assert dec[0][3] == pytest.approx(eps / (1 + eps) if side > 0 else eps, rel=1e-2)
    assert res[3][0] <= dec[0][3]   # the per-request minimum covers it


@pytest.mark.parametrize("eps", [1e-3, 1e-4])
@pytest.mark.parametrize("side", [-1, +1])
def test_race_margin_near_tie(eps, side):
    """Root-only tree (a leaf: the final sample is the race at round 0, V = 2).  E_k = -ln U_k with
    U_k = ((w_k >> 9) + 0.5) 2^-23, w_k = word k of Philox(rid, 0, 2 << 28, offset).  With
    p0 / p1 = (1 + side eps) E0 / E1 the keys p_k / E_k differ by the factor (1 + side eps): the
    winner is 0 for side +1 and 1 for side -1, the margin eps / (1 + eps) resp. eps."""
    rid = 7
    w = _words(rid, 0, 2 << 28)
    E = [-np.log(((w[k] >> 9) + 0.5) * 2.0 ** -23) for k in (0, 1)]
    ratio = (1 + side * eps) * E[0] / E[1]
    logits = np.array([[[np.log(ratio), 0.0]]], np.float32)
    res = oracle.verify_mss(logits, np.zeros((1, 1), np.int32), np.array([[-1]], np.int32),
                            np.array([1], np.int32), np.zeros((1, 1, 2), np.float32), seed=SEED, offset=OFF,
                            request_ids=np.array([rid], np.int32))
    dec = res.decisions[0]
    assert len(dec) == 1 and dec[0][:2] == (0, -1)
    assert dec[0][2] == (0 if side > 0 else 1) == res[1][0, 0]
    expect = eps / (1 + eps) if side > 0 else eps
    assert dec[0][3] == pytest.approx(expect, rel=2e-3)
    # naive sampling draws the same race at a leaf (R25): same record
    ns = oracle.verify_ns(logits, np.zeros((1, 1), np.int32), np.array([[-1]], np.int32), np.array([1], np.int32),
                          seed=SEED, offset=OFF, request_ids=np.array([rid], np.int32))
    assert ns.decisions[0][0][:3] == dec[0][:3]
    assert ns.decisions[0][0][3] == pytest.approx(dec[0][3], rel=1e-12)


def test_decision_log_follows_the_pick_order():
    """Disjoint supports (p[x] = 0 for every drafted token): every child of the root is rejected
    (margin INFINITY: the p[x] > 0 guard decides, not a float comparison), in the order the integer
    pick s = H[((w0 >> 8) |H|) >> 24] over the remaining children gives (R9), then one race."""
    V = 4
    par = np.array([[-1, 0, 0, 0, 0]], np.int32)
    toks = np.array([[0, 2, 3, 2, 3]], np.int32)
    logits = np.full((1, 5, V), -1e30, np.float32)
    logits[0, :, :2] = 0.0                      # p = (1/2, 1/2, 0, 0)
    draft = np.zeros((1, 5, V), np.float32)
    draft[0, 1:, 2:] = 0.5                      # q = (0, 0, 1/2, 1/2)
    rid = 11
    res = oracle.verify_mss(logits, toks, par, np.array([5], np.int32), draft, seed=SEED, offset=OFF,
                            request_ids=np.array([rid], np.int32))
    H, order = [1, 2, 3, 4], []
    for rnd in range(4):
        w = _words(rid, (0 << 8) | rnd, 0)
        s = H[((w[0] >> 8) * len(H)) >> 24]
        order.append(s)
        H.remove(s)
    dec = res.decisions[0]
    assert [d[1] for d in dec[:4]] == order
    assert all(d[0] == 0 and d[2] == 0 and d[3] == np.inf for d in dec[:4])
    assert dec[4][:2] == (0, -1) and dec[4][2] in (0, 1) and res[2][0] == 1


# ------------------------------------------------------------------------------------------------
# host logic of the comparison (tests/mss_compare.py) on constructed logs
# ------------------------------------------------------------------------------------------------
# a log for: node 0 tests child 3 (reject), child 1 (accept); node 1 tests child 2 (reject); race at 1
LOG = [(0, 3, 0, 0.5), (0, 1, 1, 2e-6), (1, 2, 0, 0.3), (1, -1, 17, 0.2)]
O_NODES, O_TOKS = [0, 1], [5, 17]


def test_first_divergence_cases():
    assert first_divergent_decision(O_NODES, O_TOKS, O_NODES, O_TOKS, LOG) is None
    # same path, different bonus token: the race at node 1
    assert first_divergent_decision([0, 1], [5, 18], O_NODES, O_TOKS, LOG) == 3
    # GPU accepted child 3 at the root, which the oracle rejected first: decision 0
    assert first_divergent_decision([0, 3], [9, 4], O_NODES, O_TOKS, LOG) == 0
    # GPU rejected child 1 (oracle accepted it) and raced at the root: decision 1
    assert first_divergent_decision([0], [6], O_NODES, O_TOKS, LOG) == 1
    # GPU went on from node 1 to child 2 (oracle rejected it): decision 2
    assert first_divergent_decision([0, 1, 2], [5, 8, 1], O_NODES, O_TOKS, LOG) == 2


def test_compare_sampled_excuses_only_near_ties():
    ref = oracle.VerifyResult((np.array([[0, 1, -1]]), np.array([[5, 17, -1]]), np.array([2]), np.array([2e-6])))
    ref.decisions = [LOG]
    # divergence at decision 1 (margin 2e-6 < 1e-5): excused, but the cap is int(1e-4 * 1) = 0
    with pytest.raises(AssertionError, match="boundary-excused"):
        compare_sampled((np.array([[0, -1, -1]]), np.array([[6, -1, -1]]), np.array([1])), ref)
    assert compare_sampled((np.array([[0, -1, -1]]), np.array([[6, -1, -1]]), np.array([1])), ref,
                           fraction=1.0)[0][0] == 0
    # divergence at decision 0 (margin 0.5): never excused, although the request's minimum is 2e-6
    with pytest.raises(AssertionError, match="not excused"):
        compare_sampled((np.array([[0, 3, -1]]), np.array([[9, 4, -1]]), np.array([2])), ref, fraction=1.0)
    # identical: nothing to excuse
    assert compare_sampled((ref[0], ref[1], ref[2]), ref) == []
