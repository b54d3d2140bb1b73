"""GPU-vs-oracle comparison of the sampling verifiers (MSS, c4; naive sampling, NEXT-3).

SURVEY §8(c) c4: both sides draw the same Philox uniforms and take integer picks, so the GPU (fp32)
and the oracle (fp64) can only disagree at a decision whose outcome sits within rounding of its
boundary.  A mismatch is *boundary-excused* only when the FIRST decision at which the two paths
diverge has a relative margin below 1e-5 in the oracle's decision log; at most 1e-4 of the compared
requests may be excused, and every excused request is printed.  Everything else is bit-exact.

The oracle's log (``oracle.verify_mss(...).decisions``) lists, per request, the records
(node u, child s or -1 for the final race, value, margin) in the order Alg. 2 (L403-425) takes them.
This module is host logic only (no GPU); ``tests/test_mss_compare.py`` checks it on constructed logs.
"""
from __future__ import annotations

import numpy as np

EXCUSE_MARGIN = 1e-5
EXCUSE_FRACTION = 1e-4


def first_divergent_decision(g_nodes, g_tokens, o_nodes, o_tokens, decisions):
    """Index into ``decisions`` (the oracle's log of one request) of the first decision at which the
    GPU path (g_nodes/g_tokens, trimmed to n_accepted) and the oracle path diverge; None when they
    are identical.

    Both sides walk the same nodes while they agree, and at a node they test the children in the
    same order (the pick is integer arithmetic on the same counters).  At the first node u where
    they part, the candidates are: the oracle's test of the child the GPU accepted (the oracle
    rejected it, or never reached it because it accepted an earlier child), the oracle's test of the
    child the oracle accepted (the GPU rejected it), and, when both raced at u, the race itself.
    The earliest candidate in the oracle's order is the first differing decision."""
    g_nodes, o_nodes = list(g_nodes), list(o_nodes)
    if g_nodes == o_nodes and list(g_tokens) == list(o_tokens):
        return None
    k = 1
    while k < len(g_nodes) and k < len(o_nodes) and g_nodes[k] == o_nodes[k]:
        k += 1
    u = o_nodes[k - 1]
    g_next = g_nodes[k] if k < len(g_nodes) else None
    o_next = o_nodes[k] if k < len(o_nodes) else None
    at_u = [i for i, d in enumerate(decisions) if d[0] == u]
    if not at_u:
        raise AssertionError(f"oracle log has no decision at node {u}")
    if g_next is None and o_next is None:
        races = [i for i in at_u if decisions[i][1] == -1]
        if not races:
            raise AssertionError(f"oracle log has no race at node {u}")
        return races[0]
    cands = []
    for child in (g_next, o_next):
        if child is None:
            continue
        tests = [i for i in at_u if decisions[i][1] == child]
        if tests:
            cands.append(tests[0])
    if not cands:
        # the GPU accepted a child the oracle never tested: the oracle accepted an earlier child,
        # whose test is the divergence (covered above), so this cannot happen on a consistent log
        raise AssertionError(f"no candidate decision at node {u}: gpu {g_next} oracle {o_next}")
    return min(cands)


def compare_sampled(got, ref, *, label="", excuse=EXCUSE_MARGIN, fraction=EXCUSE_FRACTION):
    """got = (accepted_nodes, accepted_tokens, n_accepted) from the GPU (tensors or arrays); ref =
    the oracle's VerifyResult.  Asserts bit-exactness up to boundary-excused requests and returns the
    list of excused (request, margin, record)."""
    an, at, na = [x.cpu().numpy() if hasattr(x, "cpu") else np.asarray(x) for x in got]
    r_an, r_at, r_na = ref[0], ref[1], ref[2]
    B = len(na)
    excused, unexcused = [], []
    for b in range(B):
        if na[b] == r_na[b] and np.array_equal(an[b], r_an[b]) and np.array_equal(at[b], r_at[b]):
            continue
        if na[b] <= 0 or r_na[b] <= 0:
            unexcused.append((b, None, "an invalid-tree / empty result on one side only"))
            continue
        n, rn = int(na[b]), int(r_na[b])
        i = first_divergent_decision(an[b][:n], at[b][:n], r_an[b][:rn], r_at[b][:rn], ref.decisions[b])
        if i is None:  # equal paths but different padding: not a decision difference
            unexcused.append((b, None, "padding differs"))
            continue
        rec = ref.decisions[b][i]
        (excused if rec[3] < excuse else unexcused).append((b, rec[3], rec))
    for b, m, rec in excused:
        print(f"[mss-compare {label}] request {b} boundary-excused: first divergent decision {rec} "
              f"(relative margin {m:.3e} < {excuse:g})")
    assert not unexcused, f"{label}: sampled-verify mismatches not excused by the margin rule: {unexcused[:10]}"
    cap = int(fraction * B)
    assert len(excused) <= cap, f"{label}: {len(excused)} boundary-excused requests of {B} (cap {cap})"
    return excused
