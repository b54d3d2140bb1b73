"""GPU parity of NEXT-2 token-tree construction (§3) against the
oracle: expansion topology, expansion steps (top-k tokens bit-exact, draft rows = softmax of the
parent's SSM logits to 1e-6), the full Fig. 3 example, and token tree merge (bit-exact,
including the Fig. 2 example and invalid inputs)."""
import numpy as np
import pytest
import torch

import oracle
import workloads as W
from tests.test_gpu_parity import DEV

pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    import paper_conf_asplos_miaoozcwzwzyssc24_b200 as spi


def _topology(expansion, B, Nmax=None, V=16):
    n = 1 + sum(int(np.prod(expansion[:i + 1])) for i in range(len(expansion)))
    Nmax = Nmax or n
    shape = spi.make_shape(B, Nmax, 1, 1, Nmax, vocab=V, max_depth=max(len(expansion), 1))
    par = torch.empty((B, Nmax), dtype=torch.int32, device=DEV)
    dep = torch.empty_like(par)
    nn = torch.empty((B,), dtype=torch.int32, device=DEV)
    spi.specinfer_expansion_topology(shape, list(expansion), par, dep, nn)
    return shape, par, dep, nn, n


@pytest.mark.parametrize("expansion", [(), (2, 2, 1), (1, 1, 3, 1, 1, 1, 1, 1), (8, 4, 1, 1, 1, 1, 1, 1),
                                       (1, 2, 2, 2, 2, 2, 2)])
def test_expansion_topology(expansion):
    shape, par, dep, nn, n = _topology(expansion, 3, V=8)
    bpar, bdep = oracle.expansion_tree_bfs(list(expansion))
    dpar, _, order = oracle.dfs_linearize(bpar)
    assert nn.tolist() == [n] * 3
    for b in range(3):
        assert par[b].tolist() == dpar
        assert dep[b].tolist() == [bdep[o] for o in order]


def _oracle_expand(ssm_rows, par_dfs, dep_dfs, level):
    """tokens the oracle's top-k gives the children of each depth-`level` node (DFS order)."""
    out = {}
    frontier = [u for u in range(len(par_dfs)) if dep_dfs[u] == level]
    for f, u in enumerate(frontier):
        kids = [c for c in range(len(par_dfs)) if par_dfs[c] == u]
        for c, t in zip(kids, oracle.expand_topk(ssm_rows[f], len(kids))):
            out[c] = t
    return out


@pytest.mark.parametrize("expansion,V", [((2, 2, 1), 50), ((8, 4, 1), 50272), ((1, 1, 3, 1), 32000), ((3, 2), 7)])
def test_expand_steps_parity(expansion, V):
    B = 4
    shape, par, dep, nn, n = _topology(expansion, B, V=V)
    toks = torch.full((B, n), -1, dtype=torch.int32, device=DEV)
    toks[:, 0] = 1
    draft = torch.zeros((B, n, V), dtype=torch.float32, device=DEV)
    g = torch.Generator(device=DEV).manual_seed(V)
    pd, dd = par[0].tolist(), dep[0].tolist()
    expect = {}
    qrows = {}
    for level in range(len(expansion)):
        F = sum(1 for u in range(n) if dd[u] == level)
        lg = torch.randint(-4, 4, (B, F, V), generator=g, device=DEV).float() * 0.5   # ties
        spi.specinfer_expand_step(shape, level, lg, 0.8, par, dep, nn, toks, draft)
        frontier = [u for u in range(n) if dd[u] == level]
        for b in range(B):
            rows = lg[b].cpu().numpy()
            for c, t in _oracle_expand(rows, pd, dd, level).items():
                expect[(b, c)] = t
                f = frontier.index(pd[c])
                qrows[(b, c)] = oracle.ssm_distribution(rows[f], 0.8)
    torch.cuda.synchronize()
    got = toks.cpu().numpy()
    dr = draft.cpu().numpy()
    for (b, c), t in expect.items():
        assert got[b, c] == t, (b, c)
        np.testing.assert_allclose(dr[b, c], qrows[(b, c)], rtol=1e-5, atol=1e-7)


def test_fig3_expansion_on_gpu(golden):
    g = golden("fig3_expansion.json")
    steps = g["tokens_by_step"]
    vocab = sorted({w for s in g["sequences"] for w in s})
    ids = {w: i for i, w in enumerate(vocab)}
    V = len(vocab)
    shape, par, dep, nn, n = _topology(g["expansion"], 1, V=V)
    toks = torch.full((1, n), -1, dtype=torch.int32, device=DEV)
    toks[0, 0] = ids[steps["root"]]
    pd, dd = par[0].tolist(), dep[0].tolist()
    for level in range(len(g["expansion"])):
        frontier = [u for u in range(n) if dd[u] == level]
        lg = torch.full((1, len(frontier), V), -10.0, device=DEV)
        tk = toks[0].tolist()
        for f, u in enumerate(frontier):
            # the SSM ranks the figure's tokens for this node first, in order
            for r, w in enumerate(steps[str(level)][vocab[tk[u]]]):
                lg[0, f, ids[w]] = 10.0 - r
        spi.specinfer_expand_step(shape, level, lg, 1.0, par, dep, nn, toks)
        torch.cuda.synchronize()
    tk = toks[0].tolist()
    seqs = []
    for p in oracle.leaf_paths(par.cpu().numpy(), nn.cpu().numpy())[0]:
        seqs.append([vocab[tk[u]] for u in p])
    assert sorted(map(tuple, seqs)) == sorted(map(tuple, g["sequences"]))
    assert pd == g["dfs_parent"]


def _merge_gpu(trees_per_req, Nmax, Dmax=16):
    B = len(trees_per_req)
    T = max(len(t) for t in trees_per_req)
    Nin = max(len(p) for ts in trees_per_req for p, _ in ts)
    ip = torch.full((B, T, Nin), -1, dtype=torch.int32)
    it = torch.zeros((B, T, Nin), dtype=torch.int32)
    inn = torch.zeros((B, T), dtype=torch.int32)
    for b, ts in enumerate(trees_per_req):
        for t, (p, k) in enumerate(ts):
            ip[b, t, :len(p)] = torch.tensor(p)
            it[b, t, :len(k)] = torch.tensor(k)
            inn[b, t] = len(p)
    shape = spi.make_shape(B, Nmax, 1, 1, Nmax, max_depth=Dmax)
    outs = [torch.empty((B, Nmax), dtype=torch.int32, device=DEV) for _ in range(3)]
    nn = torch.empty((B,), dtype=torch.int32, device=DEV)
    nmap = torch.empty((B, T, Nin), dtype=torch.int32, device=DEV)
    ws = spi.alloc_workspace(shape, DEV)
    ws.zero_()
    spi.specinfer_tree_merge(shape, ip.to(DEV), it.to(DEV), inn.to(DEV), *outs, nn, nmap, ws)
    bits = spi.specinfer_read_device_status(ws)
    return [o.cpu().numpy() for o in outs], nn.cpu().numpy(), nmap.cpu().numpy(), bits


def test_tree_merge_parity_and_fig2(golden):
    g = golden("fig2_merge.json")
    vocab = sorted({w for s in g["inputs"] for w in s})
    ids = {w: i for i, w in enumerate(vocab)}
    fig2 = [(list(range(-1, len(s) - 1)), [ids[w] for w in s]) for s in g["inputs"]]
    rng = np.random.default_rng(4)
    reqs = [fig2]
    for _ in range(30):
        ts = []
        for _ in range(int(rng.integers(1, 6))):
            n = int(rng.integers(1, 20))
            par, _ = W.random_tree(n, 7, 3, rng)
            tok = rng.integers(0, 4, n).astype(int)
            tok[0] = 9
            ts.append((list(par), list(tok)))
        reqs.append(ts)
    (par, dep, tok), nn, nmap, bits = _merge_gpu(reqs, 128)
    assert bits == 0
    assert [vocab[t] for t in tok[0, :nn[0]]] == g["merged_tokens"]
    assert list(par[0, :nn[0]]) == g["merged_parent"]
    for b, ts in enumerate(reqs):
        rp, rt, rd, rmaps = oracle.tree_merge(ts)
        assert nn[b] == len(rp)
        assert list(par[b, :nn[b]]) == rp and list(tok[b, :nn[b]]) == rt and list(dep[b, :nn[b]]) == rd
        for t, m in enumerate(rmaps):
            assert list(nmap[b, t, :len(m)]) == m


def test_tree_merge_invalid():
    reqs = [[([-1], [1]), ([-1, 0], [2, 3])],          # roots differ
            [([-1, 0, 0], [1, 2, 3])],                    # fine
            [([-1, 0, 0, 1, 2, 3], [1, 2, 3, 4, 5, 6])]]  # 6 nodes > Nmax 5
    (par, dep, tok), nn, nmap, bits = _merge_gpu(reqs, 5)
    assert nn.tolist() == [0, 3, 0] and bits & 1
    assert (nmap[0] == -1).all() and (nmap[2] == -1).all()


def test_tree_merge_depth_beyond_dmax():
    """A merged tree deeper than Dmax is reported like every other bad input (header contract):
    n_nodes 0, node_map -1, padding rows (parent -1, depth 0, token -1), BAD_TREE; other requests of
    the batch are unaffected."""
    reqs = [[([-1, 0, 1, 2], [1, 2, 3, 4])],              # depth 3 > Dmax 2
            [([-1, 0, 1], [1, 2, 3]), ([-1, 0], [1, 5])]]  # depth 2: fine
    (par, dep, tok), nn, nmap, bits = _merge_gpu(reqs, 8, Dmax=2)
    assert nn.tolist() == [0, 4] and bits & 1
    assert (nmap[0] == -1).all()
    assert (par[0] == -1).all() and (dep[0] == 0).all() and (tok[0] == -1).all()
    rp, rt, rd, _ = oracle.tree_merge(reqs[1])
    assert list(par[1, :4]) == rp and list(tok[1, :4]) == rt and list(dep[1, :4]) == rd
