"""Oracle pins for routing, the bandwidth allocation and the
PP auto-partition, by brute force and by the max-min fairness invariants."""
import itertools
from fractions import Fraction as Fr

import numpy as np
import pytest

import oracle
from paper_conf_isca_libwmvgjbj025_b200 import workloads as W
from tests import ratsim


# ---------------- routing: exhaustive enumeration (CF15) ----------------
def all_simple_paths(n, adj, s, d):
    out = []

    def dfs(u, nodes, links):
        if u == d:
            out.append((list(nodes), list(links)))
            return
        for v, e in adj.get(u, []):
            if v not in nodes:
                nodes.append(v)
                links.append(e)
                dfs(v, nodes, links)
                nodes.pop()
                links.pop()
    dfs(s, [s], [])
    return out


@pytest.mark.parametrize("seed", range(40))
def test_route_is_lexicographically_smallest_shortest_path(seed):
    rng = np.random.Generator(np.random.PCG64(seed))
    n = int(rng.integers(2, 8))
    pairs = [(a, b) for a in range(n) for b in range(n) if a != b and rng.random() < 0.35]
    if not pairs:
        pairs = [(0, 1)]
    links = np.zeros(len(pairs), W.LINK_DTYPE)
    for i, (a, b) in enumerate(pairs):
        links[i] = (a, b, 1.0, 0.0)
    topo = W.Topology("r", n, n, links, np.arange(n, dtype=np.uint32))
    adj = {}
    for e, (a, b) in enumerate(pairs):
        adj.setdefault(a, []).append((b, e))
    for s in range(n):
        for d in range(n):
            got = oracle.route(topo, s, d)
            if s == d:
                assert got == []
                continue
            paths = all_simple_paths(n, adj, s, d)
            if not paths:
                assert got is None
                continue
            h = min(len(p[1]) for p in paths)
            best = min(p for p in paths if len(p[1]) == h)
            assert got == best[1], (s, d)


# ---------------- water-filling: invariants + exact rational (CF16) ----------------
def random_wf(rng, dyadic=False):
    nl = int(rng.integers(1, 7))
    nf = int(rng.integers(1, 9))
    if dyadic:
        bw = [float(2 ** int(rng.integers(0, 5))) for _ in range(nl)]
    else:
        bw = [float(rng.uniform(0.1, 10.0)) for _ in range(nl)]
    routes = []
    for _ in range(nf):
        h = int(rng.integers(1, min(3, nl) + 1))
        routes.append([int(x) for x in rng.choice(nl, h, replace=False)])
    return bw, routes


@pytest.mark.parametrize("seed", range(300))
def test_waterfill_maxmin_invariants_and_exact(seed):
    rng = np.random.Generator(np.random.PCG64(seed))
    bw, routes = random_wf(rng, dyadic=seed % 3 == 0)
    rate, rounds = oracle.waterfill(bw, routes)
    # capacity
    load = [0.0] * len(bw)
    for f, r in enumerate(routes):
        for e in r:
            load[e] += rate[f]
    for e in range(len(bw)):
        assert load[e] <= bw[e] * (1 + 1e-12)
    # every flow has a saturated bottleneck on which its rate is maximal (max-min fairness)
    for f, r in enumerate(routes):
        ok = False
        for e in r:
            sat = load[e] >= bw[e] * (1 - 1e-12)
            mx = max(rate[g] for g, rg in enumerate(routes) if e in rg)
            if sat and rate[f] >= mx * (1 - 1e-12):
                ok = True
        assert ok, (f, r)
    # exact-rational progressive filling
    er, erounds = ratsim.progressive_fill([Fr(b) for b in bw], routes)
    for f in range(len(routes)):
        assert abs(rate[f] - float(er[f])) <= 2e-16 * float(er[f]) * 8
    if all(Fr(float(x)) == x and (x.denominator & (x.denominator - 1)) == 0 for x in er) and \
            all((len(r) == 1) for r in routes):
        # single-hop flows with dyadic shares: every intermediate value is exact in fp64
        assert [Fr(x) for x in rate] == er and rounds == erounds
    # order independence: permuting the flows permutes the rates bitwise
    perm = rng.permutation(len(routes))
    rate2, rounds2 = oracle.waterfill(bw, [routes[i] for i in perm])
    assert rounds2 == rounds
    assert all(rate2[q] == rate[perm[q]] for q in range(len(routes)))
    # scaling: bw * 2^k -> rates * 2^k bitwise
    rate3, _ = oracle.waterfill([b * 8.0 for b in bw], routes)
    assert all(rate3[f] == rate[f] * 8.0 for f in range(len(routes)))


def test_waterfill_textbook_example():
    """Two links of capacity 1; flow A crosses both, B only link 0, C only link 1:
    fair share 1/2 each (single bottleneck level).  Then a 3-level instance."""
    rate, rounds = oracle.waterfill([1.0, 1.0], [[0, 1], [0], [1]])
    assert list(rate) == [0.5, 0.5, 0.5] and rounds == 1
    # link0 cap 1 shared by A,B; link1 cap 10 shared by A,C -> A=B=0.5, C=9.5
    rate, rounds = oracle.waterfill([1.0, 10.0], [[0, 1], [0], [1]])
    assert list(rate) == [0.5, 0.5, 9.5] and rounds == 2


# ---------------- PP auto-partition: exhaustive enumeration ----------------
@pytest.mark.parametrize("seed", range(12))
def test_partition_matches_exhaustive_search(seed):
    rng = np.random.Generator(np.random.PCG64(100 + seed))
    tr = W.random_trace(rng, n_layers=int(rng.integers(2, 8)), max_ops_per_layer=3)
    if seed % 2:  # force ties
        tr.ops["time_s"] = 2.0 ** -10 * rng.integers(1, 3, len(tr.ops))
    L = tr.n_layers
    lc = [0.0] * L
    for op in tr.ops:
        lc[op["layer"]] = lc[op["layer"]] + op["time_s"]
    for S in range(1, L + 1):
        best = None
        for cuts in itertools.combinations(range(1, L), S - 1):
            b = (0,) + cuts + (L,)
            worst = 0.0
            for s in range(S):
                c = 0.0
                for l in range(b[s], b[s + 1]):
                    c = c + lc[l]
                worst = max(worst, c)
            key = (worst, (0,) + cuts)
            if best is None or key < best:
                best = key
        assert tuple(oracle.partition(tr, S)) == best[1], (S, L)
