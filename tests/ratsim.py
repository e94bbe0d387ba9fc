"""Exact-rational re-simulation of an explicit task graph (test pin for the oracle).

An independent, deliberately naive implementation of the timeline semantics
(R12-R17: BFS routing, latency-first flows, max-min progressive
filling, instant fixed point) over ``fractions.Fraction``.  It consumes the task
graph the C oracle exports (oracle.export_graph) or a hand/random-built graph in
the same layout, so it pins the oracle's discrete-event engine and network model
without sharing any of its code.  Only for tiny graphs (it is O(n^2) per instant).
"""
from __future__ import annotations

from collections import deque
from fractions import Fraction as Fr

TASK, FLOW, BARRIER = 0, 1, 2


def bfs_route(n_nodes, links, src, dst):
    """Shortest path by hops; among equals the lexicographically smallest node sequence.
    Implemented as a full search of all shortest paths (different algorithm from the oracle's)."""
    if src == dst:
        return []
    out = {}
    for e, (a, b, _, _) in enumerate(links):
        out.setdefault(a, []).append((b, e))
    dist = {src: 0}
    q = deque([src])
    while q:
        u = q.popleft()
        for v, _ in out.get(u, []):
            if v not in dist:
                dist[v] = dist[u] + 1
                q.append(v)
    if dst not in dist:
        return None
    best = None

    def dfs(u, path_nodes, path_links):
        nonlocal best
        if u == dst:
            cand = (list(path_nodes), list(path_links))
            if best is None or cand[0] < best[0]:
                best = cand
            return
        for v, e in out.get(u, []):
            if dist.get(v) == dist[u] + 1 and dist[v] <= dist[dst]:
                path_nodes.append(v)
                path_links.append(e)
                dfs(v, path_nodes, path_links)
                path_nodes.pop()
                path_links.pop()
    dfs(src, [src], [])
    return best[1]


def progressive_fill(bw, routes):
    """Exact max-min fair rates for flows with given routes (link ids) and link capacities."""
    rate = [None] * len(routes)
    res = {e: Fr(b) for e, b in enumerate(bw)}
    unfrozen = set(range(len(routes)))
    rounds = 0
    while unfrozen:
        cnt = {}
        for f in unfrozen:
            for e in routes[f]:
                cnt[e] = cnt.get(e, 0) + 1
        share = {e: res[e] / c for e, c in cnt.items()}
        s = min(share.values())
        fr = [f for f in unfrozen if any(share[e] == s for e in routes[f])]
        for f in fr:
            rate[f] = s
            for e in routes[f]:
                res[e] -= s
        unfrozen -= set(fr)
        rounds += 1
    return rate, rounds


def simulate(g, n_nodes, links, bw_scale=1, lat_scale=1):
    """links: list of (src, dst, bw, lat).  Returns (T, done_time per node, stats)."""
    n = len(g["type"])
    typ = [int(x) for x in g["type"]]
    deps = [[int(d) for d in g["dep_ids"][g["dep_off"][i]:g["dep_off"][i + 1]]] for i in range(n)]
    dependents = [[] for _ in range(n)]
    for i in range(n):
        for d in deps[i]:
            dependents[d].append(i)
    bw = [Fr(l[2]) * Fr(bw_scale) for l in links]
    lat = [Fr(l[3]) * Fr(lat_scale) for l in links]
    route, L = {}, {}
    for i in range(n):
        if typ[i] == FLOW:
            r = bfs_route(n_nodes, links, int(g["src"][i]), int(g["dst"][i]))
            if r is None:
                raise ValueError("no route")
            route[i] = r
            L[i] = sum((lat[e] for e in r), Fr(0))
    queues = {}
    for i in range(n):
        if typ[i] == TASK:
            queues.setdefault(int(g["gpu"][i]), []).append(i)
    head = {q: 0 for q in queues}
    running = {q: None for q in queues}
    done = [None] * n
    # a barrier whose flags carry need + 1 in bits 8.. completes once `need` dependencies are done (R28)
    ndeps = [(int(g["flags"][i]) >> 8) - 1 if typ[i] == BARRIER and (int(g["flags"][i]) >> 8) > 0 else len(deps[i])
             for i in range(n)]
    released = set()
    end, tact, rem, rate, tupd, tdrain = {}, {}, {}, {}, {}, {}
    latent, active = set(), set()
    t = Fr(0)
    stats = dict(wf_calls=0, rounds=0, max_active=0)

    def complete(i):
        done[i] = t
        for d in dependents[i]:
            ndeps[d] -= 1

    while True:
        again = True
        dirty = False
        while again:
            changed = True
            while changed:
                changed = False
                for q in queues:
                    k = running[q]
                    if k is not None and end[k] == t:
                        complete(k)
                        running[q] = None
                        changed = True
                for f in list(active):
                    if tdrain[f] == t:
                        active.discard(f)
                        complete(f)
                        dirty = changed = True
                for f in list(latent):
                    if tact[f] == t:
                        latent.discard(f)
                        if Fr(g["bytes"][f]) == 0 or not route[f]:
                            complete(f)
                        else:
                            active.add(f)
                            rem[f] = Fr(g["bytes"][f])
                            tupd[f] = t
                            rate[f] = Fr(0)
                            tdrain[f] = None
                            dirty = True
                        changed = True
                for i in range(n):
                    if typ[i] != TASK and done[i] is None and i not in released and ndeps[i] <= 0:
                        if typ[i] == BARRIER:
                            complete(i)
                        else:
                            released.add(i)
                            tact[i] = t + L[i]
                            latent.add(i)
                        changed = True
                for q in queues:
                    if running[q] is None and head[q] < len(queues[q]):
                        k = queues[q][head[q]]
                        if ndeps[k] <= 0:
                            running[q] = k
                            head[q] += 1
                            end[k] = t + Fr(g["dur"][k])
                            changed = True
            again = False
            if dirty:
                dirty = False
                fl = sorted(active)
                for f in fl:
                    if tupd[f] < t:
                        rem[f] = max(Fr(0), rem[f] - rate[f] * (t - tupd[f]))
                        tupd[f] = t
                rates, rounds = progressive_fill(bw, [route[f] for f in fl])
                stats["wf_calls"] += 1
                stats["rounds"] += rounds
                stats["max_active"] = max(stats["max_active"], len(fl))
                for f, r in zip(fl, rates):
                    rate[f] = r
                    tdrain[f] = t + rem[f] / r
                    if tdrain[f] == t:
                        again = True
        if all(d is not None for d in done):
            return t, done, stats
        cands = [end[running[q]] for q in queues if running[q] is not None]
        cands += [tact[f] for f in latent] + [tdrain[f] for f in active]
        if not cands:
            raise RuntimeError("deadlock")
        t = min(cands)
