"""Brute force over all injective vertex maps — an independent pin for the oracle.

Used only on tiny graphs (n <= 10, k <= 5).  It enumerates every injective
k-tuple of data vertices and keeps those that map every query edge onto a data
edge (the plain definition of Emb(Q, D), Def. 2-4, read as
non-induced per reading P1).  It knows nothing about orders, candidate lists,
intersections or tries.
"""
from itertools import permutations


def adjacency_sets(g):
    return [set(int(x) for x in g.neighbors(v)) for v in range(g.n)]


def embeddings(g, q):
    adj = adjacency_sets(g)
    out = []
    for f in permutations(range(g.n), q.k):
        if all(f[v] in adj[f[u]] for u, v in q.edges):
            out.append(tuple(f))
    return sorted(out)


def level_sizes(g, q, order):
    """|L_j| for j = 0..k: injective maps of order[0..j-1] that preserve the
    query edges among those positions and satisfy deg(f(S[i])) >= deg_Q(S[i])."""
    adj = adjacency_sets(g)
    qd = q.degrees()
    qe = {(u, v) for u, v in q.edges} | {(v, u) for u, v in q.edges}
    sizes = [0]
    for j in range(1, q.k + 1):
        pos = order[:j]
        cnt = 0
        for f in permutations(range(g.n), j):
            if any(len(adj[f[i]]) < qd[pos[i]] for i in range(j)):
                continue
            ok = True
            for a in range(j):
                for b in range(a + 1, j):
                    if (pos[a], pos[b]) in qe and f[b] not in adj[f[a]]:
                        ok = False
                        break
                if not ok:
                    break
            cnt += ok
        sizes.append(cnt)
    return sizes


# ------------------------------------------------------------------- directed
def di_embeddings(g, q):
    """Injective maps f with (u, v) in arcs(Q) => (f(u), f(v)) in arcs(D)."""
    arcs = {(int(a), int(b)) for a, b in g.arcs()}
    return sorted(f for f in permutations(range(g.n), q.k) if all((f[u], f[v]) in arcs for u, v in q.arcs))


def di_level_sizes(g, q, order):
    """|L_j| for the directed trie: injective maps of order[0..j-1] preserving
    the arcs among those positions with outdeg/indeg >= the query's."""
    arcs = {(int(a), int(b)) for a, b in g.arcs()}
    od, idg = g.out_degrees(), g.in_degrees()
    qo = [sum(1 for u, _ in q.arcs if u == a) for a in range(q.k)]
    qi = [sum(1 for _, v in q.arcs if v == a) for a in range(q.k)]
    sizes = [0]
    for j in range(1, q.k + 1):
        pos = order[:j]
        ix = {p: i for i, p in enumerate(pos)}
        inner = [(ix[u], ix[v]) for u, v in q.arcs if u in ix and v in ix]
        cnt = 0
        for f in permutations(range(g.n), j):
            if any(od[f[i]] < qo[pos[i]] or idg[f[i]] < qi[pos[i]] for i in range(j)):
                continue
            cnt += all((f[a], f[b]) in arcs for a, b in inner)
        sizes.append(cnt)
    return sizes
