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
