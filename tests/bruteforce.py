"""Brute-force betweenness by explicit path enumeration (pin for the oracle).

No BFS, no path-count recursion, no dependency recursion: for every ordered
pair (s, t) enumerate ALL simple s-t paths by depth-first search, keep the ones
of minimum length, and count directly
    sigma_st     = number of shortest s-t paths
    sigma_st(v)  = number of those that pass through v (interior)
Then Eq. (1) restricted to sources in R gives
    BC(v) = sum_{s in R, s != v} sum_{t != s, v} sigma_st(v) / sigma_st
and the dependency of v on s is the inner sum (Brandes' pair dependencies,
whose recursion is Eq. (2)).  Exponential: n <= 9 only.
"""

from __future__ import annotations

from fractions import Fraction

INF = 2**31 - 1


def all_simple_paths(adj, s, t):
    out = []
    stack = [(s, [s])]
    while stack:
        v, path = stack.pop()
        if v == t:
            out.append(path)
            continue
        for w in adj[v]:
            if w not in path:
                stack.append((w, path + [w]))
    return out


def brute_force(n, edges, roots):
    """Returns (d[k][n], sigma[k][n], delta[k][n] as Fractions, bc[n] as Fractions)."""
    adj = [[] for _ in range(n)]
    for u, v in edges:
        adj[u].append(v)
        adj[v].append(u)
    d = [[INF] * n for _ in roots]
    sig = [[0] * n for _ in roots]
    dl = [[Fraction(0)] * n for _ in roots]
    bc = [Fraction(0)] * n
    for i, s in enumerate(roots):
        d[i][s] = 0
        sig[i][s] = 1
        for t in range(n):
            if t == s:
                continue
            paths = all_simple_paths(adj, s, t)
            if not paths:
                continue
            L = min(len(p) - 1 for p in paths)
            short = [p for p in paths if len(p) - 1 == L]
            d[i][t] = L
            sig[i][t] = len(short)
            for v in range(n):
                if v in (s, t):
                    continue
                through = sum(1 for p in short if v in p[1:-1])
                if through:
                    dl[i][v] += Fraction(through, len(short))
        for v in range(n):
            if v != s:
                bc[v] += dl[i][v]
    return d, sig, dl, bc
