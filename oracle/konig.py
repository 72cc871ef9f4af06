"""König edge colouring of a regular bipartite multigraph. ORACLE — test infrastructure only.

PAPER.md Thm 6 (L515): "A regular bipartite graph with degree Δ is
Δ-edge-colorable" (refs [20], [21]); Fig. 5 (L527-L529). The paper gives no
algorithm. This is the textbook constructive proof (alternating paths),
deliberately a different algorithm from the product's Euler split:

  for each uncoloured edge (u, v):
      alpha <- a colour missing at u, beta <- a colour missing at v
      if alpha is used at v: swap alpha/beta along the alpha/beta path from v
      colour (u, v) with alpha

After the swap alpha is missing at v; the path cannot reach u (it would have
odd length between the two sides while u misses alpha), so alpha stays
missing at u. O(E * Δ * path) time: small graphs only.
"""
from __future__ import annotations


def edge_colour(n_left: int, n_right: int, edges, degree: int) -> list[int]:
    """Colour each edge (u, v), u in [0,n_left), v in [0,n_right), with one of
    ``degree`` colours so that no two edges sharing an endpoint share a colour.

    ``edges`` is a list of (u, v) pairs (multi-edges allowed). Every node must
    have degree <= ``degree`` (Δ). Returns colour[e] for each edge index e.
    """
    # at[node][colour] = edge index using that colour at that node, or -1.
    # left nodes are 0..n_left-1, right nodes n_left..n_left+n_right-1.
    n_nodes = n_left + n_right
    at = [[-1] * degree for _ in range(n_nodes)]
    colour = [-1] * len(edges)
    ends = [(u, n_left + v) for (u, v) in edges]

    def missing(node: int) -> int:
        row = at[node]
        for c in range(degree):
            if row[c] < 0:
                return c
        raise ValueError("node degree exceeds the colour count")

    for e, (u, v) in enumerate(ends):
        alpha = missing(u)
        beta = missing(v)
        if alpha != beta and at[v][alpha] >= 0:
            # collect the maximal path from v whose edges alternate alpha, beta
            path = []
            node, want = v, alpha
            while True:
                f = at[node][want]
                if f < 0:
                    break
                path.append(f)
                a, b = ends[f]
                node = b if a == node else a
                want = beta if want == alpha else alpha
            # swap alpha <-> beta on the path (clear first, then re-set)
            for f in path:
                a, b = ends[f]
                at[a][colour[f]] = -1
                at[b][colour[f]] = -1
            for f in path:
                a, b = ends[f]
                colour[f] = beta if colour[f] == alpha else alpha
                at[a][colour[f]] = f
                at[b][colour[f]] = f
        colour[e] = alpha
        at[u][alpha] = e
        at[v][alpha] = e
    return colour


def is_proper(n_left: int, n_right: int, edges, colour, degree: int) -> bool:
    """Every colour < degree, and no node has two edges of one colour."""
    seen = set()
    for (u, v), c in zip(edges, colour):
        if not (0 <= c < degree):
            return False
        for key in (("L", u, c), ("R", v, c)):
            if key in seen:
                return False
            seen.add(key)
    return True
