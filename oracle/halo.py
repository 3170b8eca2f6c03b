"""Oracle: re-indexing, forward graphAllgather, backward (flat and tree order).  Plain numpy.

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).
"""
import numpy as np


def local_rows(part, m):
    """Re-indexing of §4.1: each GPU d sees its local vertices V^l_d as rows.

    Reading (R2): loc[v] = number of w < v with part[w] = part[v] (ascending global id).
    Returns (loc int64[N], n_local int64[m]).
    """
    part = np.asarray(part)
    loc = np.empty(part.shape[0], dtype=np.int64)
    n_local = np.zeros(m, dtype=np.int64)
    for d in range(m):
        vs = np.nonzero(part == d)[0]          # ascending ids
        loc[vs] = np.arange(vs.shape[0])
        n_local[d] = vs.shape[0]
    return loc, n_local


def required_bruteforce(n, edges, part, m):
    """V^r_d of §4.1: the direct neighbours of d's local vertices that live on other
    GPUs.  Reading (R3): an edge u->v means v aggregates u (eq. 1), so u is
    required by part[v] when part[u] != part[v].  Explicit loop; each list in ascending id (a set;
    the halo ROW order is the caller's choice, R1)."""
    need = [set() for _ in range(m)]
    for (u, v) in edges:
        if part[u] != part[v]:
            need[part[v]].add(u)
    return [sorted(s) for s in need]


def forward(local_emb, R, part, loc):
    """graphAllgather forward (§4.2): after the call GPU d holds the embedding of every
    vertex in its remote set.  H_d[i, :] = E[R_d[i], :] with E[v] = local_emb[part[v]][loc[v]].

    local_emb: list of m arrays [n_local_d x dim]; R: list of m int arrays (halo row order).
    Returns a list of m arrays [|R_d| x dim] (exact copies; compare through a uint32 view)."""
    m = len(local_emb)
    out = []
    for d in range(m):
        Rd = np.asarray(R[d], dtype=np.int64)
        dim = local_emb[0].shape[1]
        H = np.empty((Rd.shape[0], dim), dtype=local_emb[0].dtype)
        for s in range(m):
            sel = np.nonzero(part[Rd] == s)[0]
            H[sel] = local_emb[s][loc[Rd[sel]]]
        out.append(H)
    return out


def forward_loops(local_emb, R, part, loc):
    """Per-element Python loops twin of forward() (brute force for tiny inputs)."""
    out = []
    for d in range(len(local_emb)):
        dim = local_emb[0].shape[1]
        H = np.zeros((len(R[d]), dim), dtype=local_emb[0].dtype)
        for i, u in enumerate(R[d]):
            for col in range(dim):
                H[i, col] = local_emb[part[u]][loc[u], col]
        out.append(H)
    return out


def contributors(R, n):
    """contrib[u] = [(d, i) for d ascending, i with R_d[i] = u]; |contrib[u]| = |D_u|
    (D_u of §5.1)."""
    contrib = [[] for _ in range(n)]
    for d in range(len(R)):
        for i, u in enumerate(R[d]):
            contrib[int(u)].append((d, i))
    return contrib


def backward_flat(L_local, G, R, part, loc):
    """Backward of graphAllgather (§2; §6.1; §6.2).

    Gradients of the remote copies flow back to the owner and are summed into the owner row.
    Reading (R5/R6): the result is emb_grad_in + the contributions, folded in a fixed
    order: own/local term first, then contributor GPUs in ascending id, each an fp32 add:
        out[loc u] = ((L[loc u] + G_c1[i1]) + G_c2[i2]) + ...,   c1 < c2 < ...
    A vertex appears at most once in each R_c, so the fancy-index update per c below is exactly
    one sequential fp32 add per contributor, in ascending c.
    """
    m = len(L_local)
    out = [np.array(L, dtype=np.float32, copy=True) for L in L_local]
    for c in range(m):
        Rc = np.asarray(R[c], dtype=np.int64)
        for s in range(m):
            sel = np.nonzero(part[Rc] == s)[0]
            rows = loc[Rc[sel]]
            out[s][rows] = (out[s][rows] + G[c][sel]).astype(np.float32)
    return out


def backward_flat_loops(L_local, G, R, part, loc):
    """Per-vertex Python loop twin of backward_flat() (brute force for tiny inputs)."""
    n = part.shape[0]
    out = [np.array(L, dtype=np.float32, copy=True) for L in L_local]
    contrib = contributors(R, n)
    for u in range(n):
        s, r = part[u], loc[u]
        acc = out[s][r].copy()
        for (c, i) in contrib[u]:
            acc = (acc + G[c][i]).astype(np.float32)
        out[s][r] = acc
    return out


def backward_tree_vertex(u, tree_edges_u, L_row, G, pos):
    """Backward along the reversed plan for ONE vertex u (§6.1: stages reversed, send
    and receive tables swapped).  Reading (R6):
        val(x) = (((own(x) + val(y1)) + val(y2)) ...)   children y ascending by GPU id,
        own(x) = G_x[pos_x(u)] if x requested u; a pure relay starts from val(y1);
        root:   out = ((L + val(y1)) + val(y2)) ...
    tree_edges_u: list of (parent, child); pos: dict d -> halo row of u on d (requesters only).
    """
    children = {}
    for (p, c) in tree_edges_u:
        children.setdefault(p, []).append(c)
    for p in children:
        children[p].sort()
    root_candidates = set(children) - {c for (_, c) in tree_edges_u}
    assert len(root_candidates) <= 1

    def val(x):
        acc = None
        if x in pos:
            acc = np.array(G[x][pos[x]], dtype=np.float32, copy=True)
        for y in children.get(x, []):
            vy = val(y)
            acc = vy if acc is None else (acc + vy).astype(np.float32)
        return acc

    acc = np.array(L_row, dtype=np.float32, copy=True)
    root = next(iter(root_candidates)) if root_candidates else None
    if root is not None:
        for y in children[root]:
            acc = (acc + val(y)).astype(np.float32)
    return acc


def backward_tree(L_local, G, R, part, loc, edges, vertices=None):
    """backward_tree_vertex for every vertex (or the sampled `vertices`).

    edges: int array [E x 4] of (u, parent, child, stage) (the plan is data here, not code).
    Returns out (list of m arrays) when vertices is None, else a dict u -> row."""
    n = part.shape[0]
    posmap = [dict() for _ in range(n)] if vertices is None else {int(u): {} for u in vertices}
    for d in range(len(R)):
        for i, u in enumerate(R[d]):
            u = int(u)
            if vertices is None or u in posmap:
                posmap[u][d] = i
    by_u = {}
    for (u, p, c, _k) in np.asarray(edges).reshape(-1, 4):
        u = int(u)
        if vertices is None or u in posmap:
            by_u.setdefault(u, []).append((int(p), int(c)))
    if vertices is not None:
        return {int(u): backward_tree_vertex(int(u), by_u.get(int(u), []),
                                             L_local[part[u]][loc[u]], G, posmap[int(u)])
                for u in vertices}
    out = [np.array(L, dtype=np.float32, copy=True) for L in L_local]
    for u, te in by_u.items():
        out[part[u]][loc[u]] = backward_tree_vertex(u, te, L_local[part[u]][loc[u]], G, posmap[u])
    return out


def fanout(R, n):
    """|D_u| for every vertex (the backward closed form G=1, L=0 => out[u] = |D_u|)."""
    f = np.zeros(n, dtype=np.int64)
    for d in range(len(R)):
        f[np.asarray(R[d], dtype=np.int64)] += 1
    return f
