"""Oracle: reference SPST planner, Algorithm 1 with incrementalLinkCost (Algorithm 2), §5.2
(PAPER.md P:1200-1321).  Plain Python, for small instances.  TEST INFRASTRUCTURE ONLY.

Readings where the paper is silent (R7-R12):
  * vertices planned: only u with D_u non-empty, ascending id, then "randomly shuffled"
     by Fisher-Yates driven by splitmix64(seed): for i = n-1..1: j = next() % (i+1);
  * Dijkstra (Alg. 1 line 7) is node-labelled and multi-source: every x in N_src starts with label
    (cost 0, depth(x)); relaxing x->y uses C(depth(x)+1, x->y) (the weight of link e
    is C(i, e) when e is i hops from s_u); labels compare (cost, depth, gpu id); nodes of N_src and
    settled nodes are never re-entered; neighbours are relaxed in ascending id; a label is replaced
    only by a strictly smaller (cost, depth);
  * line 8: the target is the unreached d in D_u with the smallest (cost, depth, d);
  * lines 5-11 stop as soon as D_u is inside N_src;
  * Algorithm 2 is evaluated literally: C(i, e) = costFunc(S + {(i, e)}) - costFunc(S), with
    costFunc the §5.1 cost model over integer ticks (oracle/cost.py semantics).
"""
import numpy as np

_GOLD = 0x9E3779B97F4A7C15
_MASK = (1 << 64) - 1


def _mix64(z):
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & _MASK
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & _MASK
    return z ^ (z >> 31)


def shuffle_order(vertices, seed):
    """Fisher-Yates with the sequential splitmix64 stream (state starts at seed)."""
    a = list(vertices)
    state = seed & _MASK
    for i in range(len(a) - 1, 0, -1):
        state = (state + _GOLD) & _MASK
        j = _mix64(state) % (i + 1)
        a[i], a[j] = a[j], a[i]
    return a


class CostState:
    """Per-stage hop loads of the partial plan S and costFunc(S) (§5.1)."""

    def __init__(self, topo):
        self.topo = topo
        self.w = np.asarray(topo.hop_ticks, dtype=np.int64)
        self.load = np.zeros((topo.m, len(self.w)), dtype=np.int64)    # stage 0 unused
        # t_i^k of a link is the max over its hops, t^k the max over links: i.e. the max over the
        # hops that belong to some link
        used = sorted({h for hops in topo.links.values() for h in hops})
        self.used = np.asarray(used, dtype=np.int64)

    def cost_func(self, load=None):
        """t(S) = sum_{k=1}^{m-1} max_i max_j c_ij^k * w_ij."""
        load = self.load if load is None else load
        if self.used.size == 0:
            return 0
        return int((load[1:, self.used] * self.w[self.used]).max(axis=1).sum())

    def incremental(self, k, link):
        """Algorithm 2 line 6: C(k, e) = costFunc(S + {(k, e)}) - costFunc(S)."""
        trial = self.load.copy()
        for h in self.topo.link(*link):
            trial[k, h] += 1
        return self.cost_func(trial) - self.cost_func()

    def add(self, k, link):
        for h in self.topo.link(*link):
            self.load[k, h] += 1


def _dijkstra(topo, state, nsrc_depth):
    """Multi-source node-labelled Dijkstra from N_src (Alg. 1 line 7).  Returns label, pred."""
    m = topo.m
    INF = None
    label = [INF] * m            # (cost, depth)
    pred = [-1] * m
    for x, dx in nsrc_depth.items():
        label[x] = (0, dx)
    settled = [False] * m
    while True:
        best = None
        for x in range(m):
            if not settled[x] and label[x] is not None:
                key = (label[x][0], label[x][1], x)
                if best is None or key < best:
                    best = key
        if best is None:
            break
        x = best[2]
        settled[x] = True
        cx, dx = label[x]
        k = dx + 1
        if k > m - 1:
            continue
        for y in range(m):
            if y == x or settled[y] or y in nsrc_depth or topo.link(x, y) is None:
                continue
            c = state.incremental(k, (x, y))
            new = (cx + c, k)
            if label[y] is None or new < label[y]:
                label[y] = new
                pred[y] = x
    return label, pred


def spst(topo, owner, D, seed, order=None):
    """Algorithm 1.  owner: dict u -> s_u; D: dict u -> set of requesting GPUs (D_u).

    Returns (edges, cost): edges = list of (u, parent, child, stage), vertices in planning order,
    each tree's edges in (stage, child) order (R26), and the final costFunc(S).  Raises ValueError if some d in D_u is unreachable."""
    if order is None:
        order = shuffle_order(sorted(u for u in D if D[u]), seed)
    state = CostState(topo)
    edges = []
    for u in order:
        su = owner[u]
        depth = {su: 0}                       # N_src with tree depths
        remaining = set(D[u]) - {su}
        tree = []
        while remaining:
            # line 6 (Algorithm 2) is evaluated inside _dijkstra on demand; S is fixed meanwhile
            label, pred = _dijkstra(topo, state, depth)
            cands = [(label[d][0], label[d][1], d) for d in remaining if label[d] is not None]
            if not cands:
                raise ValueError("vertex %d: GPUs %s unreachable" % (u, sorted(remaining)))
            _c, _dep, target = min(cands)
            path = []
            y = target
            while y not in depth:
                path.append((pred[y], y))
                y = pred[y]
            path.reverse()
            for (p, c) in path:                # lines 9-10
                k = depth[p] + 1
                depth[c] = k
                tree.append((u, p, c, k))
                state.add(k, (p, c))
                remaining.discard(c)
        # T_u is a set of edges: listed in the canonical (stage, child) order (R26)
        edges.extend(sorted(tree, key=lambda e: (e[3], e[2])))
    return edges, state.cost_func()


def relation_from_lists(R, part):
    """s_u and D_u (§5.1) from the GPUs' required lists."""
    owner, D = {}, {}
    for d in range(len(R)):
        for u in R[d]:
            u = int(u)
            owner[u] = int(part[u])
            D.setdefault(u, set()).add(d)
    return owner, D
