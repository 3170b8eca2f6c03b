"""Synthetic graphs, partitions and required lists (inputs only; see synth/__init__.py)."""
from dataclasses import dataclass
import numpy as np

from ._lib import lib

# R-MAT quadrant probabilities (a, b, c, d) chosen in SURVEY §8(d): Orkut-like max degree and few
# isolated vertices.  Graph500's (0.57, 0.19, 0.19) is kept as a stress variant only.
RMAT_DEFAULT = (0.45, 0.22, 0.22)
RMAT_GRAPH500 = (0.57, 0.19, 0.19)


def _ptr(a):
    return a.ctypes.data if a is not None else None


def permutation(n, seed):
    out = np.empty(n, dtype=np.int64)
    lib().synth_permutation(n, seed, _ptr(out))
    return out


def partition(n, m, seed):
    """Balanced random partition part[v] = perm[v] mod m (stand-in for METIS)."""
    part = np.empty(n, dtype=np.int32)
    lib().synth_partition(n, m, seed, _ptr(part))
    return part


def rmat_edges(n, e, seed, abc=RMAT_DEFAULT):
    """Exactly e distinct directed R-MAT edges u->v (no self-loops), sorted by (u, v)."""
    src = np.empty(e, dtype=np.int32)
    dst = np.empty(e, dtype=np.int32)
    rc = lib().synth_rmat(n, e, seed, abc[0], abc[1], abc[2], _ptr(src), _ptr(dst))
    if rc != 0:
        raise ValueError("synth_rmat failed (n=%d e=%d)" % (n, e))
    return src, dst


def required_lists(src, dst, part, m):
    """R_d ordered by ascending (owner, id), returned as CSR (req_ptr[m+1], req_ids)."""
    n = part.shape[0]
    src = np.ascontiguousarray(src, dtype=np.int32)
    dst = np.ascontiguousarray(dst, dtype=np.int32)
    part = np.ascontiguousarray(part, dtype=np.int32)
    ptr = np.zeros(m + 1, dtype=np.int64)
    L = lib()
    L.synth_required(n, src.shape[0], _ptr(src), _ptr(dst), _ptr(part), m, _ptr(ptr), None)
    ids = np.empty(int(ptr[m]), dtype=np.int64)
    L.synth_required(n, src.shape[0], _ptr(src), _ptr(dst), _ptr(part), m, _ptr(ptr), _ptr(ids))
    return ptr, ids


def required_lists_numpy(src, dst, part, m):
    """Same as required_lists, in numpy (used to cross-check the C helper on small graphs)."""
    src = np.asarray(src, dtype=np.int64)
    dst = np.asarray(dst, dtype=np.int64)
    part = np.asarray(part)
    cut = part[src] != part[dst]
    pairs = np.unique(np.stack([src[cut], part[dst[cut]].astype(np.int64)], axis=1), axis=0)
    lists = []
    for d in range(m):
        u = pairs[pairs[:, 1] == d, 0]
        order = np.lexsort((u, part[u]))
        lists.append(u[order])
    ptr = np.zeros(m + 1, dtype=np.int64)
    ptr[1:] = np.cumsum([len(x) for x in lists])
    ids = np.concatenate(lists) if lists else np.zeros(0, np.int64)
    return ptr, ids.astype(np.int64)


def shuffle_lists(req_ptr, req_ids, seed):
    """Per-GPU seeded shuffle of the halo order (tests: the ABI keeps the caller's R_d order)."""
    out = req_ids.copy()
    m = req_ptr.shape[0] - 1
    for d in range(m):
        a, b = int(req_ptr[d]), int(req_ptr[d + 1])
        if b - a > 1:
            p = permutation(b - a, seed + 7919 * d)
            out[a:b] = req_ids[a:b][p]
    return out


@dataclass
class Graph:
    n: int
    m: int
    src: np.ndarray
    dst: np.ndarray
    part: np.ndarray
    req_ptr: np.ndarray
    req_ids: np.ndarray

    def R(self, d):
        return self.req_ids[self.req_ptr[d]:self.req_ptr[d + 1]]


def make_graph(n, e, m, graph_seed=1, part_seed=101, abc=RMAT_DEFAULT, keep_edges=True):
    src, dst = rmat_edges(n, e, graph_seed, abc)
    part = partition(n, m, part_seed)
    req_ptr, req_ids = required_lists(src, dst, part, m)
    if not keep_edges:
        src = dst = None
    return Graph(n, m, src, dst, part, req_ptr, req_ids)
