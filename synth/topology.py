"""Link-cost topology descriptors: the planner's input D(V', E') (§5.1).

A link i->j between two GPUs is a list of physical hops; each hop h has a bandwidth b_h.  The cost
model charges a stage the max over hops of load x per-row cost, so hops shared by
several links (e.g. a QPI bus) model contention (Table 3).

Per-hop cost is an integer number of ticks per row: w_h = round(1e5 / GBps_h) (SURVEY §8(c) reading
"Cost arithmetic and ties"); this is part of the INPUT, identical for the oracle and the C planner.
"""
from dataclasses import dataclass, field
from typing import Dict, List, Tuple

import numpy as np

# PAPER.md Table 1, GB/s
NV2, NV1, PCIE, QPI = 48.35, 24.22, 11.13, 9.56
B200_NVLINK = 900.0  # NVLink 5, per direction per GPU through NVSwitch


def ticks_of(gbps):
    return int(round(1e5 / gbps))


@dataclass
class Topology:
    name: str
    m: int
    hop_gbps: List[float]
    hop_names: List[str]
    links: Dict[Tuple[int, int], List[int]] = field(default_factory=dict)

    @property
    def hop_ticks(self):
        return [ticks_of(g) for g in self.hop_gbps]

    def link(self, i, j):
        return self.links.get((i, j))

    def csr(self):
        """(hop_ticks int64[H], link_ptr int64[m*m+1], link_hops int32[]) for dgcl_set_topology."""
        ptr = np.zeros(self.m * self.m + 1, dtype=np.int64)
        hops = []
        for i in range(self.m):
            for j in range(self.m):
                hl = self.links.get((i, j), []) if i != j else []
                hops.extend(hl)
                ptr[i * self.m + j + 1] = ptr[i * self.m + j] + len(hl)
        return (np.asarray(self.hop_ticks, dtype=np.int64), ptr,
                np.asarray(hops, dtype=np.int32))


class _Builder:
    def __init__(self, name, m):
        self.t = Topology(name, m, [], [])

    def hop(self, name, gbps):
        self.t.hop_names.append(name)
        self.t.hop_gbps.append(gbps)
        return len(self.t.hop_gbps) - 1

    def link(self, i, j, hops):
        self.t.links[(i, j)] = list(hops)


def uniform_nvswitch(m, gbps=B200_NVLINK):
    """8xB200 NVSwitch box: link i->j = {egress_i, ingress_j}, each 900 GB/s."""
    b = _Builder("uniform_nvswitch", m)
    eg = [b.hop("egress%d" % i, gbps) for i in range(m)]
    ig = [b.hop("ingress%d" % i, gbps) for i in range(m)]
    for i in range(m):
        for j in range(m):
            if i != j:
                b.link(i, j, [eg[i], ig[j]])
    return b.t


def dgx1_like(scale=B200_NVLINK / NV2):
    """Forced non-uniform model after the paper's DGX-1 (Fig. 3).

    Quads {0-3}, {4-7} fully connected by NV2; cross pairs i<->i+4 by NV1; every other pair goes
    PCIe_up(i) -> QPI(socket i -> socket j) -> PCIe_down(j) with the QPI hop shared per direction.
    Table-1 speeds scaled so NV2 = 900 GB/s.
    """
    m = 8
    b = _Builder("dgx1_like", m)
    up = [b.hop("pcie_up%d" % i, PCIE * scale) for i in range(m)]
    down = [b.hop("pcie_down%d" % i, PCIE * scale) for i in range(m)]
    qpi = {(0, 1): b.hop("qpi0to1", QPI * scale), (1, 0): b.hop("qpi1to0", QPI * scale)}
    for i in range(m):
        for j in range(m):
            if i == j:
                continue
            if i // 4 == j // 4:
                b.link(i, j, [b.hop("nv2_%d_%d" % (i, j), NV2 * scale)])
            elif abs(i - j) == 4:
                b.link(i, j, [b.hop("nv1_%d_%d" % (i, j), NV1 * scale)])
            else:
                b.link(i, j, [up[i], qpi[(i // 4, j // 4)], down[j]])
    return b.t


def ring(m=8, fast=B200_NVLINK, slow_factor=10.0):
    """Forced ring model: fast links only to i+-1 (mod m), every other pair 10x slower."""
    b = _Builder("ring", m)
    for i in range(m):
        for j in range(m):
            if i == j:
                continue
            near = (j - i) % m in (1, m - 1)
            b.link(i, j, [b.hop("l%d_%d" % (i, j), fast if near else fast / slow_factor)])
    return b.t


def fig6(nvlink_pairs=((0, 1), (1, 2), (2, 3)), nv=NV1):
    """PAPER.md Fig. 6 topology as read in SURVEY §4: NVLink chain d1-d2-d3-d4 (GPUs 0-3), GPUs
    {0,1} on socket 0 and {2,3} on socket 1; cross-socket pairs without NVLink go
    PCIe_up(src) -> QPI(src socket -> dst socket) -> PCIe_down(dst) (P:1049-1052, P:1067-1071,
    P:1159-1162).  Speeds from Table 1 (NV1 24.22, PCIe 11.13, QPI 9.56 GB/s)."""
    m = 4
    b = _Builder("fig6", m)
    up = [b.hop("pcie_up%d" % i, PCIE) for i in range(m)]
    down = [b.hop("pcie_down%d" % i, PCIE) for i in range(m)]
    qpi = {(0, 1): b.hop("qpi0to1", QPI), (1, 0): b.hop("qpi1to0", QPI)}
    nvp = set()
    for (i, j) in nvlink_pairs:
        nvp.add((i, j))
        nvp.add((j, i))
    for i in range(m):
        for j in range(m):
            if i == j:
                continue
            if (i, j) in nvp:
                b.link(i, j, [b.hop("nv_%d_%d" % (i, j), nv)])
            elif i // 2 != j // 2:
                b.link(i, j, [up[i], qpi[(i // 2, j // 2)], down[j]])
            # same-socket pairs without NVLink: none in Fig. 6 (0-1 and 2-3 have NVLink)
    return b.t


def fig6_pcie():
    """Fig. 6 variant used for the P:1185-1190 contention example: only 0-1 and 2-3 have NVLink,
    so 0->2 and 1->2 both cross PCIe-QPI-PCIe and share the QPI hop."""
    t = fig6(nvlink_pairs=((0, 1), (2, 3)))
    t.name = "fig6_pcie"
    return t


def by_name(name, m=8):
    if name == "uniform_nvswitch":
        return uniform_nvswitch(m)
    if name == "dgx1_like":
        return dgx1_like()
    if name == "ring":
        return ring(m)
    if name == "fig6":
        return fig6()
    if name == "fig6_pcie":
        return fig6_pcie()
    raise ValueError(name)
