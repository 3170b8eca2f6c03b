"""The NCCL "peer-to-peer" baseline arm of the multi-GPU bench (measurement code, not product).

PAPER.md §7.1 compares DGCL against the peer-to-peer scheme (Table 2 P:566-573 shows
its per-link times): every GPU packs the rows each peer requested by its send list, sends them
point to point, and the receiver unpacks them into its halo.  Here that scheme is written with
stock PyTorch ops and torch.distributed point-to-point calls (NCCL on GPUs: grouped ncclSend /
ncclRecv through batch_isend_irecv; gloo on CPU for the tests):

  forward   pack   sendbuf_d = emb.index_select(0, send[d])      for every requester d
            send / recv (one group)
            unpack halo.index_copy_(0, recv[s], recvbuf_s)      for every owner s
  backward  pack   sendbuf_s = halo_grad.index_select(0, recv[s])
            send / recv (reversed lists)
            fold   emb_grad.index_add_(0, send[d], recvbuf_d)   for d ascending

Each index_add_ has unique row indices, so every element receives exactly one fp32 add per
requester, in ascending requester order: the same fixed order as DESIGN.md R6 (own term first,
then requesters ascending), hence bit-identical to the flat oracle.  The lists are derived here
from the partition and the required lists (the ABI's inputs) and checked against oracle.halo by
tests/test_p2p_baseline.py.
"""
import numpy as np


def p2p_lists(part, req_ptr, req_ids, me, world):
    """Send / receive index lists of rank `me` for the direct (peer-to-peer) exchange.

    send[d]: local rows (ascending-id re-indexing of §4.1) of my vertices in R_d, in
             R_d's order; recv[s]: positions i in R_me with part[R_me[i]] == s (ascending i)."""
    part = np.asarray(part)
    n = part.shape[0]
    loc = np.empty(n, np.int64)
    for d in range(world):
        vs = np.nonzero(part == d)[0]
        loc[vs] = np.arange(vs.shape[0])
    R = [np.asarray(req_ids[req_ptr[d]:req_ptr[d + 1]], np.int64) for d in range(world)]
    send = [np.zeros(0, np.int64) if d == me else loc[R[d][part[R[d]] == me]]
            for d in range(world)]
    recv = [np.zeros(0, np.int64) if s == me else np.nonzero(part[R[me]] == s)[0].astype(np.int64)
            for s in range(world)]
    return send, recv


class P2PExchange:
    """One rank of the peer-to-peer exchange over a torch.distributed process group."""

    def __init__(self, part, req_ptr, req_ids, rank, world, device, group=None):
        import torch
        self.rank, self.world, self.group = rank, world, group
        send, recv = p2p_lists(part, req_ptr, req_ids, rank, world)
        self.send = [torch.from_numpy(a).to(device) for a in send]
        self.recv = [torch.from_numpy(a).to(device) for a in recv]
        self.n_send = [len(a) for a in send]
        self.n_recv = [len(a) for a in recv]
        self.device = device

    def _exchange(self, bufs_out, shapes_in, dtype):
        import torch
        import torch.distributed as dist
        ins = [torch.empty(shapes_in[p], dtype=dtype, device=self.device) if shapes_in[p][0] else
               None for p in range(self.world)]
        ops = []
        for p in range(self.world):
            if p == self.rank:
                continue
            if bufs_out[p] is not None:
                ops.append(dist.P2POp(dist.isend, bufs_out[p], p, self.group))
            if ins[p] is not None:
                ops.append(dist.P2POp(dist.irecv, ins[p], p, self.group))
        if ops:
            for r in dist.batch_isend_irecv(ops):
                r.wait()
        return ins

    def forward(self, emb, halo):
        """halo[i] = emb_global[R_me[i]] for every i (rows of emb's full pitch)."""
        width = emb.shape[1]
        out = [emb.index_select(0, self.send[d]) if self.n_send[d] else None
               for d in range(self.world)]
        ins = self._exchange(out, [(self.n_recv[s], width) for s in range(self.world)], emb.dtype)
        for s in range(self.world):
            if ins[s] is not None:
                halo[:, :width].index_copy_(0, self.recv[s], ins[s])
        return halo

    def backward(self, halo_grad, emb_grad):
        """emb_grad += the requesters' halo-gradient rows, requesters in ascending id."""
        width = halo_grad.shape[1]
        out = [halo_grad.index_select(0, self.recv[s]) if self.n_recv[s] else None
               for s in range(self.world)]
        ins = self._exchange(out, [(self.n_send[d], width) for d in range(self.world)],
                             halo_grad.dtype)
        for d in range(self.world):
            if ins[d] is not None:
                emb_grad[:, :width].index_add_(0, self.send[d], ins[d])
        return emb_grad

    def bytes_out_in(self, row_bytes):
        return (sum(self.n_send) * row_bytes, sum(self.n_recv) * row_bytes)
