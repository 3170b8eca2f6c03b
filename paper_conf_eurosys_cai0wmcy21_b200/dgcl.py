"""Python API over the C ABI (include/dgcl.h).  Argument marshalling only.

PyTorch provides device memory (the workspace and user tensors), streams, and the process group
that exchanges required lists and IPC blobs at setup (§6.3).  Every step of
the hot path runs in libdgcl.so's kernels.

Paper API (§4.2; Listing 1) -> here:
  init()                                 -> init(part, dims, ...) / loopback(...)
  buildCommInfo(graph, topology)         -> Context.build_plan(R lists, topology, seed)
  graphAllgather(localEmbeddings)        -> Context.forward(...) / graph_allgather(...)
  (autograd backward of graphAllgather)  -> Context.backward(...) / GraphAllgather.backward
"""
import ctypes

import numpy as np

from . import _abi
from ._abi import DGCLError, check, lib

__all__ = ["Context", "init", "loopback", "DGCLError", "GraphAllgather", "graph_allgather"]


def _np(a, dtype):
    return np.ascontiguousarray(np.asarray(a), dtype=dtype)


def _stream_ptr(stream):
    import torch
    if stream is None:
        stream = torch.cuda.current_stream()
    return ctypes.c_void_p(stream.cuda_stream)


class Context:
    """One dgcl_ctx (a rank, or all ranks of a loopback job)."""

    def __init__(self, handle, world, rank, part, dims, loopback, device):
        self._h = handle
        self.world = world
        self.rank = rank
        self.part = part
        self.dims = list(dims)
        self.loopback = loopback
        self.device = device
        self.workspace = None
        self.n_local = np.bincount(part, minlength=world).astype(np.int64) if len(part) else \
            np.zeros(world, np.int64)
        self.row_off = np.concatenate([[0], np.cumsum(self.n_local)]).astype(np.int64)
        self.n_halo = None
        self.halo_off = None

    # ---- lifecycle --------------------------------------------------------------------------
    @property
    def handle(self):
        if self._h is None:
            raise DGCLError(_abi.ESTATE, "context destroyed")
        return self._h

    def destroy(self):
        if self._h is not None:
            lib().dgcl_destroy(self._h)
            self._h = None
            self.workspace = None

    def __del__(self):
        try:
            self.destroy()
        except Exception:
            pass

    def set_topology(self, topo):
        """topo: synth.Topology-like object with .csr() -> (hop_ticks, link_ptr, link_hops)."""
        ticks, ptr, hops = topo.csr()
        ticks = _np(ticks, np.int64)
        ptr = _np(ptr, np.int64)
        hops = _np(hops, np.int32)
        t = _abi.Topology(len(ticks), ticks.ctypes.data, ptr.ctypes.data,
                          hops.ctypes.data if hops.size else None)
        check(lib().dgcl_set_topology(self.handle, ctypes.byref(t)), self.handle)

    def build_plan(self, req_ptr, req_ids, seed=0, topology=None, trees=None):
        """buildCommInfo: plan from ALL ranks' required lists (CSR).

        trees: a saved plan, [E x 4] (u, parent, child, stage) as plan_export() returns it (e.g.
        np.save'd by an earlier run): used instead of running SPST, after the plan invariants are
        checked (checkpoint/resume of the planning step)."""
        if topology is not None:
            self.set_topology(topology)
        req_ptr = _np(req_ptr, np.int64)
        req_ids = _np(req_ids, np.int64)
        ids = req_ids.ctypes.data if req_ids.size else None
        if trees is None:
            check(lib().dgcl_build_plan(self.handle, req_ptr.ctypes.data, ids,
                                        ctypes.c_uint64(seed)), self.handle)
        else:
            E = np.asarray(trees)
            u = np.ascontiguousarray(E[:, 0], np.int64)
            pc = [np.ascontiguousarray(E[:, i], np.int32) for i in (1, 2, 3)]
            n = len(u)
            ptr = lambda a: a.ctypes.data if n else None
            check(lib().dgcl_build_plan_from_trees(self.handle, req_ptr.ctypes.data, ids, n,
                                                   ptr(u), ptr(pc[0]), ptr(pc[1]), ptr(pc[2])),
                  self.handle)
        nl = np.zeros(self.world, np.int64)
        nh = np.zeros(self.world, np.int64)
        check(lib().dgcl_rank_rows(self.handle, nl.ctypes.data, nh.ctypes.data), self.handle)
        self.n_halo = nh
        self.halo_off = np.concatenate([[0], np.cumsum(nh)]).astype(np.int64)

    def set_option(self, key, value):
        check(lib().dgcl_set_option(self.handle, key.encode(), int(value)), self.handle)

    # ---- workspace --------------------------------------------------------------------------
    def workspace_bytes(self):
        b = ctypes.c_size_t(0)
        check(lib().dgcl_workspace_bytes(self.handle, ctypes.byref(b)), self.handle)
        return b.value

    def register_workspace(self, tensor=None):
        """Allocate (torch) and register the device workspace; the tensor is kept alive here."""
        import torch
        if tensor is None:
            n = self.workspace_bytes()
            tensor = torch.empty(max(n, 256), dtype=torch.uint8, device="cuda:%d" % self.device)
        check(lib().dgcl_register_workspace(self.handle, ctypes.c_void_p(tensor.data_ptr()),
                                            tensor.numel()), self.handle)
        self.workspace = tensor
        return tensor

    def halo_view(self, layer):
        """(byte offset, rows, pitch) of the halo of `layer` inside the workspace."""
        off = ctypes.c_size_t(0)
        rows = ctypes.c_int64(0)
        pitch = ctypes.c_int64(0)
        check(lib().dgcl_halo_view(self.handle, layer, ctypes.byref(off), ctypes.byref(rows),
                                   ctypes.byref(pitch)), self.handle)
        return off.value, rows.value, pitch.value

    def halo(self, layer):
        """torch view [rows x pitch] float32 of the registered halo of `layer`."""
        import torch
        off, rows, pitch = self.halo_view(layer)
        nbytes = rows * pitch * 4
        return self.workspace[off:off + nbytes].view(torch.float32).view(rows, pitch)

    def pitch(self, layer):
        return self.halo_view(layer)[2]

    def ipc_export(self):
        buf = ctypes.create_string_buffer(_abi.IPC_BLOB_BYTES)
        n = ctypes.c_size_t(_abi.IPC_BLOB_BYTES)
        check(lib().dgcl_ipc_export(self.handle, buf, ctypes.byref(n)), self.handle)
        return buf.raw[:_abi.IPC_BLOB_BYTES]

    def ipc_import(self, blobs):
        data = b"".join(bytes(b).ljust(_abi.IPC_BLOB_BYTES, b"\0") for b in blobs)
        check(lib().dgcl_ipc_import(self.handle, data, _abi.IPC_BLOB_BYTES), self.handle)

    # ---- hot path ---------------------------------------------------------------------------
    def _rows(self):
        return int(len(self.part)) if self.loopback else int(self.n_local[self.rank])

    def _check_arg(self, name, t, layer, rows):
        """The C side sees a pointer and a pitch only: refuse what it cannot check (dtype, device,
        column stride, row count, pitch >= dim) before any out-of-bounds access could happen.
        Raises DGCLError(EINVAL) like the library's own argument checks."""
        import torch

        def bad(msg):
            raise DGCLError(_abi.EINVAL, "%s: %s" % (name, msg))
        if not isinstance(t, torch.Tensor):
            bad("must be a torch tensor")
        if t.dtype != torch.float32:
            bad("must be float32 (got %s)" % t.dtype)
        if not t.is_cuda or t.device.index != self.device:
            bad("must live on cuda:%d (got %s)" % (self.device, t.device))
        if t.dim() != 2 or (t.shape[0] > 0 and t.stride(1) != 1):
            bad("must be a 2-D row-major [rows x pitch] tensor")
        if t.shape[0] < rows:
            bad("has %d rows < %d" % (t.shape[0], rows))
        if 0 <= layer < len(self.dims):   # (a bad layer is the library's EINVAL)
            dim = self.dims[layer]
            if t.shape[1] < dim or (t.shape[0] > 1 and t.stride(0) < dim):
                bad("pitch < dim %d" % dim)

    def _halo_rows(self):
        return int(self.halo_off[-1]) if self.loopback else int(self.n_halo[self.rank])

    def forward(self, layer, emb, halo=None, stream=None):
        """graphAllgather forward: emb (device float32 [rows x pitch]) -> the halo view."""
        self._check_arg("emb", emb, layer, self._rows())
        h = halo if halo is not None else None
        check(lib().dgcl_dispatch_forward(
            self.handle, layer, ctypes.c_void_p(emb.data_ptr()), emb.stride(0),
            ctypes.c_void_p(h.data_ptr()) if h is not None else None, _stream_ptr(stream)),
            self.handle)
        return self.halo(layer)

    def backward(self, layer, halo_grad, emb_grad, stream=None):
        """emb_grad (in/out) += fixed-order fold of halo_grad along the reversed plan."""
        self._check_arg("halo_grad", halo_grad, layer, self._halo_rows())
        self._check_arg("emb_grad", emb_grad, layer, self._rows())
        check(lib().dgcl_dispatch_backward(
            self.handle, layer, ctypes.c_void_p(halo_grad.data_ptr()), halo_grad.stride(0),
            ctypes.c_void_p(emb_grad.data_ptr()), emb_grad.stride(0), _stream_ptr(stream)),
            self.handle)
        return emb_grad

    def forward_host(self, layer, host_emb, host_halo, stream=None):
        """End-to-end forward with host buffers (float32 numpy or pinned torch CPU tensors)."""
        check(lib().dgcl_forward_host(self.handle, layer, _host_ptr(host_emb),
                                      _host_ptr(host_halo), _stream_ptr(stream)), self.handle)

    def backward_host(self, layer, host_halo_grad, host_emb_grad, stream=None):
        check(lib().dgcl_backward_host(self.handle, layer, _host_ptr(host_halo_grad),
                                       _host_ptr(host_emb_grad), _stream_ptr(stream)), self.handle)

    # ---- introspection ----------------------------------------------------------------------
    TRACE_DTYPE = np.dtype([("t_start", "<u8"), ("t_ready", "<u8"), ("t_done", "<u8"),
                            ("sm", "<u4"), ("tag", "<u4")])

    def trace(self, layer, direction=0, rank=0):
        """Per-item timeline of the last launch (option "trace"): a structured array with
        t_start / t_ready / t_done (%globaltimer ns), sm, and op, dir, exec, dst, stage decoded
        from the tag."""
        n = ctypes.c_int64(0)
        check(lib().dgcl_trace_read(self.handle, layer, direction, rank, None, ctypes.byref(n)),
              self.handle)
        rec = np.zeros(n.value, self.TRACE_DTYPE)
        check(lib().dgcl_trace_read(self.handle, layer, direction, rank,
                                    rec.ctypes.data if n.value else None, ctypes.byref(n)),
              self.handle)
        out = {k: rec[k] for k in rec.dtype.names}
        t = rec["tag"]
        out.update(op=t & 15, dir=(t >> 4) & 15, exec=(t >> 8) & 255, dst=(t >> 16) & 255,
                   stage=(t >> 24) & 31, block=t >> 29)
        return out

    def plan_info(self):
        s = _abi.PlanStats()
        check(lib().dgcl_plan_info(self.handle, ctypes.byref(s)), self.handle)
        return s.as_dict()

    def plan_counts(self):
        """Forward rows [K x world x world] per (stage, src, dst)."""
        K = self.plan_info()["n_stages"]
        out = np.zeros((max(K, 1), self.world, self.world), np.int64)
        if K:
            check(lib().dgcl_plan_counts(self.handle, out.ctypes.data), self.handle)
        return out[:K]

    def plan_export(self):
        """Tree edges [E x 4] of (u, parent, child, stage) in planning order."""
        n = ctypes.c_int64(0)
        check(lib().dgcl_plan_export(self.handle, ctypes.byref(n), None, None, None, None),
              self.handle)
        u = np.zeros(n.value, np.int64)
        p = np.zeros(n.value, np.int32)
        c = np.zeros(n.value, np.int32)
        k = np.zeros(n.value, np.int32)
        check(lib().dgcl_plan_export(self.handle, ctypes.byref(n), u.ctypes.data, p.ctypes.data,
                                     c.ctypes.data, k.ctypes.data), self.handle)
        return np.stack([u, p.astype(np.int64), c.astype(np.int64), k.astype(np.int64)], axis=1)

    def device_barrier(self, stream=None):
        """Device-side start barrier over the ranks on `stream` (timing protocol)."""
        check(lib().dgcl_device_barrier(self.handle, _stream_ptr(stream)), self.handle)

    def wait_arrival(self, src=-1, dst=-1, stream=None):
        """Enqueue on `stream` a wait until the rows from `src` (-1: all sources) of the latest
        forward call have landed on `dst` (-1: this rank; loopback: a virtual rank)."""
        check(lib().dgcl_stream_wait_arrival(self.handle, dst, src, _stream_ptr(stream)),
              self.handle)

    # ---- NVSwitch multicast (option "multicast"; see dgcl.h) ---------------------------------
    def multicast_bytes(self):
        """(region bytes, multicast rows) of the plan (0, 0 when nothing is multicast)."""
        b = ctypes.c_size_t(0)
        r = ctypes.c_int64(0)
        check(lib().dgcl_multicast_bytes(self.handle, ctypes.byref(b), ctypes.byref(r)),
              self.handle)
        return b.value, r.value

    def multicast_open(self, fd=None):
        """Rank 0: create the multicast object, return its POSIX fd.  Others: import `fd`."""
        v = ctypes.c_int32(-1 if fd is None else int(fd))
        check(lib().dgcl_multicast_open(self.handle, ctypes.byref(v)), self.handle)
        return v.value

    def multicast_add(self):
        check(lib().dgcl_multicast_add(self.handle), self.handle)

    def multicast_bind(self):
        check(lib().dgcl_multicast_bind(self.handle), self.handle)

    def launch_count(self):
        v = ctypes.c_uint64(0)
        check(lib().dgcl_launch_count(self.handle, ctypes.byref(v)), self.handle)
        return v.value

    def check(self):
        check(lib().dgcl_check(self.handle), self.handle)

    # ---- verification aid (loopback, CPU; never used by forward/backward) -------------------
    def debug_hostsim_forward(self, layer, emb, halo):
        emb = _np(emb, np.float32)
        assert halo.dtype == np.float32 and halo.flags.c_contiguous
        check(lib().dgcl_debug_hostsim_forward(self.handle, layer, emb.ctypes.data,
                                               halo.ctypes.data), self.handle)

    def debug_check_protocol(self, layer, direction=0, mutate=0):
        """Host check of one launch's flag protocol (dgcl.h); raises DGCLError on a violation."""
        buf = ctypes.create_string_buffer(512)
        check(lib().dgcl_debug_check_protocol(self.handle, layer, direction, mutate, buf, 512),
              self.handle)
        return buf.value.decode()

    def debug_hostsim_backward(self, layer, halo_grad, emb_grad):
        halo_grad = _np(halo_grad, np.float32)
        assert emb_grad.dtype == np.float32 and emb_grad.flags.c_contiguous
        check(lib().dgcl_debug_hostsim_backward(self.handle, layer, halo_grad.ctypes.data,
                                                emb_grad.ctypes.data), self.handle)


def multicast_supported(device=0):
    """CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED of `device`."""
    v = ctypes.c_int32(0)
    check(lib().dgcl_multicast_supported(int(device), ctypes.byref(v)))
    return bool(v.value)


def multicast_selftest(device=0, nbytes=1 << 21):
    """(status, message) of the library's one-device multicast self-test (dgcl.h)."""
    buf = ctypes.create_string_buffer(256)
    st = lib().dgcl_debug_multicast_selftest(int(device), int(nbytes), buf, 256)
    return st, buf.value.decode()


def _setup_multicast(ctx, group=None):
    """Collective: rank 0 creates the multicast object and hands its POSIX fd to every other rank
    over a Unix socket (SCM_RIGHTS), every rank adds its device, then binds and maps its memory
    (dgcl_multicast_open / _add / _bind)."""
    import os
    import socket
    import uuid

    import torch.distributed as dist
    rank = dist.get_rank(group)
    world = dist.get_world_size(group)
    srv = None
    name = [None]
    if rank == 0:
        name = ["\0dgcl-mc-%d-%s" % (os.getpid(), uuid.uuid4().hex)]
        srv = socket.socket(socket.AF_UNIX, socket.SOCK_STREAM)
        srv.bind(name[0])
        srv.listen(world)
    dist.broadcast_object_list(name, src=0, group=group)
    try:
        if rank == 0:
            fd = ctx.multicast_open()
            for _ in range(world - 1):
                conn, _ = srv.accept()
                socket.send_fds(conn, [b"m"], [fd])
                conn.close()
            os.close(fd)
        else:
            s = socket.socket(socket.AF_UNIX, socket.SOCK_STREAM)
            s.connect(name[0])
            _msg, fds, _flags, _addr = socket.recv_fds(s, 1, 1)
            s.close()
            ctx.multicast_open(fds[0])
            os.close(fds[0])
    finally:
        if srv is not None:
            srv.close()
    ctx.multicast_add()
    dist.barrier(group=group)
    ctx.multicast_bind()
    dist.barrier(group=group)


def _host_ptr(a):
    if isinstance(a, np.ndarray):
        assert a.dtype == np.float32 and a.flags.c_contiguous
        return ctypes.c_void_p(a.ctypes.data)
    return ctypes.c_void_p(a.data_ptr())


def loopback(world, part, dims, device=0, flags=_abi.LOOPBACK_FUSED):
    """All `world` virtual ranks on one GPU (device < 0: host-only planning context)."""
    part = _np(part, np.int32)
    dims = _np(dims, np.int32)
    h = ctypes.c_void_p()
    check(lib().dgcl_init_loopback(world, device, part.shape[0], part.ctypes.data, len(dims),
                                   dims.ctypes.data, flags, ctypes.byref(h)))
    return Context(h, world, 0, part, dims, True, device)


def init(part, dims, rank, world, device):
    """init() of §4.2 for one rank of a `world`-GPU job."""
    part = _np(part, np.int32)
    dims = _np(dims, np.int32)
    h = ctypes.c_void_p()
    check(lib().dgcl_init(rank, world, device, part.shape[0], part.ctypes.data, len(dims),
                          dims.ctypes.data, ctypes.byref(h)))
    return Context(h, world, rank, part, dims, False, device)


def build_plan_distributed(ctx, my_required, topology=None, seed=0, group=None):
    """buildCommInfo over a process group: all-gather every rank's required list (its halo row
    order), then every rank runs the identical deterministic plan (no master)."""
    import torch.distributed as dist
    world = dist.get_world_size(group)
    lists = [None] * world
    dist.all_gather_object(lists, np.asarray(my_required, dtype=np.int64), group=group)
    ptr = np.zeros(world + 1, np.int64)
    ptr[1:] = np.cumsum([len(x) for x in lists])
    ids = np.concatenate(lists) if ptr[-1] else np.zeros(0, np.int64)
    ctx.build_plan(ptr, ids, seed=seed, topology=topology)
    return ptr, ids


def setup_distributed(part, dims, my_required, topology=None, seed=0, group=None, device=None,
                      options=None):
    """Collective setup over a torch.distributed process group (any backend).

    my_required: this rank's required vertex ids R_me (its halo row order).  The lists of all ranks
    are all-gathered so every rank runs the identical deterministic plan (no master on
    the data path); workspaces are allocated with torch, IPC blobs all-gathered and imported.
    options: {key: value} for dgcl_set_option before planning (the same on every rank).
    """
    import torch
    import torch.distributed as dist
    rank = dist.get_rank(group)
    world = dist.get_world_size(group)
    if device is None:
        device = torch.cuda.current_device()
    ctx = init(part, dims, rank, world, device)
    for k, v in (options or {}).items():
        ctx.set_option(k, v)
    build_plan_distributed(ctx, my_required, topology=topology, seed=seed, group=group)
    ctx.register_workspace()
    blobs = [None] * world
    dist.all_gather_object(blobs, ctx.ipc_export(), group=group)
    if world > 1:
        ctx.ipc_import(blobs)
    dist.barrier(group=group)
    if world > 1 and ctx.multicast_bytes()[1] > 0:
        _setup_multicast(ctx, group)
    return ctx


class GraphAllgather:
    """autograd Function: graphAllgather with the non-atomic backward.

    forward(ctx_dgcl, layer, emb) -> [local; halo] rows (the paper's returned embeddings contain
    local and remote rows); backward splits the gradient, adds the halo part into the
    local part through dispatch_backward.  Built lazily so importing this module needs no torch.
    """
    _fn = None

    @classmethod
    def apply(cls, dctx, layer, emb):
        if cls._fn is None:
            import torch

            class _F(torch.autograd.Function):
                @staticmethod
                def forward(fctx, emb_, dctx_, layer_):
                    # rows whose pitch or base is not 16-B aligned (e.g. a contiguous [n, 602]
                    # tensor) are laid out at the library pitch first, so the launch takes the
                    # bulk-copy executor (the 4-byte register path serves them at ~0.4 of peak)
                    p = dctx_.pitch(layer_)
                    src = emb_
                    if emb_.dim() == 2 and ((emb_.stride(0) * 4) % 16 or emb_.data_ptr() % 16 or
                                            emb_.stride(1) != 1):
                        src = torch.zeros(emb_.shape[0], p, dtype=emb_.dtype, device=emb_.device)
                        src[:, :emb_.shape[1]] = emb_
                    halo = dctx_.forward(layer_, src)
                    fctx.dctx = dctx_
                    fctx.layer = layer_
                    fctx.n = emb_.shape[0]
                    return torch.cat([emb_, halo[:, :emb_.shape[1]]], dim=0)

                @staticmethod
                def backward(fctx, g):
                    n = fctx.n
                    d = fctx.dctx
                    p = d.pitch(fctx.layer)
                    eg = torch.zeros(n, p, dtype=g.dtype, device=g.device)
                    eg[:, :g.shape[1]] = g[:n]
                    hg = torch.zeros(g.shape[0] - n, p, dtype=g.dtype, device=g.device)
                    hg[:, :g.shape[1]] = g[n:]
                    d.backward(fctx.layer, hg, eg)
                    return eg[:, :g.shape[1]], None, None

            cls._fn = _F
        return cls._fn.apply(emb, dctx, layer)


def graph_allgather(dctx, layer, emb):
    return GraphAllgather.apply(dctx, layer, emb)
