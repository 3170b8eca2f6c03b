"""ctypes binding of include/dgcl.h (argument marshalling only; every step runs in libdgcl.so).

Loading fails loudly if the in-tree library is missing: there is no CPU fallback.
"""
import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
# DGCL_LIBRARY: load another in-tree build (A/B performance comparisons); default the package's.
LIB_PATH = os.environ.get("DGCL_LIBRARY") or os.path.join(_HERE, "libdgcl.so")

STATUS = {0: "DGCL_OK", 1: "DGCL_EINVAL", 2: "DGCL_ESTATE", 3: "DGCL_ECUDA", 4: "DGCL_ENOMEM",
          5: "DGCL_ETIMEOUT", 6: "DGCL_EPLAN"}
OK, EINVAL, ESTATE, ECUDA, ENOMEM, ETIMEOUT, EPLAN = range(7)
LOOPBACK_FUSED, LOOPBACK_PER_RANK = 0, 1
IPC_BLOB_BYTES = 256

# every symbol include/dgcl.h declares (tests check the library exports all of them)
SYMBOLS = [
    "dgcl_init", "dgcl_init_loopback", "dgcl_set_topology", "dgcl_build_plan",
    "dgcl_build_plan_from_trees",
    "dgcl_workspace_bytes", "dgcl_register_workspace", "dgcl_halo_view", "dgcl_rank_rows",
    "dgcl_ipc_export", "dgcl_ipc_import", "dgcl_dispatch_forward", "dgcl_dispatch_backward",
    "dgcl_forward_host", "dgcl_backward_host", "dgcl_plan_info", "dgcl_plan_counts",
    "dgcl_plan_export", "dgcl_set_option", "dgcl_trace_read", "dgcl_device_barrier",
    "dgcl_stream_wait_arrival", "dgcl_multicast_supported", "dgcl_multicast_bytes",
    "dgcl_multicast_open", "dgcl_multicast_add", "dgcl_multicast_bind",
    "dgcl_debug_multicast_selftest", "dgcl_debug_check_protocol",
    "dgcl_launch_count", "dgcl_check",
    "dgcl_last_error",
    "dgcl_strerror", "dgcl_destroy", "dgcl_debug_hostsim_forward", "dgcl_debug_hostsim_backward",
]


class DGCLError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__("%s: %s" % (STATUS.get(status, status), msg))
        self.status = status


class Topology(ctypes.Structure):
    _fields_ = [("n_hops", ctypes.c_int32), ("hop_ticks", ctypes.c_void_p),
                ("link_ptr", ctypes.c_void_p), ("link_hops", ctypes.c_void_p)]


class PlanStats(ctypes.Structure):
    _fields_ = [("world", ctypes.c_int32), ("n_stages", ctypes.c_int32),
                ("n_vertices_planned", ctypes.c_int64), ("n_deliveries", ctypes.c_int64),
                ("n_tree_edges", ctypes.c_int64), ("n_relay_rows", ctypes.c_int64),
                ("model_cost_ticks", ctypes.c_int64), ("table_bytes", ctypes.c_int64),
                ("planner_seconds", ctypes.c_double), ("lowering_seconds", ctypes.c_double),
                ("n_fwd_groups", ctypes.c_int32), ("n_bwd_groups", ctypes.c_int32),
                ("n_multicast_rows", ctypes.c_int64)]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


_lib = None


def lib():
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError("libdgcl.so not built (%s); run `make -C %s dgcl` or "
                              "__graft_entry__.build()" % (LIB_PATH, os.path.dirname(_HERE)))
        L = ctypes.CDLL(LIB_PATH)
        P, I32, I64, U64, SZ = (ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64, ctypes.c_uint64,
                                ctypes.c_size_t)
        pp = ctypes.POINTER(ctypes.c_void_p)
        sig = {
            "dgcl_init": [I32, I32, I32, I64, P, I32, P, pp],
            "dgcl_init_loopback": [I32, I32, I64, P, I32, P, I32, pp],
            "dgcl_set_topology": [P, ctypes.POINTER(Topology)],
            "dgcl_build_plan": [P, P, P, U64],
            "dgcl_build_plan_from_trees": [P, P, P, I64, P, P, P, P],
            "dgcl_workspace_bytes": [P, ctypes.POINTER(SZ)],
            "dgcl_register_workspace": [P, P, SZ],
            "dgcl_halo_view": [P, I32, ctypes.POINTER(SZ), ctypes.POINTER(I64), ctypes.POINTER(I64)],
            "dgcl_rank_rows": [P, P, P],
            "dgcl_ipc_export": [P, P, ctypes.POINTER(SZ)],
            "dgcl_ipc_import": [P, P, SZ],
            "dgcl_dispatch_forward": [P, I32, P, I64, P, P],
            "dgcl_dispatch_backward": [P, I32, P, I64, P, I64, P],
            "dgcl_forward_host": [P, I32, P, P, P],
            "dgcl_backward_host": [P, I32, P, P, P],
            "dgcl_plan_info": [P, ctypes.POINTER(PlanStats)],
            "dgcl_plan_counts": [P, P],
            "dgcl_plan_export": [P, ctypes.POINTER(I64), P, P, P, P],
            "dgcl_set_option": [P, ctypes.c_char_p, I64],
            "dgcl_trace_read": [P, I32, I32, I32, P, ctypes.POINTER(I64)],
            "dgcl_device_barrier": [P, P],
            "dgcl_stream_wait_arrival": [P, I32, I32, P],
            "dgcl_multicast_supported": [I32, ctypes.POINTER(I32)],
            "dgcl_multicast_bytes": [P, ctypes.POINTER(SZ), ctypes.POINTER(I64)],
            "dgcl_multicast_open": [P, ctypes.POINTER(I32)],
            "dgcl_multicast_add": [P],
            "dgcl_multicast_bind": [P],
            "dgcl_debug_multicast_selftest": [I32, I64, ctypes.c_char_p, SZ],
            "dgcl_debug_check_protocol": [P, I32, I32, I32, ctypes.c_char_p, SZ],
            "dgcl_launch_count": [P, ctypes.POINTER(U64)],
            "dgcl_check": [P],
            "dgcl_destroy": [P],
            "dgcl_debug_hostsim_forward": [P, I32, P, P],
            "dgcl_debug_hostsim_backward": [P, I32, P, P],
        }
        for name, args in sig.items():
            f = getattr(L, name)
            f.argtypes = args
            f.restype = ctypes.c_int
        L.dgcl_last_error.argtypes = [P]
        L.dgcl_last_error.restype = ctypes.c_char_p
        L.dgcl_strerror.argtypes = [ctypes.c_int]
        L.dgcl_strerror.restype = ctypes.c_char_p
        _lib = L
    return _lib


def check(status, ctx=None):
    if status != OK:
        msg = lib().dgcl_last_error(ctx).decode() if ctx else lib().dgcl_strerror(status).decode()
        raise DGCLError(status, msg)
