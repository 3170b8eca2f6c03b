"""ctypes loader for synth/_synth.so (built from synth/csrc/synth.cpp by the repo Makefile)."""
import ctypes
import os
import subprocess
import threading

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "_synth.so")
_lock = threading.Lock()
_lib = None


def _build():
    root = os.path.dirname(_HERE)
    subprocess.check_call(["make", "-s", "-C", root, "synth"])


def lib():
    global _lib
    with _lock:
        if _lib is None:
            src = os.path.join(_HERE, "csrc", "synth.cpp")
            if not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(src):
                _build()
            L = ctypes.CDLL(_SO)
            i64, u64, i32 = ctypes.c_int64, ctypes.c_uint64, ctypes.c_int32
            vp = ctypes.c_void_p
            L.synth_permutation.argtypes = [i64, u64, vp]
            L.synth_partition.argtypes = [i64, i32, u64, vp]
            L.synth_rmat.argtypes = [i64, i64, u64, ctypes.c_double, ctypes.c_double,
                                     ctypes.c_double, vp, vp]
            L.synth_rmat.restype = ctypes.c_int
            L.synth_required.argtypes = [i64, i64, vp, vp, vp, i32, vp, vp]
            L.synth_required.restype = ctypes.c_int
            L.synth_fill.argtypes = [vp, i64, i64, i64, vp, u64, u64, i32]
            L.synth_num_threads.restype = ctypes.c_int
            _lib = L
    return _lib
