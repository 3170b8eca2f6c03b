"""Hash-defined fp32 row values (inputs).  value(seed, stream, key, col) — see synth.cpp synth_fill.

Embedding row of global vertex v at layer l:   key = v,  stream = STREAM_EMB + l
Halo-gradient row i of GPU d at layer l:       key = i,  stream = STREAM_HGRAD + 64*l + d
Incoming emb_grad row of global vertex v:      key = v,  stream = STREAM_EGRAD + l
Because every element is a pure function of (seed, stream, key, col), the oracle can recompute any
sampled element without the GPU's buffers.
"""
import numpy as np

from ._lib import lib

MODES = {"uniform": 0, "ones": 1, "int": 2, "bits": 3}
STREAM_EMB = 0x100
STREAM_HGRAD = 0x20000
STREAM_EGRAD = 0x300

_K0 = np.uint64(0x9E3779B97F4A7C15)
_K1 = np.uint64(0xD1B54A32D192ED03)
_K2 = np.uint64(0xABC98388FB8FAC03)
_K3 = np.uint64(0xC2B2AE3D27D4EB4F)


def fill_values(rows, dim, pitch=None, keys=None, seed=3, stream=STREAM_EMB, mode="uniform"):
    """[rows x pitch] float32 array (padding columns zero), filled by the C helper (OpenMP)."""
    pitch = dim if pitch is None else pitch
    out = np.empty((rows, pitch), dtype=np.float32)
    k = None
    if keys is not None:
        k = np.ascontiguousarray(keys, dtype=np.int64)
        assert k.shape[0] == rows
    lib().synth_fill(out.ctypes.data, rows, pitch, dim, k.ctypes.data if k is not None else None,
                     seed, stream, MODES[mode])
    return out


def _sm64(x):
    with np.errstate(over="ignore"):
        z = x + np.uint64(0x9E3779B97F4A7C15)
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        return z ^ (z >> np.uint64(31))


def fill_values_numpy(keys, cols, seed=3, stream=STREAM_EMB, mode="uniform"):
    """Element-wise numpy twin of synth_fill: value at (keys[i], cols[j]) -> [len(keys), len(cols)].

    Used by tests/oracle to recompute sampled elements independently of any device buffer.
    """
    keys = np.asarray(keys, dtype=np.uint64)[:, None]
    cols = np.asarray(cols, dtype=np.uint64)[None, :]
    with np.errstate(over="ignore"):
        xr = np.uint64(seed) * _K0 ^ np.uint64(stream) * _K3 ^ keys * _K1
        h = _sm64(xr ^ (cols * _K2))
    if mode == "uniform":
        return ((h >> np.uint64(40)).astype(np.float64) * (1.0 / 8388608.0) - 1.0).astype(np.float32)
    if mode == "ones":
        return np.ones(h.shape, dtype=np.float32)
    if mode == "int":
        return ((h >> np.uint64(60)).astype(np.int64) - 8).astype(np.float32)
    if mode == "bits":
        return (h >> np.uint64(32)).astype(np.uint32).view(np.float32)
    raise ValueError(mode)
