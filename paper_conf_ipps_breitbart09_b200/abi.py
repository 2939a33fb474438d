"""Thin ctypes binding of libboids.so (include/boids.h): same names, argument
marshalling only.  Every step of the Boids path runs in the library's CUDA
kernels; there is no Python or CPU fallback -- importing this module on a
machine without the built library raises.

Host arrays are numpy float32 AoS ((count, 3) or (count,)), exactly as the C ABI
takes them.
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(HERE, "libboids.so")

BOIDS_OK, BOIDS_EINVAL, BOIDS_ECUDA, BOIDS_ENCCL, BOIDS_ENOMEM = 0, -1, -2, -3, -4
BOIDS_BRUTE, BOIDS_GRID = 0, 1
BOIDS_INIT_OPENSTEER, BOIDS_INIT_WORLD = 0, 1
BOIDS_STEER_THESIS, BOIDS_STEER_OPENSTEER = 0, 1
BOIDS_KERNEL_FUSED, BOIDS_KERNEL_SIMPLE, BOIDS_KERNEL_CLUSTER = 0, 1, 2
BOIDS_OPT_RECORD_STEERING, BOIDS_OPT_KERNEL, BOIDS_OPT_PROFILE, BOIDS_OPT_CLUSTER, BOIDS_OPT_PHASES = 1, 2, 3, 4, 5
BOIDS_OPT_RESORT, BOIDS_OPT_VOTE_U, BOIDS_OPT_SYMMETRIC, BOIDS_OPT_BALANCE, BOIDS_OPT_GRAPH = 6, 7, 8, 9, 10
BOIDS_OPT_SMALL = 11
BOIDS_PROF_CLASSES = 6
PROF_NAMES = ("fused_or_search", "update", "binning", "grid_search", "route", "search_prep")

# Every symbol include/boids.h declares (tests/test_abi.py checks the header against this).
EXPORTS = (
    "boids_default_params", "boids_create", "boids_create_shard", "boids_set_stream",
    "boids_set_option", "boids_step", "boids_step_shard", "boids_shard_buffers",
    "boids_get_state", "boids_set_state", "boids_get_neighbors", "boids_get_steering",
    "boids_sync", "boids_info", "boids_get_profile", "boids_get_phases", "boids_destroy", "boids_last_error",
    "boids_get_think_state", "boids_set_think_state", "boids_readback_begin", "boids_readback_wait",
    "boids_get_accel", "boids_set_accel", "boids_bench_update",
    "boids_create_spatial", "boids_step_spatial", "boids_spatial_outbox", "boids_spatial_inbox",
    "boids_spatial_unpack", "boids_spatial_owned", "boids_spatial_bounds",
    "boids_symshard_prep", "boids_symshard_search", "boids_symshard_finish", "boids_symshard_buffers",
)
SPATIAL_HALO_F4, SPATIAL_MIG_F4 = 2, 8  # float4 per halo / migrant record (include/boids.h)
# boids_info_t.last_path
BOIDS_PATH_FUSED, BOIDS_PATH_SCAN, BOIDS_PATH_SYM, BOIDS_PATH_GRID, BOIDS_PATH_SIMPLE, BOIDS_PATH_THINK, \
    BOIDS_PATH_SMALL = range(7)


class BoidsError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"boids error {code}: {msg}")
        self.code = code


class boids_params(C.Structure):
    _fields_ = [
        ("search_radius", C.c_float), ("w_separation", C.c_float), ("w_alignment", C.c_float),
        ("w_cohesion", C.c_float), ("max_force", C.c_float), ("max_speed", C.c_float),
        ("mass", C.c_float), ("world_radius", C.c_float), ("init_radius", C.c_float),
        ("init_speed_frac", C.c_float), ("max_neighbors", C.c_int32), ("search_mode", C.c_int32),
        ("init_mode", C.c_int32), ("think_every", C.c_int32), ("steer_mode", C.c_int32),
    ]


class boids_info_t(C.Structure):
    _fields_ = [
        ("n", C.c_int64), ("lo", C.c_int64), ("hi", C.c_int64), ("slice", C.c_int64),
        ("rank", C.c_int32), ("world", C.c_int32), ("kernel", C.c_int32), ("cluster", C.c_int32),
        ("launches", C.c_int64), ("slow_groups", C.c_int64), ("vote_groups", C.c_int64),
        ("fallbacks", C.c_int64), ("grid_pairs", C.c_int64), ("step_index", C.c_int64),
        ("last_path", C.c_int32), ("reserved0", C.c_int32), ("steps_sorted", C.c_int64),
        ("graph_launches", C.c_int64),
    ]


_lib = None


def load(path: str = LIB_PATH):
    """Load libboids.so.  Raises if it has not been built (no fallback exists)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(path):
        raise ImportError(f"{path} is missing: build it with `python -m paper_conf_ipps_breitbart09_b200.build` "
                          "(the Boids path has no CPU fallback)")
    L = C.CDLL(path)
    vp, P, i64, i32, f32 = C.c_void_p, C.POINTER(boids_params), C.c_int64, C.c_int32, C.c_float
    fp = C.POINTER(C.c_float)
    ip = C.POINTER(C.c_int32)
    sig = {
        "boids_default_params": (None, [P]),
        "boids_create": (C.c_int, [i64, P, C.c_uint64, C.POINTER(vp)]),
        "boids_create_shard": (C.c_int, [i64, P, C.c_uint64, i32, i32, C.POINTER(vp)]),
        "boids_set_stream": (C.c_int, [vp, vp]),
        "boids_set_option": (C.c_int, [vp, i32, i64]),
        "boids_step": (C.c_int, [vp, f32, i32]),
        "boids_step_shard": (C.c_int, [vp, f32]),
        "boids_shard_buffers": (C.c_int, [vp, C.POINTER(vp), C.POINTER(vp), C.POINTER(i64)]),
        "boids_get_state": (C.c_int, [vp, fp, fp, fp, fp, fp]),
        "boids_set_state": (C.c_int, [vp, fp, fp, fp, fp, fp]),
        "boids_get_accel": (C.c_int, [vp, fp]),
        "boids_set_accel": (C.c_int, [vp, fp]),
        "boids_get_neighbors": (C.c_int, [vp, ip, ip]),
        "boids_get_steering": (C.c_int, [vp, fp]),
        "boids_sync": (C.c_int, [vp]),
        "boids_info": (C.c_int, [vp, C.POINTER(boids_info_t)]),
        "boids_get_profile": (C.c_int, [vp, C.POINTER(C.c_double), C.POINTER(i64), i32]),
        "boids_get_phases": (C.c_int, [vp, C.POINTER(C.c_uint64), i64]),
        "boids_readback_begin": (C.c_int, [vp, fp]),
        "boids_readback_wait": (C.c_int, [vp]),
        "boids_get_think_state": (C.c_int, [vp, C.POINTER(i64), fp]),
        "boids_set_think_state": (C.c_int, [vp, i64, fp]),
        "boids_bench_update": (C.c_int, [vp, f32, i32, C.POINTER(C.c_double)]),
        "boids_create_spatial": (C.c_int, [i64, P, C.c_uint64, i32, i32, C.POINTER(vp)]),
        "boids_step_spatial": (C.c_int, [vp, f32]),
        "boids_spatial_outbox": (C.c_int, [vp, ip, ip, C.POINTER(vp), C.POINTER(vp), C.POINTER(i64), C.POINTER(i64)]),
        "boids_spatial_inbox": (C.c_int, [vp, C.POINTER(vp), C.POINTER(vp), C.POINTER(i64), C.POINTER(i64)]),
        "boids_spatial_unpack": (C.c_int, [vp, i64, i64]),
        "boids_spatial_owned": (C.c_int, [vp, C.POINTER(C.c_uint8)]),
        "boids_spatial_bounds": (C.c_int, [vp, ip, ip]),
        "boids_symshard_prep": (C.c_int, [vp]),
        "boids_symshard_search": (C.c_int, [vp]),
        "boids_symshard_finish": (C.c_int, [vp, f32]),
        "boids_symshard_buffers": (C.c_int, [vp] + [C.POINTER(vp)] * 6 + [ip]),
        "boids_destroy": (None, [vp]),
        "boids_last_error": (C.c_char_p, []),
    }
    for name, (res, args) in sig.items():
        f = getattr(L, name)
        f.restype = res
        f.argtypes = args
    _lib = L
    return L


def _check(rc: int):
    if rc != BOIDS_OK:
        raise BoidsError(rc, load().boids_last_error().decode(errors="replace"))


def _fptr(a):
    return None if a is None else a.ctypes.data_as(C.POINTER(C.c_float))


def _iptr(a):
    return None if a is None else a.ctypes.data_as(C.POINTER(C.c_int32))


def _f32(a, shape):
    a = np.ascontiguousarray(a, dtype=np.float32)
    return a.reshape(shape)


# ---------------------------------------------------------------- same names
def boids_default_params(**overrides) -> boids_params:
    p = boids_params()
    load().boids_default_params(C.byref(p))
    for k, v in overrides.items():
        setattr(p, k, v)
    return p


def boids_create(n: int, params: boids_params | None = None, seed: int = 1) -> int:
    h = C.c_void_p()
    _check(load().boids_create(n, C.byref(params or boids_default_params()), C.c_uint64(seed), C.byref(h)))
    return h.value


def boids_create_shard(n: int, params: boids_params | None, seed: int, rank: int, world: int) -> int:
    h = C.c_void_p()
    _check(load().boids_create_shard(n, C.byref(params or boids_default_params()), C.c_uint64(seed),
                                     rank, world, C.byref(h)))
    return h.value


def boids_set_stream(h: int, stream_ptr: int | None):
    _check(load().boids_set_stream(h, stream_ptr or None))


def boids_set_option(h: int, option: int, value: int):
    _check(load().boids_set_option(h, option, value))


def boids_step(h: int, dt: float, steps: int = 1):
    _check(load().boids_step(h, C.c_float(dt), steps))


def boids_step_shard(h: int, dt: float):
    _check(load().boids_step_shard(h, C.c_float(dt)))


def boids_shard_buffers(h: int):
    send, full, nbytes = C.c_void_p(), C.c_void_p(), C.c_int64()
    _check(load().boids_shard_buffers(h, C.byref(send), C.byref(full), C.byref(nbytes)))
    return send.value, full.value, nbytes.value


def boids_info(h: int) -> boids_info_t:
    info = boids_info_t()
    _check(load().boids_info(h, C.byref(info)))
    return info


_spans: dict = {}


def _count(h: int) -> int:
    """Owned agents of a handle (hi - lo); cached -- a handle's span never changes."""
    if h not in _spans:
        k = boids_info(h)
        _spans[h] = k.hi - k.lo
    return _spans[h]


def boids_get_state(h: int, out: dict | None = None) -> dict:
    cnt = _count(h)
    out = out or dict(pos=np.empty((cnt, 3), np.float32), fwd=np.empty((cnt, 3), np.float32),
                      up=np.empty((cnt, 3), np.float32), side=np.empty((cnt, 3), np.float32),
                      speed=np.empty(cnt, np.float32))
    _check(load().boids_get_state(h, _fptr(out.get("pos")), _fptr(out.get("fwd")), _fptr(out.get("up")),
                                  _fptr(out.get("side")), _fptr(out.get("speed"))))
    return out


def boids_set_state(h: int, state: dict):
    cnt = _count(h)
    pos = _f32(state["pos"], (cnt, 3))
    fwd = _f32(state["fwd"], (cnt, 3))
    up = _f32(state["up"], (cnt, 3))
    side = None if state.get("side") is None else _f32(state["side"], (cnt, 3))
    speed = _f32(state["speed"], (cnt,))
    _check(load().boids_set_state(h, _fptr(pos), _fptr(fwd), _fptr(up), _fptr(side), _fptr(speed)))


def boids_get_accel(h: int):
    """steer_mode BOIDS_STEER_OPENSTEER: smoothed accelerations (count, 3) of the owned agents."""
    acc = np.empty((_count(h), 3), np.float32)
    _check(load().boids_get_accel(h, _fptr(acc)))
    return acc


def boids_set_accel(h: int, acc):
    _check(load().boids_set_accel(h, _fptr(_f32(acc, (_count(h), 3)))))


def boids_get_neighbors(h: int):
    cnt = _count(h)
    idx = np.empty((cnt, 7), np.int32)
    c = np.empty(cnt, np.int32)
    _check(load().boids_get_neighbors(h, _iptr(idx), _iptr(c)))
    return idx, c


def boids_get_steering(h: int):
    F = np.empty((_count(h), 3), np.float32)
    _check(load().boids_get_steering(h, _fptr(F)))
    return F


def boids_sync(h: int):
    _check(load().boids_sync(h))


def boids_get_profile(h: int, reset: bool = True):
    ms = (C.c_double * BOIDS_PROF_CLASSES)()
    n = (C.c_int64 * BOIDS_PROF_CLASSES)()
    _check(load().boids_get_profile(h, ms, n, 1 if reset else 0))
    return {PROF_NAMES[i]: (ms[i], n[i]) for i in range(BOIDS_PROF_CLASSES)}


def boids_get_phases(h: int, ctas: int):
    out = np.zeros((ctas, 8), np.uint64)
    _check(load().boids_get_phases(h, out.ctypes.data_as(C.POINTER(C.c_uint64)), ctas * 8))
    return out


def boids_readback_begin(h: int, host16) -> None:
    """host16: float32 (count, 4, 4), C-contiguous, ideally pinned; must outlive the readback."""
    if host16.dtype != np.float32 or not host16.flags["C_CONTIGUOUS"] or host16.size != _count(h) * 16:
        raise ValueError("host16 must be a C-contiguous float32 array of count*16 elements")
    _check(load().boids_readback_begin(h, _fptr(host16)))


def boids_readback_wait(h: int) -> None:
    _check(load().boids_readback_wait(h))


def boids_get_think_state(h: int):
    t = C.c_int64()
    F = np.empty((_count(h), 3), np.float32)
    _check(load().boids_get_think_state(h, C.byref(t), _fptr(F)))
    return t.value, F


def boids_set_think_state(h: int, step_index: int, fstore=None):
    F = None if fstore is None else _f32(fstore, (_count(h), 3))
    _check(load().boids_set_think_state(h, step_index, _fptr(F)))


def boids_bench_update(h: int, dt: float, reps: int = 1) -> float:
    """Mean duration (ms) of `reps` standalone k_update launches (state untouched)."""
    ms = C.c_double()
    _check(load().boids_bench_update(h, dt, reps, C.byref(ms)))
    return ms.value


def boids_create_spatial(n: int, params=None, seed: int = 1, rank: int = 0, world: int = 1) -> int:
    h = C.c_void_p()
    _check(load().boids_create_spatial(n, C.byref(params or boids_default_params()), C.c_uint64(seed), rank, world,
                                       C.byref(h)))
    return h.value


def boids_step_spatial(h: int, dt: float):
    _check(load().boids_step_spatial(h, C.c_float(dt)))


def boids_spatial_outbox(h: int, world: int):
    """(halo_counts (world,), mig_counts (world,), halo_out ptr, mig_out ptr, cap_halo, cap_mig)."""
    hc = np.zeros(world, np.int32)
    mc = np.zeros(world, np.int32)
    ho, mo, ch, cm = C.c_void_p(), C.c_void_p(), C.c_int64(), C.c_int64()
    _check(load().boids_spatial_outbox(h, _iptr(hc), _iptr(mc), C.byref(ho), C.byref(mo), C.byref(ch), C.byref(cm)))
    return hc, mc, ho.value, mo.value, ch.value, cm.value


def boids_spatial_inbox(h: int):
    """(halo_in ptr, mig_in ptr, cap_halo_in, cap_mig_in)."""
    hi, mi, ch, cm = C.c_void_p(), C.c_void_p(), C.c_int64(), C.c_int64()
    _check(load().boids_spatial_inbox(h, C.byref(hi), C.byref(mi), C.byref(ch), C.byref(cm)))
    return hi.value, mi.value, ch.value, cm.value


def boids_spatial_unpack(h: int, n_halo: int, n_mig: int):
    _check(load().boids_spatial_unpack(h, n_halo, n_mig))


def boids_spatial_owned(h: int) -> np.ndarray:
    own = np.zeros(_count(h), np.uint8)
    _check(load().boids_spatial_owned(h, own.ctypes.data_as(C.POINTER(C.c_uint8))))
    return own.astype(bool)


def boids_spatial_bounds(h: int, world: int):
    zb = np.zeros(world + 1, np.int32)
    r = np.zeros(1, np.int32)
    _check(load().boids_spatial_bounds(h, _iptr(zb), _iptr(r)))
    return zb, int(r[0])


def boids_symshard_prep(h: int):
    _check(load().boids_symshard_prep(h))


def boids_symshard_search(h: int):
    _check(load().boids_symshard_search(h))


def boids_symshard_finish(h: int, dt: float):
    _check(load().boids_symshard_finish(h, C.c_float(dt)))


def boids_symshard_buffers(h: int):
    """dict of device pointers: lim_send, lim_full, hits, hitcnt, recv, rcnt; and hits_cap."""
    ps = [C.c_void_p() for _ in range(6)]
    cap = np.zeros(1, np.int32)
    _check(load().boids_symshard_buffers(h, *[C.byref(x) for x in ps], _iptr(cap)))
    names = ("lim_send", "lim_full", "hits", "hitcnt", "recv", "rcnt")
    out = {k: v.value for k, v in zip(names, ps)}
    out["hits_cap"] = int(cap[0])
    return out


def boids_destroy(h: int):
    if h:
        _spans.pop(h, None)
        load().boids_destroy(h)


def boids_last_error() -> str:
    return load().boids_last_error().decode(errors="replace")
