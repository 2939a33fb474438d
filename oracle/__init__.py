"""CPU oracle for one Boids step -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s cpu_baseline /
``--impl reference`` legs may import this package.  The product package
``paper_conf_ipps_breitbart09_b200`` never does (a test greps for it).

``boids_oracle.c`` is the oracle (plain C, fp32, no fused ops, single thread);
this module only compiles it with gcc and marshals numpy arrays through ctypes.
See the header of ``boids_oracle.c`` for the PAPER.md passages each function
follows and DESIGN.md for the readings of the paper it adopts.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "boids_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
# Appendix A: no contraction, no fast-math, IEEE binary32 through SSE.
CFLAGS = ["-O2", "-std=c11", "-ffp-contract=off", "-fno-fast-math", "-fPIC", "-shared"]

_lock = threading.Lock()
_lib = None


class OracleParams(C.Structure):
    _fields_ = [
        ("search_radius", C.c_float),
        ("w_separation", C.c_float),
        ("w_alignment", C.c_float),
        ("w_cohesion", C.c_float),
        ("max_force", C.c_float),
        ("max_speed", C.c_float),
        ("mass", C.c_float),
        ("world_radius", C.c_float),
        ("init_radius", C.c_float),
        ("init_speed_frac", C.c_float),
        ("max_neighbors", C.c_int32),
        ("search_mode", C.c_int32),
        ("init_mode", C.c_int32),
        ("think_every", C.c_int32),
        ("steer_mode", C.c_int32),
    ]


def build(force: bool = False) -> str:
    """Compile liboracle.so with gcc (Appendix A flags) if missing or stale."""
    with _lock:
        stale = (not os.path.exists(_LIB)) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC)
        if force or stale:
            tmp = _LIB + f".tmp{os.getpid()}"
            subprocess.check_call(["gcc", *CFLAGS, "-o", tmp, _SRC, "-lm"])
            os.replace(tmp, _LIB)
    return _LIB


def lib():
    global _lib
    if _lib is None:
        L = C.CDLL(build())
        f32p = np.ctypeslib.ndpointer(np.float32, flags="C_CONTIGUOUS")
        i32p = np.ctypeslib.ndpointer(np.int32, flags="C_CONTIGUOUS")
        i64p = np.ctypeslib.ndpointer(np.int64, flags="C_CONTIGUOUS")
        P = C.POINTER(OracleParams)
        L.oracle_default_params.argtypes = [P]
        L.oracle_init.argtypes = [C.c_int64, P, C.c_uint64, f32p, f32p, f32p, f32p, f32p]
        L.oracle_search.argtypes = [C.c_int64, f32p, C.c_float, i32p, i32p]
        L.oracle_search_one.argtypes = [C.c_int64, f32p, C.c_float, C.c_int64, i32p, i32p]
        L.oracle_steer_one.argtypes = [f32p, f32p, C.c_int64, i32p, C.c_int32, P, f32p]
        L.oracle_modify_one.argtypes = [f32p, f32p, f32p, f32p, C.c_float, f32p, P, C.c_float,
                                        f32p, f32p, f32p, f32p, f32p, f32p]
        L.oracle_step.argtypes = ([C.c_int64, P, C.c_float] + [f32p] * 5 + [f32p] * 5
                                  + [i32p, i32p, f32p, f32p])
        L.oracle_step_sample.argtypes = ([C.c_int64, P, C.c_float] + [f32p] * 5 + [C.c_int64, i64p]
                                         + [f32p] * 5 + [i32p, i32p, f32p, f32p])
        L.oracle_step_think.argtypes = ([C.c_int64, P, C.c_float, C.c_int64] + [f32p] * 5 + [f32p] * 5
                                        + [i32p, i32p, f32p, f32p, f32p])
        L.oracle_step_think_sample.argtypes = ([C.c_int64, P, C.c_float, C.c_int64] + [f32p] * 5
                                               + [C.c_int64, i64p] + [f32p] * 5 + [i32p, i32p, f32p, f32p, f32p])
        L.oracle_run.argtypes = [C.c_int64, P, C.c_float, C.c_int32] + [f32p] * 6
        L.oracle_run.restype = C.c_int
        _lib = L
    return _lib


def default_params(**overrides) -> OracleParams:
    p = OracleParams()
    lib().oracle_default_params(C.byref(p))
    for k, v in overrides.items():
        setattr(p, k, v)
    return p


def _f32(a, shape=None):
    a = np.ascontiguousarray(a, dtype=np.float32)
    return a if shape is None else a.reshape(shape)


class State(dict):
    """Host AoS state: pos/fwd/up/side (n,3) float32 and speed (n,) float32; with
    steer_mode 1 also acc (n,3), the smoothed accelerations (zero if absent)."""

    @property
    def n(self) -> int:
        return int(self["pos"].shape[0])

    def copy(self) -> "State":
        return State({k: v.copy() for k, v in self.items()})


def init(n: int, params: OracleParams | None = None, seed: int = 1) -> State:
    """DESIGN.md Appendix B initial state."""
    p = params or default_params()
    s = State(pos=np.zeros((n, 3), np.float32), fwd=np.zeros((n, 3), np.float32),
              up=np.zeros((n, 3), np.float32), side=np.zeros((n, 3), np.float32),
              speed=np.zeros(n, np.float32))
    lib().oracle_init(n, C.byref(p), C.c_uint64(seed & (2**64 - 1)), s["pos"], s["fwd"],
                      s["up"], s["side"], s["speed"])
    return s


def search(pos, radius: float = 9.0):
    """Listing 5.2 for every agent: (idx7 (n,7) int32 -1 padded, cnt (n,) int32)."""
    pos = _f32(pos, (-1, 3))
    n = pos.shape[0]
    idx = np.empty((n, 7), np.int32)
    cnt = np.empty(n, np.int32)
    lib().oracle_search(n, pos, C.c_float(radius), idx, cnt)
    return idx, cnt


def search_one(pos, i: int, radius: float = 9.0):
    pos = _f32(pos, (-1, 3))
    idx = np.empty(7, np.int32)
    cnt = np.empty(1, np.int32)
    lib().oracle_search_one(pos.shape[0], pos, C.c_float(radius), i, idx, cnt)
    return idx, int(cnt[0])


def steer_one(pos, fwd, i: int, idx7, cnt: int, params: OracleParams | None = None):
    p = params or default_params()
    F = np.empty(3, np.float32)
    lib().oracle_steer_one(_f32(pos, (-1, 3)), _f32(fwd, (-1, 3)), i,
                           np.ascontiguousarray(idx7, np.int32), cnt, C.byref(p), F)
    return F


def modify_one(pos, fwd, up, side, speed, force, dt: float, params: OracleParams | None = None, acc=None):
    """acc: steer_mode 1 smoothed acceleration (3,) before the step; the result's
    "acc" is the one after it."""
    p = params or default_params()
    outs = [np.empty(3, np.float32) for _ in range(4)] + [np.empty(1, np.float32)]
    a = np.array(acc if acc is not None else np.zeros(3), np.float32).reshape(3)
    lib().oracle_modify_one(_f32(pos), _f32(fwd), _f32(up), _f32(side), C.c_float(speed),
                            _f32(force), C.byref(p), C.c_float(dt), *outs, a)
    return dict(pos=outs[0], fwd=outs[1], up=outs[2], side=outs[3], speed=float(outs[4][0]), acc=a)


def _state_arrays(s):
    return [_f32(s[k], (-1, 3)) for k in ("pos", "fwd", "up", "side")] + [_f32(s["speed"])]


def _acc_in(s, n):
    """A private copy of the smoothed accelerations (updated in place by the C side)."""
    a = s.get("acc") if hasattr(s, "get") else None
    return np.zeros((n, 3), np.float32) if a is None else np.array(a, np.float32, copy=True).reshape(n, 3)


def _with_acc(out, acc, p):
    if p.steer_mode == 1:
        out["acc"] = acc
    return out


def step(s: State, dt: float, params: OracleParams | None = None):
    """One synchronous step S_t -> S_{t+1}.  Returns (State, idx7, cnt, force)."""
    p = params or default_params()
    n = s.n
    ins = _state_arrays(s)
    out = State(pos=np.empty((n, 3), np.float32), fwd=np.empty((n, 3), np.float32),
                up=np.empty((n, 3), np.float32), side=np.empty((n, 3), np.float32),
                speed=np.empty(n, np.float32))
    idx = np.empty((n, 7), np.int32)
    cnt = np.empty(n, np.int32)
    F = np.empty((n, 3), np.float32)
    acc = _acc_in(s, n)
    lib().oracle_step(n, C.byref(p), C.c_float(dt), *ins, out["pos"], out["fwd"], out["up"],
                      out["side"], out["speed"], idx, cnt, F, acc)
    return _with_acc(out, acc, p), idx, cnt, F


def step_sample(s: State, agents, dt: float, params: OracleParams | None = None):
    """One synchronous step evaluated only for `agents` (each searched against all n)."""
    p = params or default_params()
    agents = np.ascontiguousarray(agents, np.int64)
    m = agents.shape[0]
    out = State(pos=np.empty((m, 3), np.float32), fwd=np.empty((m, 3), np.float32),
                up=np.empty((m, 3), np.float32), side=np.empty((m, 3), np.float32),
                speed=np.empty(m, np.float32))
    idx = np.empty((m, 7), np.int32)
    cnt = np.empty(m, np.int32)
    F = np.empty((m, 3), np.float32)
    acc = np.ascontiguousarray(_acc_in(s, s.n)[agents])
    lib().oracle_step_sample(s.n, C.byref(p), C.c_float(dt), *_state_arrays(s), m, agents,
                             out["pos"], out["fwd"], out["up"], out["side"], out["speed"],
                             idx, cnt, F, acc)
    return _with_acc(out, acc, p), idx, cnt, F


def step_think(s: State, dt: float, t: int, fstore, idx7, cnt, params: OracleParams | None = None):
    """One step with think frequency params.think_every at step index t.

    idx7 (n,7), cnt (n,), fstore (n,3) are the carried think state (copied, not
    modified).  Returns (State, idx7, cnt, fstore, F_used)."""
    p = params or default_params()
    n = s.n
    out = State(pos=np.empty((n, 3), np.float32), fwd=np.empty((n, 3), np.float32),
                up=np.empty((n, 3), np.float32), side=np.empty((n, 3), np.float32),
                speed=np.empty(n, np.float32))
    idx = np.array(idx7, np.int32, copy=True).reshape(n, 7)
    c = np.array(cnt, np.int32, copy=True).reshape(n)
    fs = np.array(fstore, np.float32, copy=True).reshape(n, 3)
    F = np.empty((n, 3), np.float32)
    acc = _acc_in(s, n)
    lib().oracle_step_think(n, C.byref(p), C.c_float(dt), t, *_state_arrays(s), out["pos"], out["fwd"],
                            out["up"], out["side"], out["speed"], idx, c, fs, F, acc)
    return _with_acc(out, acc, p), idx, c, fs, F


def step_think_sample(s: State, agents, dt: float, t: int, fstore, idx7=None, cnt=None,
                      params: OracleParams | None = None):
    """step_think evaluated only for `agents`.  fstore (len(agents), 3), idx7
    (len(agents), 7), cnt (len(agents),) are the sampled agents' carried think
    state (copied).  Returns (State, idx7, cnt, fstore, F_used) per sampled agent."""
    p = params or default_params()
    agents = np.ascontiguousarray(agents, np.int64)
    m = agents.shape[0]
    out = State(pos=np.empty((m, 3), np.float32), fwd=np.empty((m, 3), np.float32),
                up=np.empty((m, 3), np.float32), side=np.empty((m, 3), np.float32),
                speed=np.empty(m, np.float32))
    idx = np.full((m, 7), -1, np.int32) if idx7 is None else np.array(idx7, np.int32, copy=True).reshape(m, 7)
    c = np.full(m, -1, np.int32) if cnt is None else np.array(cnt, np.int32, copy=True).reshape(m)
    fs = np.array(fstore, np.float32, copy=True).reshape(m, 3)
    F = np.empty((m, 3), np.float32)
    acc = np.ascontiguousarray(_acc_in(s, s.n)[agents])
    lib().oracle_step_think_sample(s.n, C.byref(p), C.c_float(dt), t, *_state_arrays(s), m, agents, out["pos"],
                                   out["fwd"], out["up"], out["side"], out["speed"], idx, c, fs, F, acc)
    return _with_acc(out, acc, p), idx, c, fs, F


def run(s: State, dt: float, steps: int, params: OracleParams | None = None) -> State:
    p = params or default_params()
    s = State({k: np.array(v, np.float32, copy=True) for k, v in s.items()})
    arrs = _state_arrays(s)
    acc = _acc_in(s, s.n)
    rc = lib().oracle_run(s.n, C.byref(p), C.c_float(dt), steps, *arrs, acc)
    if rc != 0:
        raise MemoryError("oracle_run")
    return _with_acc(State(pos=arrs[0], fwd=arrs[1], up=arrs[2], side=arrs[3], speed=arrs[4]), acc, p)
