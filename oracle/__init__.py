"""Oracle for the cuAlign NetAlignBP hot path -- TEST INFRASTRUCTURE ONLY.

Plain single-threaded fp64 CPU implementation written from the paper
(/root/reference/PAPER.md; see cualign_oracle.c's header for the passage each
function follows).  Only tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / --impl reference legs may import this package.  It shares no
code with the CUDA library and never imports it.

Python side: ctypes marshalling only; all arithmetic is in cualign_oracle.c,
except the tiny brute-force references in brute.py and the step-by-step
locally-dominant matching in ld_matching.py (used as pins).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "cualign_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

OTHERMAX_LITERAL = 0x1
ROUND_DAMPED = 0x2


def build(force: bool = False) -> str:
    """Compile the oracle (gcc -O2 -ffp-contract=off: no FMA, reading Z26)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + ".tmp%d" % os.getpid()
        subprocess.check_call(["gcc", "-O2", "-ffp-contract=off", "-fno-fast-math", "-std=c11",
                               "-fPIC", "-shared", "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


class RoundInfo(ctypes.Structure):
    _fields_ = [("iter", ctypes.c_int32), ("source", ctypes.c_int32),
                ("improved", ctypes.c_int32), ("best_iter", ctypes.c_int32),
                ("card_y", ctypes.c_int32), ("card_z", ctypes.c_int32),
                ("score_y", ctypes.c_double), ("score_z", ctypes.c_double),
                ("weight_y", ctypes.c_double), ("weight_z", ctypes.c_double),
                ("score", ctypes.c_double), ("best_score", ctypes.c_double),
                ("overlap_y", ctypes.c_int64), ("overlap_z", ctypes.c_int64)]

    def as_dict(self):
        return {name: getattr(self, name) for name, _ in self._fields_}


_lib = None


def _load():
    global _lib
    if _lib is None:
        lib = ctypes.CDLL(build())
        P = ctypes.c_void_p
        lib.orc_create.restype = P
        lib.orc_create.argtypes = [ctypes.c_int32, P, P, ctypes.c_int32, P, P,
                                   ctypes.c_int64, P, P, P,
                                   ctypes.c_double, ctypes.c_double, ctypes.c_int32]
        lib.orc_free.argtypes = [P]
        lib.orc_m.restype = ctypes.c_int64
        lib.orc_m.argtypes = [P]
        lib.orc_s.restype = ctypes.c_int64
        lib.orc_s.argtypes = [P]
        lib.orc_p.restype = ctypes.c_int32
        lib.orc_p.argtypes = [P]
        lib.orc_get_S.argtypes = [P, P, P, P]
        lib.orc_get_state.argtypes = [P, P, P, P, P, P, P]
        lib.orc_set_state.argtypes = [P, P, P, P, ctypes.c_int32]
        lib.orc_step.argtypes = [P, ctypes.c_double, ctypes.c_double]
        lib.orc_greedy.restype = ctypes.c_int32
        lib.orc_greedy.argtypes = [P, P, P]
        lib.orc_evaluate.restype = ctypes.c_double
        lib.orc_evaluate.argtypes = [P, P, P, P, P]
        lib.orc_round.argtypes = [P, ctypes.POINTER(RoundInfo), P, P]
        lib.orc_get_best.argtypes = [P, P, P, P]
        lib.orc_align.argtypes = [P, ctypes.c_int32, ctypes.c_double, ctypes.POINTER(RoundInfo)]
        lib.orc_create_light.restype = P
        lib.orc_create_light.argtypes = [ctypes.c_int32, ctypes.c_int32, ctypes.c_int64, P, P, P]
        _lib = lib
    return _lib


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


class Oracle:
    """Handle over one problem (A, B, L, alpha, beta) and its BP state."""

    def __init__(self, A, B, L, alpha: float, beta: float, flags: int = 0):
        lib = _load()
        self._keep = [np.ascontiguousarray(A.rowptr, dtype=np.int64),
                      np.ascontiguousarray(A.col, dtype=np.int32),
                      np.ascontiguousarray(B.rowptr, dtype=np.int64),
                      np.ascontiguousarray(B.col, dtype=np.int32),
                      np.ascontiguousarray(L.a, dtype=np.int32),
                      np.ascontiguousarray(L.b, dtype=np.int32),
                      np.ascontiguousarray(L.w, dtype=np.float64)]
        Ap, Aj, Bp, Bj, La, Lb, w = self._keep
        self.n_a, self.n_b, self.m = int(A.n), int(B.n), int(L.a.shape[0])
        self.alpha, self.beta, self.flags = float(alpha), float(beta), int(flags)
        self._h = lib.orc_create(self.n_a, _ptr(Ap), _ptr(Aj), self.n_b, _ptr(Bp), _ptr(Bj),
                                 self.m, _ptr(La), _ptr(Lb), _ptr(w),
                                 self.alpha, self.beta, self.flags)
        self.s = int(lib.orc_s(self._h))

    def close(self):
        if getattr(self, "_h", None):
            _load().orc_free(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    @property
    def p(self) -> int:
        return int(_load().orc_p(self._h))

    def get_S(self):
        rowptr = np.zeros(self.m + 1, dtype=np.int64)
        col = np.zeros(max(self.s, 1), dtype=np.int32)
        tau = np.zeros(max(self.s, 1), dtype=np.int64)
        _load().orc_get_S(self._h, _ptr(rowptr), _ptr(col), _ptr(tau))
        return rowptr, col[:self.s], tau[:self.s]

    def get_state(self):
        m, s = max(self.m, 1), max(self.s, 1)
        out = {k: np.zeros(m) for k in ("yc", "zc", "yp", "zp", "d")}
        Sp = np.zeros(s)
        _load().orc_get_state(self._h, _ptr(out["yc"]), _ptr(out["zc"]), _ptr(out["yp"]),
                              _ptr(out["zp"]), _ptr(out["d"]), _ptr(Sp))
        out = {k: v[:self.m] for k, v in out.items()}
        out["Sp"] = Sp[:self.s]
        out["p"] = self.p
        return out

    def set_state(self, yp, zp, Sp, p: int):
        yp = np.ascontiguousarray(yp, dtype=np.float64)
        zp = np.ascontiguousarray(zp, dtype=np.float64)
        Sp = np.ascontiguousarray(Sp, dtype=np.float64)
        _load().orc_set_state(self._h, _ptr(yp), _ptr(zp), _ptr(Sp), int(p))

    def step(self, g: float, h: float):
        """Alg. 2 lines 9-16 once with the given g = gamma^p, h = 1 - g."""
        _load().orc_step(self._h, float(g), float(h))

    def step_gamma(self, gamma: float):
        p = self.p + 1
        g = gamma_power(gamma, p)
        self.step(g, 1.0 - g)

    def greedy(self, x):
        x = np.ascontiguousarray(x, dtype=np.float64)
        mate = np.zeros(max(self.n_a, 1), dtype=np.int32)
        card = _load().orc_greedy(self._h, _ptr(x), _ptr(mate))
        return mate[:self.n_a], int(card)

    def evaluate(self, mate_a):
        mate_a = np.ascontiguousarray(mate_a, dtype=np.int32)
        wt = ctypes.c_double()
        ov = ctypes.c_int64()
        raw = ctypes.c_int64()
        score = _load().orc_evaluate(self._h, _ptr(mate_a), ctypes.byref(wt),
                                     ctypes.byref(ov), ctypes.byref(raw))
        return dict(score=float(score), weight=wt.value, overlap=ov.value, raw=raw.value)

    def round(self):
        info = RoundInfo()
        my = np.zeros(max(self.n_a, 1), dtype=np.int32)
        mz = np.zeros(max(self.n_a, 1), dtype=np.int32)
        _load().orc_round(self._h, ctypes.byref(info), _ptr(my), _ptr(mz))
        d = info.as_dict()
        d["mate_y"] = my[:self.n_a]
        d["mate_z"] = mz[:self.n_a]
        return d

    def get_best(self):
        mate = np.zeros(max(self.n_a, 1), dtype=np.int32)
        sc = ctypes.c_double()
        it = ctypes.c_int32()
        _load().orc_get_best(self._h, _ptr(mate), ctypes.byref(sc), ctypes.byref(it))
        return mate[:self.n_a], sc.value, it.value

    def align(self, n_iter: int, gamma: float):
        infos = (RoundInfo * max(n_iter, 1))()
        _load().orc_align(self._h, int(n_iter), float(gamma), infos)
        return [infos[k].as_dict() for k in range(n_iter)]


class LightOracle:
    """L only (no S): the greedy matching of full-size instances."""

    def __init__(self, L):
        lib = _load()
        self._keep = [np.ascontiguousarray(L.a, dtype=np.int32), np.ascontiguousarray(L.b, dtype=np.int32),
                      np.ascontiguousarray(L.w, dtype=np.float64)]
        self.n_a, self.n_b, self.m = int(L.n_a), int(L.n_b), int(len(L.a))
        self._h = lib.orc_create_light(self.n_a, self.n_b, self.m, *[_ptr(x) for x in self._keep])

    def greedy(self, x):
        x = np.ascontiguousarray(x, dtype=np.float64)
        mate = np.zeros(max(self.n_a, 1), dtype=np.int32)
        card = _load().orc_greedy(self._h, _ptr(x), _ptr(mate))
        return mate[:self.n_a], int(card)

    def close(self):
        if getattr(self, "_h", None):
            _load().orc_free(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def gamma_power(gamma: float, p: int) -> float:
    """g = gamma^p (reading Z2).  Python's float ** int calls the C pow()."""
    return float(gamma) ** float(p)
