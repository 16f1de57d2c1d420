"""Thin ctypes binding over libcualign_bp.so (include/cualign_bp.h).

Argument marshalling only: every step of the path runs in the CUDA library.
There is no fallback: if the library is missing or no GPU is present, the
calls fail loudly (CuAlignError / OSError).
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
# CUALIGN_LIB: load another build of the same library (A/B measurements only)
LIB_PATH = os.environ.get("CUALIGN_LIB") or os.path.join(HERE, "lib", "libcualign_bp.so")

OK, EINVAL, ENOMEM, ECUDA, ENCCL, ESTATE = 0, -1, -2, -3, -4, -5
FLAG_DEVICE_PTRS = 0x01
FLAG_EXACT = 0x02
FLAG_OTHERMAX_LITERAL = 0x04
FLAG_ROUND_DAMPED = 0x08
FLAG_TIMING = 0x10
FLAG_MATCH_ROUNDS = 0x20
FLAG_FP32_S = 0x40

K_TOP2, K_EDGE, K_SQUARE, K_ROWSUM, K_MATCH, K_INIT, K_STATE, K_OTHER, K_EVAL, K_MATCHAUX = range(10)
KERNEL_CLASS_NAMES = ["top2", "edge", "square", "rowsum", "match", "init", "state", "other", "eval",
                      "matchaux"]
NUM_KERNEL_CLASSES = 10

# every symbol include/cualign_bp.h declares
EXPORTED = ["cualign_bp_init", "cualign_bp_iterate", "cualign_bp_round", "cualign_bp_run", "cualign_bp_run_trace",
            "cualign_bp_set_timing", "cualign_bp_get_best",
            "cualign_bp_free", "cualign_bp_get_sizes", "cualign_bp_get_S", "cualign_bp_get_state",
            "cualign_bp_set_state", "cualign_bp_get_stats", "cualign_bp_get_round_mates",
            "cualign_bp_sample_squares", "cualign_match", "cualign_last_error",
            "cualign_version", "cualign_nccl_unique_id", "cualign_quality_eval", "cualign_knn"]


class CuAlignError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"cualign status {status}: {msg}")
        self.status = status


class Graph_t(ctypes.Structure):
    _fields_ = [("n", ctypes.c_int32), ("rowptr", ctypes.c_void_p), ("col", ctypes.c_void_p)]


class Edges_t(ctypes.Structure):
    _fields_ = [("m", ctypes.c_int64), ("a", ctypes.c_void_p), ("b", ctypes.c_void_p),
                ("w", ctypes.c_void_p)]


class Params_t(ctypes.Structure):
    _fields_ = [("alpha", ctypes.c_double), ("beta", ctypes.c_double), ("gamma", ctypes.c_double),
                ("flags", ctypes.c_uint32), ("device", ctypes.c_int32), ("stream", ctypes.c_void_p),
                ("rank", ctypes.c_int32), ("world", ctypes.c_int32),
                ("nccl_unique_id", ctypes.c_void_p), ("schedule", ctypes.c_int32),
                ("square_tile_log", ctypes.c_int32)]


class RoundInfo_t(ctypes.Structure):
    _fields_ = [("iter", ctypes.c_int32), ("source", ctypes.c_int32), ("improved", ctypes.c_int32),
                ("best_iter", ctypes.c_int32), ("card_y", ctypes.c_int32), ("card_z", ctypes.c_int32),
                ("score_y", ctypes.c_double), ("score_z", ctypes.c_double),
                ("weight_y", ctypes.c_double), ("weight_z", ctypes.c_double),
                ("score", ctypes.c_double), ("best_score", ctypes.c_double),
                ("overlap_y", ctypes.c_int64), ("overlap_z", ctypes.c_int64),
                ("rounds_y", ctypes.c_int32), ("rounds_z", ctypes.c_int32)]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


class Sizes_t(ctypes.Structure):
    _fields_ = [("n_a", ctypes.c_int32), ("n_b", ctypes.c_int32), ("m", ctypes.c_int64),
                ("s", ctypes.c_int64), ("squares", ctypes.c_int64), ("max_row", ctypes.c_int64),
                ("p", ctypes.c_int32), ("fixed_point_bits", ctypes.c_int32),
                ("device_bytes", ctypes.c_int64), ("rank", ctypes.c_int32), ("world", ctypes.c_int32),
                ("edge_begin", ctypes.c_int64), ("edge_end", ctypes.c_int64),
                ("squares_local", ctypes.c_int64), ("merge_rounds", ctypes.c_int32), ("schedule", ctypes.c_int32)]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


class Stats_t(ctypes.Structure):
    _fields_ = [("launches", ctypes.c_int64),
                ("class_launches", ctypes.c_int64 * NUM_KERNEL_CLASSES),
                ("class_ms", ctypes.c_double * NUM_KERNEL_CLASSES),
                ("comm_calls", ctypes.c_int64), ("comm_bytes_in", ctypes.c_int64), ("comm_ms", ctypes.c_double)]

    def as_dict(self):
        return {"launches": self.launches, "comm_calls": self.comm_calls, "comm_bytes_in": self.comm_bytes_in,
                "comm_ms": self.comm_ms,
                "class_launches": {KERNEL_CLASS_NAMES[i]: self.class_launches[i] for i in range(NUM_KERNEL_CLASSES)},
                "class_ms": {KERNEL_CLASS_NAMES[i]: self.class_ms[i] for i in range(NUM_KERNEL_CLASSES)}}


_lib = None


def load_library():
    """Load libcualign_bp.so (built by __graft_entry__.build() or
    `python -m paper_conf_sc_xiangkfah23_b200.build`).  Raises if missing."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise OSError(f"{LIB_PATH} not found: build it with "
                      "`python -m paper_conf_sc_xiangkfah23_b200.build` (no CPU fallback exists)")
    lib = ctypes.CDLL(LIB_PATH)
    P, I32, I64, D = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64, ctypes.c_double
    lib.cualign_bp_init.restype = I32
    lib.cualign_bp_init.argtypes = [P, P, P, P, ctypes.POINTER(P)]
    lib.cualign_bp_iterate.restype = I32
    lib.cualign_bp_iterate.argtypes = [P, I32]
    lib.cualign_bp_round.restype = I32
    lib.cualign_bp_round.argtypes = [P, P]
    lib.cualign_bp_run.restype = I32
    lib.cualign_bp_run.argtypes = [P, I32, I32]
    lib.cualign_bp_run_trace.restype = I32
    lib.cualign_bp_run_trace.argtypes = [P, I32, P]
    lib.cualign_bp_set_timing.restype = I32
    lib.cualign_bp_set_timing.argtypes = [P, I32]
    lib.cualign_bp_get_best.restype = I32
    lib.cualign_bp_get_best.argtypes = [P, P, P]
    lib.cualign_bp_free.restype = None
    lib.cualign_bp_free.argtypes = [P]
    lib.cualign_bp_get_sizes.restype = I32
    lib.cualign_bp_get_sizes.argtypes = [P, P]
    lib.cualign_bp_get_S.restype = I32
    lib.cualign_bp_get_S.argtypes = [P, P, P, P]
    lib.cualign_bp_get_state.restype = I32
    lib.cualign_bp_get_state.argtypes = [P, P, P, P, P, P, P, P]
    lib.cualign_bp_set_state.restype = I32
    lib.cualign_bp_set_state.argtypes = [P, P, P, P, I32]
    lib.cualign_bp_get_round_mates.restype = I32
    lib.cualign_bp_get_round_mates.argtypes = [P, P, P]
    lib.cualign_bp_sample_squares.restype = I32
    lib.cualign_bp_sample_squares.argtypes = [P, P, I64, I64, P, P, P, P, P]
    lib.cualign_bp_get_stats.restype = I32
    lib.cualign_bp_get_stats.argtypes = [P, P, I32]
    lib.cualign_match.restype = I32
    lib.cualign_match.argtypes = [P, I32, I32, P, P, P, P, P]
    lib.cualign_knn.restype = I32
    lib.cualign_knn.argtypes = [P, I32, P, I32, I32, I32, P, P, P, P]
    lib.cualign_quality_eval.restype = I32
    lib.cualign_quality_eval.argtypes = [P, P, P, P, P, P]
    lib.cualign_last_error.restype = ctypes.c_char_p
    lib.cualign_last_error.argtypes = []
    lib.cualign_version.restype = ctypes.c_char_p
    lib.cualign_version.argtypes = []
    lib.cualign_nccl_unique_id.restype = I32
    lib.cualign_nccl_unique_id.argtypes = [P, I32]
    _lib = lib
    return lib


def _check(status):
    if status != OK:
        msg = load_library().cualign_last_error().decode(errors="replace")
        raise CuAlignError(status, msg)


def _is_torch(x):
    return type(x).__module__.startswith("torch")


def _ptr(x):
    """Data pointer of a numpy array or torch tensor (contiguity checked)."""
    if x is None:
        return None
    if _is_torch(x):
        if not x.is_contiguous():
            raise ValueError("tensor must be contiguous")
        return ctypes.c_void_p(x.data_ptr())
    if not x.flags["C_CONTIGUOUS"]:
        raise ValueError("array must be C-contiguous")
    return x.ctypes.data_as(ctypes.c_void_p)


def _as_host(x, dtype):
    return np.ascontiguousarray(np.asarray(x), dtype=dtype)


def _prep(x, np_dtype, torch_dtype_name):
    if _is_torch(x):
        import torch
        want = getattr(torch, torch_dtype_name)
        if x.dtype != want:
            x = x.to(want)
        return x.contiguous(), x.is_cuda
    return _as_host(x, np_dtype), False


def _stream_ptr(stream):
    if stream is None:
        return None
    handle = stream if isinstance(stream, int) else stream.cuda_stream  # torch.cuda.Stream
    # handle 0 is the legacy default stream: pass cudaStreamLegacy (0x1) so the
    # library runs on it instead of creating a private stream
    return ctypes.c_void_p(handle if handle else 1)


class CuAlignBP:
    """One alignment problem resident on a GPU (Alg. 2 state + S)."""

    def __init__(self, A, B, L, alpha=1.0, beta=2.0, gamma=0.99, flags=0, device=0, stream=None,
                 world=1, rank=0, nccl_id=None, schedule=0, square_tile_log=0):
        """world > 1 with nccl_id (bytes): this process is shard `rank`;
        world > 1 without nccl_id: `world` virtual shards in one handle.
        schedule / square_tile_log: result-neutral tuning (cualign_params)."""
        lib = load_library()
        Ap, dA = _prep(A.rowptr, np.int64, "int64")
        Aj, _ = _prep(A.col, np.int32, "int32")
        Bp, dB = _prep(B.rowptr, np.int64, "int64")
        Bj, _ = _prep(B.col, np.int32, "int32")
        La, dL = _prep(L.a, np.int32, "int32")
        Lb, _ = _prep(L.b, np.int32, "int32")
        w, _ = _prep(L.w, np.float64, "float64")
        on_dev = {dA, dB, dL}
        if len(on_dev) != 1:
            raise ValueError("inputs must be all host arrays or all device tensors")
        if on_dev.pop():
            flags |= FLAG_DEVICE_PTRS
        self._keep = (Ap, Aj, Bp, Bj, La, Lb, w)
        self.n_a, self.n_b, self.m = int(A.n), int(B.n), int(len(L.a))
        self.flags = flags
        ga = Graph_t(self.n_a, _ptr(Ap), _ptr(Aj))
        gb = Graph_t(self.n_b, _ptr(Bp), _ptr(Bj))
        el = Edges_t(self.m, _ptr(La), _ptr(Lb), _ptr(w))
        self.world = int(world)
        if nccl_id is not None:
            import torch  # noqa: F401  -- load torch's NCCL before the library dlopens one
        if self.world > 1 and nccl_id is None:
            rank = -1
        self._nccl_id = ctypes.create_string_buffer(bytes(nccl_id), 128) if nccl_id is not None else None
        prm = Params_t(float(alpha), float(beta), float(gamma), int(flags), int(device),
                       _stream_ptr(stream), int(rank), self.world,
                       ctypes.cast(self._nccl_id, ctypes.c_void_p) if self._nccl_id is not None else None,
                       int(schedule), int(square_tile_log))
        h = ctypes.c_void_p()
        _check(lib.cualign_bp_init(ctypes.byref(ga), ctypes.byref(gb), ctypes.byref(el),
                                   ctypes.byref(prm), ctypes.byref(h)))
        self._h = h
        self._keep = None
        sz = self.sizes()
        self.s = sz["s"]
        self.squares = sz["squares"]

    # lifecycle
    def close(self):
        if getattr(self, "_h", None):
            load_library().cualign_bp_free(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()

    # hot path
    def iterate(self, n_steps=1):
        _check(load_library().cualign_bp_iterate(self._h, int(n_steps)))

    def run(self, n_steps=1, with_round=True, iterate=True):
        """n_steps x (iterate(1) [+ round]) replayed from a CUDA graph (async)."""
        what = (1 if iterate else 0) | (2 if with_round else 0)
        _check(load_library().cualign_bp_run(self._h, int(n_steps), what))

    def run_trace(self, n_steps):
        """n_steps x (iterate + round); returns every step's round info (list of
        dicts, best_score / best_iter as of that step), copied to the host
        step by step without stalling the device (cualign_bp_run_trace)."""
        n = int(n_steps)
        arr = (RoundInfo_t * max(n, 1))()
        _check(load_library().cualign_bp_run_trace(self._h, n, ctypes.cast(arr, ctypes.c_void_p)))
        return [arr[k].as_dict() for k in range(n)]

    def set_timing(self, on=True):
        _check(load_library().cualign_bp_set_timing(self._h, 1 if on else 0))

    def round(self, sync=True):
        if not sync:
            _check(load_library().cualign_bp_round(self._h, None))
            return None
        info = RoundInfo_t()
        _check(load_library().cualign_bp_round(self._h, ctypes.byref(info)))
        return info.as_dict()

    def get_best(self, with_mate=True):
        mate = np.zeros(max(self.n_a, 1), dtype=np.int32) if with_mate else None
        info = RoundInfo_t()
        _check(load_library().cualign_bp_get_best(self._h, _ptr(mate), ctypes.byref(info)))
        return (mate[:self.n_a] if with_mate else None), info.as_dict()

    # introspection
    def sizes(self):
        sz = Sizes_t()
        _check(load_library().cualign_bp_get_sizes(self._h, ctypes.byref(sz)))
        return sz.as_dict()

    def get_S(self):
        rowptr = np.zeros(self.m + 1, dtype=np.int64)
        s = ctypes.c_int64()
        _check(load_library().cualign_bp_get_S(self._h, _ptr(rowptr), None, ctypes.byref(s)))
        col = np.zeros(max(s.value, 1), dtype=np.int32)
        _check(load_library().cualign_bp_get_S(self._h, None, _ptr(col), None))
        return rowptr, col[:s.value]

    def get_state(self, with_S=True):
        m = max(self.m, 1)
        out = {k: np.zeros(m) for k in ("yc", "zc", "yp", "zp", "d")}
        Sp = np.zeros(max(self.s, 1)) if with_S else None
        p = ctypes.c_int32()
        _check(load_library().cualign_bp_get_state(self._h, _ptr(out["yc"]), _ptr(out["zc"]),
                                                    _ptr(out["yp"]), _ptr(out["zp"]),
                                                    _ptr(out["d"]), _ptr(Sp), ctypes.byref(p)))
        out = {k: v[:self.m] for k, v in out.items()}
        if with_S:
            out["Sp"] = Sp[:self.s]
        out["p"] = p.value
        return out

    def set_state(self, yp, zp, Sp, p):
        yp = _as_host(yp, np.float64)
        zp = _as_host(zp, np.float64)
        Sp = _as_host(Sp, np.float64)
        _check(load_library().cualign_bp_set_state(self._h, _ptr(yp), _ptr(zp), _ptr(Sp), int(p)))

    def round_mates(self):
        """(M_y, M_z) of the last rounding as L edge ids per A vertex (-1 = none)."""
        my = np.zeros(max(self.n_a, 1), dtype=np.int32)
        mz = np.zeros(max(self.n_a, 1), dtype=np.int32)
        _check(load_library().cualign_bp_get_round_mates(self._h, _ptr(my), _ptr(mz)))
        return my[:self.n_a], mz[:self.n_a]

    def sample_squares(self, edges):
        """Every square {e < f} touching the given edge ids: dict with arrays
        e, f, v_ef = S^p_ef, v_fe = S^p_fe (cualign_bp_sample_squares)."""
        ed = _as_host(edges, np.int32)
        cnt = ctypes.c_int64()
        cap = 0
        while True:
            out = {"e": np.zeros(max(cap, 1), np.int32), "f": np.zeros(max(cap, 1), np.int32),
                   "v_ef": np.zeros(max(cap, 1)), "v_fe": np.zeros(max(cap, 1))}
            _check(load_library().cualign_bp_sample_squares(self._h, _ptr(ed), int(ed.shape[0]), int(cap),
                                                            _ptr(out["e"]), _ptr(out["f"]), _ptr(out["v_ef"]),
                                                            _ptr(out["v_fe"]), ctypes.byref(cnt)))
            if cnt.value <= cap:
                return {k: v[:cnt.value] for k, v in out.items()}
            cap = int(cnt.value)

    def stats(self, reset=False):
        st = Stats_t()
        _check(load_library().cualign_bp_get_stats(self._h, ctypes.byref(st), int(reset)))
        return st.as_dict()


def match(L, n_a, n_b, x, device=0, flags=0):
    """Standalone locally-dominant matching of L under weights x (host arrays
    or CUDA tensors).  Returns (mate_a, mate_b, rounds)."""
    lib = load_library()
    La, dL = _prep(L.a, np.int32, "int32")
    Lb, _ = _prep(L.b, np.int32, "int32")
    xx, dx = _prep(x, np.float64, "float64")
    if dL != dx:
        raise ValueError("L and x must both be host or both be device")
    if dL:
        flags |= FLAG_DEVICE_PTRS
    el = Edges_t(int(len(L.a)), _ptr(La), _ptr(Lb), None)
    prm = Params_t(1.0, 0.0, 1.0, int(flags), int(device), None, 0, 1, None)
    ma = np.zeros(max(n_a, 1), dtype=np.int32)
    mb = np.zeros(max(n_b, 1), dtype=np.int32)
    rounds = ctypes.c_int32()
    _check(lib.cualign_match(ctypes.byref(el), int(n_a), int(n_b), _ptr(xx), ctypes.byref(prm),
                             _ptr(ma), _ptr(mb), ctypes.byref(rounds)))
    return ma[:n_a], mb[:n_b], rounds.value


class Quality_t(ctypes.Structure):
    _fields_ = [(k, ctypes.c_int64) for k in ("n_a", "n_b", "edges_a", "edges_b", "aligned", "truth_total",
                                              "correct", "conserved", "induced")] + \
               [(k, ctypes.c_double) for k in ("nc", "ec", "ics", "s3", "ncv", "gs3", "ncv_gs3")]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


def alignment_map(mate_a, L):
    """B vertex of each A vertex from a matching given as L edge ids (-1 = none)."""
    mate_a = np.asarray(mate_a)
    lb = np.asarray(L.b, dtype=np.int32)
    return np.where(mate_a >= 0, lb[np.maximum(mate_a, 0)], -1).astype(np.int32)


def quality(A, B, map_ab, truth=None, device=0, flags=0):
    """NEXT-4 quality scores of the alignment map_ab (B vertex per A vertex,
    -1 = unaligned) against A, B and the optional ground truth (see
    cualign_quality_eval).  Returns a dict."""
    lib = load_library()
    Ap, dA = _prep(A.rowptr, np.int64, "int64")
    Aj, _ = _prep(A.col, np.int32, "int32")
    Bp, dB = _prep(B.rowptr, np.int64, "int64")
    Bj, _ = _prep(B.col, np.int32, "int32")
    mp, dm = _prep(map_ab, np.int32, "int32")
    tr, dt = (None, dm) if truth is None else _prep(truth, np.int32, "int32")
    if len({dA, dB, dm, dt}) != 1:
        raise ValueError("inputs must be all host arrays or all device tensors")
    if dA:
        flags |= FLAG_DEVICE_PTRS
    ga = Graph_t(int(A.n), _ptr(Ap), _ptr(Aj))
    gb = Graph_t(int(B.n), _ptr(Bp), _ptr(Bj))
    prm = Params_t(1.0, 0.0, 1.0, int(flags), int(device), None, 0, 1, None)
    q = Quality_t()
    _check(lib.cualign_quality_eval(ctypes.byref(ga), ctypes.byref(gb), _ptr(mp), _ptr(tr), ctypes.byref(prm),
                                    ctypes.byref(q)))
    return q.as_dict()


class KnnCandidates:
    """L built by knn(): m = n_a * k edges in canonical (a, b) order."""

    def __init__(self, n_a, n_b, a, b, w):
        self.n_a, self.n_b, self.a, self.b, self.w = int(n_a), int(n_b), a, b, w

    @property
    def m(self):
        return int(self.a.shape[0])


def knn(YA, YB, k, device=0, flags=0):
    """NEXT-2: L from embeddings (cualign_knn): the k most cosine-similar B
    vertices of every A vertex, on the tensor cores.  YA (n_a x d), YB
    (n_b x d): float32 host arrays or CUDA tensors (then the result is CUDA
    tensors too)."""
    lib = load_library()
    if _is_torch(YA) != _is_torch(YB):
        raise ValueError("YA and YB must both be host arrays or both be tensors")
    if _is_torch(YA):
        import torch
        ya, yb = YA.to(torch.float32).contiguous(), YB.to(torch.float32).contiguous()
        n_a, d = ya.shape
        n_b = yb.shape[0]
        if ya.is_cuda != yb.is_cuda:
            raise ValueError("YA and YB must be on the same side")
        dev = ya.is_cuda
    else:
        ya, yb = _as_host(YA, np.float32), _as_host(YB, np.float32)
        n_a, d = ya.shape
        n_b = yb.shape[0]
        dev = False
    if yb.shape[1] != d:
        raise ValueError("YA and YB need the same embedding dimension")
    m = n_a * k
    if dev:
        import torch
        flags |= FLAG_DEVICE_PTRS
        a = torch.empty(max(m, 1), dtype=torch.int32, device=ya.device)
        b = torch.empty(max(m, 1), dtype=torch.int32, device=ya.device)
        w = torch.empty(max(m, 1), dtype=torch.float64, device=ya.device)
    else:
        a = np.empty(max(m, 1), dtype=np.int32)
        b = np.empty(max(m, 1), dtype=np.int32)
        w = np.empty(max(m, 1), dtype=np.float64)
    prm = Params_t(1.0, 0.0, 1.0, int(flags), int(device), None, 0, 1, None)
    _check(lib.cualign_knn(_ptr(ya), int(n_a), _ptr(yb), int(n_b), int(d), int(k), ctypes.byref(prm),
                           _ptr(a), _ptr(b), _ptr(w)))
    return KnnCandidates(n_a, n_b, a[:m], b[:m], w[:m])


def version():
    return load_library().cualign_version().decode()


def nccl_unique_id() -> bytes:
    """128-byte NCCL unique id for a sharded init (create on one rank, broadcast)."""
    import torch  # noqa: F401  -- torch's NCCL must be the one loaded (the library dlopens libnccl.so.2)
    buf = ctypes.create_string_buffer(128)
    _check(load_library().cualign_nccl_unique_id(buf, 128))
    return buf.raw
