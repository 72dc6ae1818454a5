"""ctypes binding of librgsqr.so (include/rgsqr.h).  Argument marshalling only:
every step of the factorization runs in the library's CUDA kernels.  There is no
CPU fallback -- if the shared library or a CUDA device is missing, calls raise.

Column-major convention: an m x n matrix with leading dimension lda is carried
as a row-major buffer of shape (n, lda) -- i.e. a numpy/torch array ``At`` with
``A[i, j] == At[j, i]``.  numpy arrays in Fortran order (shape (m, n)) are also
accepted for host calls.
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("RGSQR_LIB", os.path.join(_HERE, "librgsqr.so"))   # (override: A/B experiments)

PRECISIONS = {"fp16": 0, "bf16": 1, "tf32": 2, "tf32x3": 3}
STORAGE = {"fp16": "fp16", "bf16": "bf16", "tf32": "fp32", "tf32x3": "fp32"}

OK, WARN_RANK_DEFICIENT = 0, 1
OPTIONS = {"leaf_width": 1, "tile_rows_min": 2, "tile_rows_max": 3, "ring_depth": 4, "algo": 5,
           "block_cols": 6, "serialize": 7, "reuse": 8, "leaf_ctas": 9, "splitk": 10, "profile": 11,
           "reorth": 12, "prefetch": 13, "fuse_small": 14, "split_pct": 15,
           "x3_chain": 16, "colchunk": 17, "eager_pct": 18,
           "chunk_mib": 19, "vshards": 20,
           "defer_pieces": 21, "phasea_pct": 22, "graph": 23}

EXPORTS = ["rgsqr_create", "rgsqr_get_unique_id", "rgsqr_create_dist", "rgsqr_destroy", "rgsqr_factor",
           "rgsqr_factor_device", "rgsqr_op_leaf", "rgsqr_op_inner", "rgsqr_op_outer", "rgsqr_set_stream",
           "rgsqr_get_stream", "rgsqr_host_alloc", "rgsqr_host_free", "rgsqr_set_option", "rgsqr_get_option",
           "rgsqr_get_stats", "rgsqr_version", "rgsqr_status_string", "rgsqr_last_error", "rgsqr_probe_link",
           "rgsqr_ooc_inner", "rgsqr_ooc_outer"]


class Stats(C.Structure):
    _fields_ = [("h2d_bytes", C.c_int64), ("d2h_bytes", C.c_int64), ("h2d_matrix_bytes", C.c_int64),
                ("d2h_matrix_bytes", C.c_int64), ("d2h_r_bytes", C.c_int64), ("d2d_bytes", C.c_int64),
                ("wall_ms", C.c_double), ("h2d_busy_ms", C.c_double), ("d2h_busy_ms", C.c_double),
                ("compute_busy_ms", C.c_double), ("overlap_ratio", C.c_double), ("pin_ms", C.c_double),
                ("arena_bytes", C.c_int64), ("arena_high_water", C.c_int64),
                ("n_leaf_launches", C.c_int64), ("n_tn_launches", C.c_int64), ("n_nn_launches", C.c_int64),
                ("n_other_launches", C.c_int64), ("n_ooc_nodes", C.c_int64), ("n_incore_nodes", C.c_int64),
                ("first_breakdown_col", C.c_int64), ("flops", C.c_int64),
                ("kern_ms", C.c_double * 4), ("kern_launches", C.c_int64 * 4),
                ("kern_flops", C.c_double * 4), ("kern_bytes", C.c_double * 4),
                ("n_colchunk_nodes", C.c_int64), ("colchunk_tail_cols", C.c_int64),
                ("ctx_device_bytes", C.c_int64), ("graph_replay", C.c_int64),
                ("graph_captures", C.c_int64)]

    def as_dict(self):
        out = {}
        for k, _ in self._fields_:
            v = getattr(self, k)
            out[k] = list(v) if k.startswith("kern_") else v
        return out


KERNEL_CLASSES = ("leaf", "inner", "outer", "other")


class RgsqrError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"{msg} (status {status})")
        self.status = status


_lib = None


def load_library(path: str = LIB_PATH):
    """Load librgsqr.so (raises if it has not been built -- no fallback)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(path):
        raise RgsqrError(-5, f"{path} missing: run `python -m paper_conf_icpp_zhangw21_b200.build`")
    lib = C.CDLL(path)
    vp, i64, i32 = C.c_void_p, C.c_int64, C.c_int
    fp = C.POINTER(C.c_float)
    sig = {
        "rgsqr_create": ([C.POINTER(vp), i32], i32),
        "rgsqr_get_unique_id": ([C.c_char_p], i32),
        "rgsqr_create_dist": ([C.POINTER(vp), i32, i32, i32, C.c_char_p], i32),
        "rgsqr_destroy": ([vp], i32),
        "rgsqr_factor": ([vp, vp, i64, i64, i64, vp, vp, i32, C.c_size_t], i32),
        "rgsqr_factor_device": ([vp, vp, i64, i64, i64, vp, vp, i32, C.c_size_t], i32),
        "rgsqr_op_leaf": ([vp, vp, i64, i64, i64, vp, i64, i32, C.POINTER(i32)], i32),
        "rgsqr_op_inner": ([vp, vp, i64, vp, i64, i64, i64, i64, vp, i64, vp, i32, i32], i32),
        "rgsqr_op_outer": ([vp, vp, i64, vp, i64, vp, i64, i64, i64, i64, i32], i32),
        "rgsqr_set_stream": ([vp, vp], i32),
        "rgsqr_get_stream": ([vp, C.POINTER(vp)], i32),
        "rgsqr_host_alloc": ([vp, C.c_size_t, C.POINTER(vp)], i32),
        "rgsqr_host_free": ([vp, vp], i32),
        "rgsqr_set_option": ([vp, i32, i64], i32),
        "rgsqr_get_option": ([vp, i32, C.POINTER(i64)], i32),
        "rgsqr_get_stats": ([vp, C.POINTER(Stats)], i32),
        "rgsqr_version": ([], i32),
        "rgsqr_status_string": ([i32], C.c_char_p),
        "rgsqr_last_error": ([vp], C.c_char_p),
        "rgsqr_probe_link": ([vp, vp, i64, i64, i64, i32, i32, C.POINTER(C.c_double)], i32),
        "rgsqr_ooc_inner": ([vp, vp, i64, vp, i64, i64, i64, i64, vp, i64, i32, i32, i64, C.c_size_t], i32),
        "rgsqr_ooc_outer": ([vp, vp, i64, vp, i64, vp, i64, i64, i64, i64, i32, i32, i64, C.c_size_t], i32),
    }
    del fp
    for name, (args, res) in sig.items():
        f = getattr(lib, name)
        f.argtypes = args
        f.restype = res
    _lib = lib
    return lib


def _ptr(x) -> int:
    if x is None:
        return None
    if isinstance(x, np.ndarray):
        return x.ctypes.data
    if hasattr(x, "data_ptr"):
        return x.data_ptr()
    return int(x)


class Handle:
    """One library context on one GPU (not thread-safe, like the C handle)."""

    def __init__(self, device: int = 0, rank: int = 0, nranks: int = 1, unique_id: bytes | None = None):
        self.lib = load_library()
        h = C.c_void_p()
        if unique_id is not None:      # distributed context (also nranks == 1: same code paths)
            rc = self.lib.rgsqr_create_dist(C.byref(h), device, rank, nranks, unique_id)
        else:
            rc = self.lib.rgsqr_create(C.byref(h), device)
        if rc < 0:
            raise RgsqrError(rc, f"rgsqr_create failed: {self.lib.rgsqr_status_string(rc).decode()}")
        self.h = h
        self.device = device

    @staticmethod
    def unique_id() -> bytes:
        lib = load_library()
        buf = C.create_string_buffer(128)
        rc = lib.rgsqr_get_unique_id(buf)
        if rc < 0:
            raise RgsqrError(rc, "rgsqr_get_unique_id failed")
        return buf.raw

    def close(self):
        if getattr(self, "h", None):
            self.lib.rgsqr_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def _check(self, rc, what):
        if rc < 0:
            raise RgsqrError(rc, f"{what}: {self.lib.rgsqr_status_string(rc).decode()}: "
                                 f"{self.lib.rgsqr_last_error(self.h).decode()}")
        return rc

    # ---- options / stats / stream ----
    def set_option(self, name: str, value: int):
        self._check(self.lib.rgsqr_set_option(self.h, OPTIONS[name], int(value)), f"set_option({name})")

    def get_option(self, name: str) -> int:
        v = C.c_int64()
        self._check(self.lib.rgsqr_get_option(self.h, OPTIONS[name], C.byref(v)), "get_option")
        return v.value

    def stats(self) -> dict:
        s = Stats()
        self._check(self.lib.rgsqr_get_stats(self.h, C.byref(s)), "get_stats")
        return s.as_dict()

    def set_stream(self, stream_ptr: int | None):
        self._check(self.lib.rgsqr_set_stream(self.h, stream_ptr), "set_stream")

    def get_stream(self) -> int:
        p = C.c_void_p()
        self._check(self.lib.rgsqr_get_stream(self.h, C.byref(p)), "get_stream")
        return p.value or 0

    def host_alloc(self, nbytes: int) -> int:
        p = C.c_void_p()
        self._check(self.lib.rgsqr_host_alloc(self.h, nbytes, C.byref(p)), "host_alloc")
        return p.value

    def host_free(self, p: int):
        self._check(self.lib.rgsqr_host_free(self.h, p), "host_free")

    def probe_link(self, host, ld: int, rows: int, cols: int, elem_bytes: int, reps: int = 4) -> dict:
        """Host-link GB/s of the executor's 2D tile copies (H2D, D2H, duplex total)."""
        out = (C.c_double * 3)()
        self._check(self.lib.rgsqr_probe_link(self.h, _ptr(host), ld, rows, cols, elem_bytes, reps, out),
                    "probe_link")
        return {"h2d": out[0], "d2h": out[1], "duplex_total": out[2]}

    # ---- factorizations ----
    def factor(self, A, lda: int, m: int, n: int, Q, R, precision: str = "fp16", budget: int = 0) -> int:
        """Host-resident factorization (A, Q, R host buffers: numpy arrays or raw pointers)."""
        return self._check(self.lib.rgsqr_factor(self.h, _ptr(A), lda, m, n, _ptr(Q), _ptr(R),
                                                 PRECISIONS[precision], int(budget)), "rgsqr_factor")

    def factor_device(self, A, lda: int, m: int, n: int, Q, R, precision: str = "fp16", budget: int = 0) -> int:
        """A, Q, R already in HBM (torch CUDA tensors or device pointers)."""
        return self._check(self.lib.rgsqr_factor_device(self.h, _ptr(A), lda, m, n, _ptr(Q), _ptr(R),
                                                        PRECISIONS[precision], int(budget)),
                           "rgsqr_factor_device")

    # ---- the out-of-core GEMMs (host buffers; Tables 1/2 of the paper) ----
    def ooc_inner(self, Q1, ldq, A2, lda, m, w1, w2, R12, ldr, precision="fp16", tiling=0, block=0, budget=0):
        """R12 = Q1^T A2 streamed from host memory (tiling 0: Fig. 3, 1: Fig. 4)."""
        return self._check(self.lib.rgsqr_ooc_inner(self.h, _ptr(Q1), ldq, _ptr(A2), lda, m, w1, w2, _ptr(R12), ldr,
                                                    PRECISIONS[precision], tiling, block, int(budget)), "ooc_inner")

    def ooc_outer(self, Q1, ldq, R12, ldr, A2, lda, m, w1, w2, precision="fp16", tiling=0, block=0, budget=0):
        """A2 <- A2 - Q1 R12 in host memory (tiling 0: Fig. 5, 1: Fig. 6)."""
        return self._check(self.lib.rgsqr_ooc_outer(self.h, _ptr(Q1), ldq, _ptr(R12), ldr, _ptr(A2), lda, m, w1, w2,
                                                    PRECISIONS[precision], tiling, block, int(budget)), "ooc_outer")

    # ---- hot-path ops (device pointers) ----
    def op_leaf(self, P, ldp, m, w, R11, ldr, precision="fp16") -> tuple[int, int]:
        brk = C.c_int(-1)
        rc = self._check(self.lib.rgsqr_op_leaf(self.h, _ptr(P), ldp, m, w, _ptr(R11), ldr,
                                                PRECISIONS[precision], C.byref(brk)), "op_leaf")
        return rc, brk.value

    def op_inner(self, Q1, ldq, A2, lda, m, w1, w2, R12, ldr, R12op=None, accumulate=False, precision="fp16"):
        return self._check(self.lib.rgsqr_op_inner(self.h, _ptr(Q1), ldq, _ptr(A2), lda, m, w1, w2, _ptr(R12),
                                                   ldr, _ptr(R12op), int(bool(accumulate)),
                                                   PRECISIONS[precision]), "op_inner")

    def op_outer(self, Q1, ldq, R12op, ldr, A2, lda, m, w1, w2, precision="fp16"):
        return self._check(self.lib.rgsqr_op_outer(self.h, _ptr(Q1), ldq, _ptr(R12op), ldr, _ptr(A2), lda,
                                                   m, w1, w2, PRECISIONS[precision]), "op_outer")
