"""paper_conf_icpp_wangzll21_b200 — B200-native texture identification (Wang et al., ICPP'21).

Thin ctypes binding over the C ABI in ``include/tid.h`` (``libtid.so``, built for
sm_100a).  Argument marshalling only: every step of the hot path runs in the
library's CUDA kernels.  Inputs may be NumPy arrays, host torch tensors or CUDA
torch tensors; PyTorch is used only as a container for device memory and streams.

There is no CPU fallback: if ``libtid.so`` is missing or the device is not an
sm_100 B200, every call raises.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("TID_LIB") or os.path.join(_HERE, "libtid.so")

TID_OK, TID_EINVAL, TID_ENOMEM, TID_ECUDA, TID_ENCCL, TID_EUNSUPPORTED, TID_ESTATE = 0, -1, -2, -3, -4, -5, -6
STATUS = {0: "TID_OK", -1: "TID_EINVAL", -2: "TID_ENOMEM", -3: "TID_ECUDA", -4: "TID_ENCCL",
          -5: "TID_EUNSUPPORTED", -6: "TID_ESTATE"}

# every symbol declared in include/tid.h
EXPORTS = ("tid_index_create", "tid_index_destroy", "tid_add_references", "tid_search", "tid_search_counts",
           "tid_verify", "tid_merge_topk", "tid_nccl_unique_id", "tid_get_info", "tid_profile", "tid_get_stats",
           "tid_set_tuning", "tid_delete_references", "tid_update_references", "tid_index_save", "tid_index_load",
           "tid_f16_prepare", "tid_f16_search_counts", "tid_host_tier_map", "tid_verify_geometric",
           "tid_last_error")


class TidError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = status


class Config(ctypes.Structure):
    _fields_ = [("device", ctypes.c_int32), ("dim", ctypes.c_int32), ("ref_kp", ctypes.c_int32),
                ("query_kp_max", ctypes.c_int32), ("ratio_num", ctypes.c_uint32), ("ratio_den", ctypes.c_uint32),
                ("hbm_budget_bytes", ctypes.c_uint64), ("host_budget_bytes", ctypes.c_uint64),
                ("id_base", ctypes.c_int64), ("rank", ctypes.c_int32), ("world_size", ctypes.c_int32),
                ("nccl_unique_id", ctypes.c_void_p), ("cache_policy", ctypes.c_int32), ("descriptor", ctypes.c_int32),
                ("f16_scale", ctypes.c_float), ("f16_rootsift", ctypes.c_int32)]


class Info(ctypes.Structure):
    _fields_ = [("num_references", ctypes.c_int64), ("hbm_references", ctypes.c_int64),
                ("host_references", ctypes.c_int64), ("hbm_bytes", ctypes.c_int64), ("host_bytes", ctypes.c_int64),
                ("num_sms", ctypes.c_int32), ("world_size", ctypes.c_int32),
                ("hbm_capacity_references", ctypes.c_int64), ("host_capacity_references", ctypes.c_int64),
                ("hbm_bytes_per_reference", ctypes.c_int64)]


class Stats(ctypes.Structure):
    _fields_ = [("match_launches", ctypes.c_int64), ("match_ms", ctypes.c_double),
                ("kernel_launches", ctypes.c_int64), ("h2d_bytes", ctypes.c_int64), ("d2h_bytes", ctypes.c_int64)]


class GeomParams(ctypes.Structure):
    _fields_ = [("border", ctypes.c_float), ("query_width", ctypes.c_float), ("query_height", ctypes.c_float),
                ("ref_width", ctypes.c_float), ("ref_height", ctypes.c_float), ("inlier_px", ctypes.c_float),
                ("iterations", ctypes.c_int32), ("seed", ctypes.c_uint64)]


class Tuning(ctypes.Structure):
    _fields_ = [("refs_per_job", ctypes.c_int32), ("grid", ctypes.c_int32), ("host_chunk_refs", ctypes.c_int64),
                ("window_refs", ctypes.c_int64)]


_lib = None


def load_library(path: str = LIB_PATH):
    """Load libtid.so (raises if it has not been built — there is no fallback)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(path):
        raise ImportError(f"{path} not found: build it with `python -m paper_conf_icpp_wangzll21_b200.build` "
                          "(no CPU fallback exists)")
    lib = ctypes.CDLL(path)
    vp, i32, i64, u32 = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64, ctypes.c_uint32
    P = ctypes.POINTER
    lib.tid_index_create.argtypes = [P(Config), P(vp)]
    lib.tid_index_destroy.argtypes = [vp]
    lib.tid_add_references.argtypes = [vp, vp, vp, i64, P(i64)]
    lib.tid_search.argtypes = [vp, vp, vp, i32, i64, i32, vp, vp, vp]
    lib.tid_search_counts.argtypes = [vp, vp, vp, i32, i64, vp, vp]
    lib.tid_verify.argtypes = [vp, vp, i32, vp, i32, i64, vp, vp, vp, vp, vp]
    lib.tid_merge_topk.argtypes = [vp, vp, vp, i32, i64, i32, vp, vp, vp]
    lib.tid_nccl_unique_id.argtypes = [vp]
    lib.tid_get_info.argtypes = [vp, P(Info)]
    lib.tid_profile.argtypes = [vp, i32]
    lib.tid_get_stats.argtypes = [vp, P(Stats)]
    lib.tid_set_tuning.argtypes = [vp, P(Tuning)]
    lib.tid_delete_references.argtypes = [vp, vp, i64]
    lib.tid_update_references.argtypes = [vp, vp, vp, vp, i64]
    lib.tid_index_save.argtypes = [vp, ctypes.c_char_p]
    lib.tid_index_load.argtypes = [vp, ctypes.c_char_p, P(i64)]
    lib.tid_f16_prepare.argtypes = [vp, vp, i64, i32, ctypes.c_float, vp, vp]
    lib.tid_f16_search_counts.argtypes = [vp, vp, i32, i64, vp, i32, i64, vp, vp]
    lib.tid_host_tier_map.argtypes = [vp, i64, P(ctypes.POINTER(ctypes.c_uint8)), P(i64)]
    lib.tid_verify_geometric.argtypes = [vp, vp, i32, vp, i32, i64, vp, vp, vp, vp, P(GeomParams), vp, vp, vp, vp, vp]
    lib.tid_last_error.restype = ctypes.c_char_p
    for name in EXPORTS[:-1]:
        getattr(lib, name).restype = ctypes.c_int
    _lib = lib
    return lib


def _check(st: int):
    if st != TID_OK:
        raise TidError(st, _lib.tid_last_error().decode())


# ----------------------------------------------------------------------------- marshalling
def _is_torch(x):
    return type(x).__module__.startswith("torch")


_TORCH_DT = {np.uint8: "torch.uint8", np.int32: "torch.int32", np.int64: "torch.int64", np.uint32: "torch.uint32",
             np.float16: "torch.float16"}


def _ptr(x, dtype=None):
    """(pointer, keepalive) of an INPUT: a numpy array (converted to a C-contiguous copy of
    `dtype` if needed) or a torch tensor (must already be contiguous and of `dtype`); None
    passes NULL."""
    if x is None:
        return None, None
    if _is_torch(x):
        if not x.is_contiguous():
            raise ValueError("tensor must be contiguous")
        if dtype is not None and str(x.dtype) != _TORCH_DT[dtype]:
            raise TypeError(f"tensor dtype {x.dtype}, expected {_TORCH_DT[dtype]}")
        return x.data_ptr(), x
    a = np.ascontiguousarray(x, dtype=dtype)
    return a.ctypes.data, a


def _out_ptr(x, shape, dtype, device: int, what: str):
    """Pointer of a caller-supplied OUTPUT buffer, checked instead of converted (a converted copy
    would silently drop the results; a smaller or narrower buffer would be overrun): exact
    shape and dtype, C-contiguous and writable, and — for a CUDA tensor — on the index's device."""
    shape = tuple(int(v) for v in shape)
    ok_dt = {_TORCH_DT[dtype]} | ({"torch.int32"} if dtype is np.uint32 else set())  # counts: 4-byte ints
    if _is_torch(x):
        if tuple(x.shape) != shape or str(x.dtype) not in ok_dt:
            raise TypeError(f"{what}: got {tuple(x.shape)} {x.dtype}, expected {shape} {_TORCH_DT[dtype]}")
        if not x.is_contiguous():
            raise ValueError(f"{what}: tensor must be contiguous")
        if x.is_cuda and x.device.index != device:
            raise ValueError(f"{what}: tensor on {x.device}, the index is on cuda:{device}")
        return x.data_ptr()
    if not isinstance(x, np.ndarray):
        raise TypeError(f"{what}: expected a numpy array or torch tensor, got {type(x).__name__}")
    if x.shape != shape or (x.dtype != np.dtype(dtype) and not (dtype is np.uint32 and x.dtype == np.int32)):
        raise TypeError(f"{what}: got {x.shape} {x.dtype}, expected {shape} {np.dtype(dtype)}")
    if not x.flags["C_CONTIGUOUS"] or not x.flags["WRITEABLE"]:
        raise ValueError(f"{what}: array must be C-contiguous and writable")
    return x.ctypes.data


def _stream(*tensors):
    for t in tensors:
        if t is not None and _is_torch(t) and t.is_cuda:
            import torch
            return torch.cuda.current_stream(t.device).cuda_stream
    return None


def _shape(x):
    return tuple(x.shape)


def nccl_unique_id() -> bytes:
    lib = load_library()
    buf = ctypes.create_string_buffer(128)
    _check(lib.tid_nccl_unique_id(buf))
    return buf.raw


class Index:
    """A reference index on one GPU (one shard when world_size > 1).  See include/tid.h."""

    def __init__(self, ref_kp: int = 256, query_kp_max: int = 1024, ratio=(4, 5), device: int = 0,
                 hbm_budget_bytes: int = 0, host_budget_bytes: int = 0, id_base: int = 0, rank: int = 0,
                 world_size: int = 1, nccl_id: bytes | None = None, cache_policy: str = "fill",
                 descriptor: str = "u8", f16_scale: float = 1.0, f16_rootsift: bool = True):
        """descriptor "u8": exact integer path; "f16": the float path (RootSIFT / scaled SIFT stored
        in fp16, tcgen05 kind::f16) — add/search still take u8 SIFT, converted on the GPU."""
        self._lib = load_library()
        self._id_buf = ctypes.create_string_buffer(nccl_id, 128) if nccl_id is not None else None
        cfg = Config(device, 128, ref_kp, query_kp_max, ratio[0], ratio[1], hbm_budget_bytes, host_budget_bytes,
                     id_base, rank, world_size,
                     ctypes.cast(self._id_buf, ctypes.c_void_p) if self._id_buf is not None else None,
                     {"fill": 0, "fifo": 1}[cache_policy], {"u8": 0, "f16": 1}[descriptor], f16_scale,
                     1 if f16_rootsift else 0)
        self.descriptor = descriptor
        h = ctypes.c_void_p()
        _check(self._lib.tid_index_create(ctypes.byref(cfg), ctypes.byref(h)))
        self._h = h
        self.ref_kp, self.device, self.world_size = ref_kp, device, world_size

    def close(self):
        if getattr(self, "_h", None) is not None and self._h.value:
            self._lib.tid_index_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    # -------------------------------------------------------------------- API
    def add_references(self, desc, kp_counts=None) -> int:
        """desc: u8 [count][ref_kp][128]; kp_counts: int32 [count] or None.  Returns first local id."""
        count, m, d = _shape(desc)
        assert m == self.ref_kp and d == 128, f"expected [count][{self.ref_kp}][128]"
        dp, k1 = _ptr(desc, np.uint8)
        kp, k2 = _ptr(kp_counts, np.int32)
        first = ctypes.c_int64()
        _check(self._lib.tid_add_references(self._h, dp, kp, count, ctypes.byref(first)))
        return first.value

    def host_tier_map(self, count: int):
        """Zero-copy fill of the pinned host tier: appends `count` references (ref_kp keypoints
        each) and returns (first local id, numpy u8 view [count][ref_kp][128] of their pinned
        storage) to be filled in place before the next search.  The view is valid while the
        index is open."""
        ptr = ctypes.POINTER(ctypes.c_uint8)()
        first = ctypes.c_int64()
        _check(self._lib.tid_host_tier_map(self._h, count, ctypes.byref(ptr), ctypes.byref(first)))
        if self.descriptor == "f16":  # fp16 values [count][ref_kp][128]
            view = np.ctypeslib.as_array(ptr, shape=(count, self.ref_kp, 256)).view(np.float16)
        else:
            view = np.ctypeslib.as_array(ptr, shape=(count, self.ref_kp, 128))
        return first.value, view

    def delete(self, local_ids):
        ids, k1 = _ptr(np.asarray(local_ids, np.int64), np.int64)
        _check(self._lib.tid_delete_references(self._h, ids, len(k1)))

    def update(self, local_ids, desc, kp_counts=None):
        ids, k1 = _ptr(np.asarray(local_ids, np.int64), np.int64)
        dp, k2 = _ptr(desc, np.uint8)
        kp, k3 = _ptr(kp_counts, np.int32)
        _check(self._lib.tid_update_references(self._h, ids, dp, kp, len(k1)))

    def save(self, path: str):
        _check(self._lib.tid_index_save(self._h, os.fsencode(path)))

    def load(self, path: str) -> int:
        first = ctypes.c_int64()
        _check(self._lib.tid_index_load(self._h, os.fsencode(path), ctypes.byref(first)))
        return first.value

    def search(self, queries, k: int, n_q=None, out=None):
        """queries u8 [B][n][128] -> (ids int64 [B][k], counts int32 [B][k]).
        ``out`` = (ids, counts) preallocated (numpy or torch, host or device)."""
        B, n, d = _shape(queries)
        assert d == 128
        qp, k1 = _ptr(queries, np.uint8)
        nqp, k2 = _ptr(n_q, np.int32)
        if out is None:
            ids, cnt = np.empty((B, k), np.int64), np.empty((B, k), np.int32)
        else:
            ids, cnt = out
        ip = _out_ptr(ids, (B, k), np.int64, self.device, "ids")
        cp = _out_ptr(cnt, (B, k), np.int32, self.device, "counts")
        _check(self._lib.tid_search(self._h, qp, nqp, n, B, k, ip, cp, _stream(queries, ids)))
        return ids, cnt

    def search_counts(self, queries, n_q=None, out=None):
        """Full local count matrix uint32 [B][num_local_references]."""
        B, n, d = _shape(queries)
        R = self.info()["num_references"]
        qp, k1 = _ptr(queries, np.uint8)
        nqp, k2 = _ptr(n_q, np.int32)
        if out is None:
            out = np.empty((B, R), np.uint32)
        op = _out_ptr(out, (B, R), np.uint32, self.device, "counts")
        _check(self._lib.tid_search_counts(self._h, qp, nqp, n, B, op, _stream(queries, out)))
        return out

    # ---- f1: float-descriptor path (RootSIFT / scaled SIFT in fp16, tcgen05 kind::f16)
    def f16_prepare(self, sift, rootsift: bool = True, scale: float = 1.0, out=None):
        """u8 SIFT [..., 128] -> fp16 [..., 128] (RootSIFT if asked, times `scale`), on the GPU.
        Returns a numpy float16 array unless ``out`` (float16 numpy / torch, host or device) is given."""
        shp = _shape(sift)
        assert shp[-1] == 128
        rows = int(np.prod(shp[:-1]))
        sp, k1 = _ptr(sift, np.uint8)
        if out is None:
            out = np.empty(shp, np.float16)
        op = _out_ptr(out, shp, np.float16, self.device, "out")
        _check(self._lib.tid_f16_prepare(self._h, sp, rows, 1 if rootsift else 0, float(scale), op,
                                         _stream(sift, out)))
        return out

    def f16_search_counts(self, q16, r16, out=None):
        """fp16 queries [B][n][128] x fp16 references [R][m][128] -> counts uint32 [B][R]."""
        B, n, d = _shape(q16)
        R, m, d2 = _shape(r16)
        assert d == 128 and d2 == 128
        qp, k1 = _ptr(q16, np.float16)
        rp, k2 = _ptr(r16, np.float16)
        if out is None:
            out = np.empty((B, R), np.uint32)
        op = _out_ptr(out, (B, R), np.uint32, self.device, "counts")
        _check(self._lib.tid_f16_search_counts(self._h, qp, n, B, rp, m, R, op, _stream(q16, out)))
        return out

    def verify(self, q, r, n_q=None, m_r=None, want_nn: bool = True, out=None):
        """Pairs q u8 [P][n][128], r u8 [P][m][128] -> (counts uint32 [P], nn int32 [P][n][4] or None)."""
        P, n, _ = _shape(q)
        P2, m, _ = _shape(r)
        assert P == P2
        qp, k1 = _ptr(q, np.uint8)
        rp, k2 = _ptr(r, np.uint8)
        nqp, k3 = _ptr(n_q, np.int32)
        mrp, k4 = _ptr(m_r, np.int32)
        if out is None:
            counts = np.empty(P, np.uint32)
            nn = np.empty((P, n, 4), np.int32) if want_nn else None
        else:
            counts, nn = out
        cp = _out_ptr(counts, (P,), np.uint32, self.device, "counts")
        np_ = None if nn is None else _out_ptr(nn, (P, n, 4), np.int32, self.device, "nn")
        _check(self._lib.tid_verify(self._h, qp, n, rp, m, P, nqp, mrp, cp, np_, _stream(q, r, counts)))
        return counts, nn

    def verify_geometric(self, q, r, q_xy, r_xy, *, border=0.0, query_size=(1e9, 1e9), ref_size=(1e9, 1e9),
                         inlier_px=3.0, iterations=256, seed=2021, n_q=None, m_r=None, want_model=True):
        """Row f4: verify pairs (q, r) like ``verify`` then edge-feature removal + 2-point similarity
        RANSAC on the keypoint coordinates q_xy float [P][n][2], r_xy float [P][m][2].
        Returns (counts, good, inliers) uint32 [P] and the model float64 [P][4] (a, b, tx, ty)."""
        P, n, _ = _shape(q)
        P2, m, _ = _shape(r)
        assert P == P2
        qp, k1 = _ptr(q, np.uint8)
        rp, k2 = _ptr(r, np.uint8)
        nqp, k3 = _ptr(n_q, np.int32)
        mrp, k4 = _ptr(m_r, np.int32)
        qx, k5 = _ptr(q_xy, np.float32)
        rx, k6 = _ptr(r_xy, np.float32)
        if _shape(q_xy) != (P, n, 2) or _shape(r_xy) != (P, m, 2):
            raise ValueError("q_xy must be [P][n][2] and r_xy [P][m][2]")
        gp = GeomParams(border, query_size[0], query_size[1], ref_size[0], ref_size[1], inlier_px, iterations, seed)
        counts, good, inl = np.empty(P, np.uint32), np.empty(P, np.uint32), np.empty(P, np.uint32)
        model = np.empty((P, 4), np.float64) if want_model else None
        _check(self._lib.tid_verify_geometric(self._h, qp, n, rp, m, P, nqp, mrp, qx, rx, ctypes.byref(gp),
                                              counts.ctypes.data, good.ctypes.data, inl.ctypes.data,
                                              None if model is None else model.ctypes.data, _stream(q, r)))
        return counts, good, inl, model

    def merge_topk(self, ids, counts):
        """ids int64 / counts int32 [G][B][k] (each list ranked) -> merged [B][k]."""
        G, B, k = _shape(ids)
        ip, k1 = _ptr(ids, np.int64)
        cp, k2 = _ptr(counts, np.int32)
        io, co = np.empty((B, k), np.int64), np.empty((B, k), np.int32)
        _check(self._lib.tid_merge_topk(self._h, ip, cp, G, B, k, io.ctypes.data, co.ctypes.data, None))
        return io, co

    def info(self) -> dict:
        i = Info()
        _check(self._lib.tid_get_info(self._h, ctypes.byref(i)))
        return {f: getattr(i, f) for f, _ in Info._fields_}

    def profile(self, enable: bool = True):
        _check(self._lib.tid_profile(self._h, 1 if enable else 0))

    def stats(self) -> dict:
        s = Stats()
        _check(self._lib.tid_get_stats(self._h, ctypes.byref(s)))
        return {f: getattr(s, f) for f, _ in Stats._fields_}

    def set_tuning(self, refs_per_job: int = 0, grid: int = 0, host_chunk_refs: int = 0, window_refs: int = 0):
        t = Tuning(refs_per_job, grid, host_chunk_refs, window_refs)
        _check(self._lib.tid_set_tuning(self._h, ctypes.byref(t)))


from .dist import shard_plan  # noqa: E402  (re-export)
