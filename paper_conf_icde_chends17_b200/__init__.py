"""B200-native Sweet KNN exact KNN join -- thin Python binding of libsweetknn.so.

Argument marshalling only: every step of the join runs in the CUDA kernels of
``csrc/`` behind the C ABI declared in ``include/sknn.h``. There is no CPU or
PyTorch fallback: if the library is missing the first call raises.

    import paper_conf_icde_chends17_b200 as sknn
    idx, dist = sknn.join(Q, T, k)            # torch CUDA tensors (or numpy on the host)
    index = sknn.build(T); idx, dist = index.query(Q, k)

Method: Chen, Ding, Shen, "Sweet KNN", ICDE 2017; the names follow
the paper (Q, T, k, clusters, calUB, groupFilter, pointFilter).
"""
from __future__ import annotations

import ctypes
import os
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("SKNN_LIB") or os.path.join(_HERE, "libsweetknn.so")

SKNN_OK = 0
STATUS = {0: "SKNN_OK", -1: "SKNN_ERR_INVALID_ARG", -2: "SKNN_ERR_NOT_DEVICE_PTR", -3: "SKNN_ERR_OOM",
          -4: "SKNN_ERR_CUDA", -5: "SKNN_ERR_UNSUPPORTED", -6: "SKNN_ERR_WRONG_DEVICE"}
PATH = {"auto": 0, "sparse": 1, "dense": 2, "brute": 3, "partial": 4}
MAPPING = {"auto": 0, "thread": 1, "warp": 2, "basic": 3}
MAX_K = 512

# every symbol include/sknn.h declares (tests check the library exports them)
ABI_SYMBOLS = ["sknn_options_default", "sknn_join", "sknn_join_ex", "sknn_build", "sknn_query",
               "sknn_merge_partials", "sknn_merge_partials_ptrs", "sknn_cluster_count", "sknn_build_assign_shard",
               "sknn_build_from_assignment", "sknn_index_free", "sknn_index_info", "sknn_index_export",
               "sknn_debug_level1", "sknn_config_decide", "sknn_error_string", "sknn_last_error",
               "sknn_version", "sknn_index_arrays", "sknn_index_create", "sknn_join_indexed",
               "sknn_level1_bounds"]
INDEX_ARRAYS = ("rows", "dist", "orig", "off", "centers", "radius", "tinfo")


class SknnError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__("%s: %s" % (STATUS.get(status, status), msg))
        self.status = status


class Options(ctypes.Structure):
    _fields_ = [("struct_size", ctypes.c_size_t), ("n_clusters_q", ctypes.c_int32),
                ("n_clusters_t", ctypes.c_int32), ("landmark_trials", ctypes.c_int32),
                ("lloyd_iters", ctypes.c_int32), ("seed", ctypes.c_uint64), ("force_path", ctypes.c_int32),
                ("mapping", ctypes.c_int32), ("dense_threshold", ctypes.c_float), ("r_factor", ctypes.c_float),
                ("out_squared", ctypes.c_int32), ("pad0", ctypes.c_int32), ("index_base", ctypes.c_int64),
                ("shard_rank", ctypes.c_int32), ("shard_count", ctypes.c_int32), ("query_batch", ctypes.c_int64),
                ("self_query", ctypes.c_int32), ("pad1", ctypes.c_int32), ("ub_in", ctypes.c_void_p),
                ("use_graph", ctypes.c_int32), ("shard_policy", ctypes.c_int32)]


class Stats(ctypes.Structure):
    _fields_ = [("struct_size", ctypes.c_size_t), ("pairs_total", ctypes.c_uint64),
                ("dist_evals_sparse", ctypes.c_uint64), ("dist_evals_dense", ctypes.c_uint64),
                ("dist_evals_brute", ctypes.c_uint64), ("center_evals", ctypes.c_uint64),
                ("cand_pairs", ctypes.c_uint64), ("dense_pairs", ctypes.c_uint64),
                ("dist_recompute", ctypes.c_uint64),
                ("ms_total", ctypes.c_float), ("ms_build_t", ctypes.c_float), ("ms_build_q", ctypes.c_float),
                ("ms_level1", ctypes.c_float), ("ms_sparse", ctypes.c_float), ("ms_dense", ctypes.c_float),
                ("ms_final", ctypes.c_float), ("mapping_used", ctypes.c_int32), ("path_used", ctypes.c_int32),
                ("mq", ctypes.c_int32), ("mt", ctypes.c_int32), ("kernel_launches", ctypes.c_int32),
                ("pad0", ctypes.c_int32), ("topk_inserts", ctypes.c_uint64),
                ("rows_loaded", ctypes.c_uint64), ("dense_terms", ctypes.c_uint32), ("pad1", ctypes.c_uint32)]

    def to_dict(self):
        d = {name: getattr(self, name) for name, _ in self._fields_ if name not in ("struct_size", "pad0", "pad1")}
        evals = self.dist_evals_sparse + self.dist_evals_dense + self.dist_evals_brute
        d["dist_evals"] = evals
        d["pruned_pct"] = 100.0 * (self.pairs_total - evals) / self.pairs_total if self.pairs_total else 0.0
        return d


class DeviceProps(ctypes.Structure):
    _fields_ = [("num_sms", ctypes.c_int32), ("max_threads_per_sm", ctypes.c_int32),
                ("smem_per_sm", ctypes.c_int32), ("max_regs_per_thread", ctypes.c_int32)]


class Config(ctypes.Structure):
    _fields_ = [("th1_bytes", ctypes.c_int32), ("th2_bytes", ctypes.c_int32), ("placement", ctypes.c_int32),
                ("partial_filter", ctypes.c_int32), ("r_max_cur", ctypes.c_int64), ("tpq_raw", ctypes.c_double),
                ("threads_per_query", ctypes.c_int32), ("mapping", ctypes.c_int32), ("mq", ctypes.c_int32),
                ("mt", ctypes.c_int32)]

    def to_dict(self):
        return {name: getattr(self, name) for name, _ in self._fields_}


_lib = None
_lock = threading.Lock()

_vp, _i64, _i32 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32


def lib():
    """Load libsweetknn.so (fails loudly when it has not been built)."""
    global _lib
    with _lock:
        if _lib is None:
            if not os.path.exists(LIB_PATH):
                raise RuntimeError("libsweetknn.so not built: run `python -m paper_conf_icde_chends17_b200.buildlib` "
                                   "(or __graft_entry__.build()); there is no CPU fallback")
            L = ctypes.CDLL(LIB_PATH)
            L.sknn_options_default.argtypes = [ctypes.POINTER(Options)]
            L.sknn_options_default.restype = None
            L.sknn_join.argtypes = [_vp, _i64, _vp, _i64, _i32, _i32, _vp, _vp, _vp]
            L.sknn_join_ex.argtypes = [_vp, _i64, _vp, _i64, _i32, _i32, _vp, _vp, ctypes.POINTER(Options),
                                       ctypes.POINTER(Stats), _vp]
            L.sknn_build.argtypes = [_vp, _i64, _i32, ctypes.POINTER(Options), ctypes.POINTER(_vp), _vp]
            L.sknn_query.argtypes = [_vp, _vp, _i64, _i32, _vp, _vp, ctypes.POINTER(Options),
                                     ctypes.POINTER(Stats), _vp]
            L.sknn_merge_partials.argtypes = [_vp, _vp, _i32, _i64, _i32, _vp, _vp, _i32, _vp]
            L.sknn_cluster_count.argtypes = [_i64, ctypes.POINTER(Options)]
            L.sknn_cluster_count.restype = _i32
            L.sknn_build_assign_shard.argtypes = [_vp, _i64, _i32, ctypes.POINTER(Options), _i64, _i64, _vp, _vp, _vp,
                                                  _vp]
            L.sknn_build_from_assignment.argtypes = [_vp, _i64, _i32, ctypes.POINTER(Options), _vp, _i32, _vp, _vp,
                                                     ctypes.POINTER(_vp), _vp]
            L.sknn_merge_partials_ptrs.argtypes = [ctypes.POINTER(_vp), ctypes.POINTER(_vp), _i32, _i64, _i64, _i64,
                                                   _i32, _vp, _vp, _i32, _vp]
            L.sknn_index_free.argtypes = [_vp]
            L.sknn_index_info.argtypes = [_vp, ctypes.POINTER(_i64), ctypes.POINTER(_i32), ctypes.POINTER(_i32),
                                          ctypes.POINTER(_i32), ctypes.POINTER(_i32)]
            L.sknn_index_export.argtypes = [_vp, _vp, _vp, _vp, _vp, _vp]
            L.sknn_debug_level1.argtypes = [_vp, _vp, _i64, _i32, ctypes.POINTER(Options), ctypes.POINTER(_i32),
                                            _vp, _vp, _vp, _vp, _i64]
            L.sknn_config_decide.argtypes = [_i64, _i64, _i32, _i32, ctypes.POINTER(DeviceProps), ctypes.c_float,
                                             ctypes.POINTER(Config)]
            L.sknn_error_string.argtypes = [_i32]
            L.sknn_error_string.restype = ctypes.c_char_p
            L.sknn_last_error.restype = ctypes.c_char_p
            L.sknn_version.restype = _i32
            L.sknn_index_arrays.argtypes = [_vp, ctypes.POINTER(_vp), ctypes.POINTER(ctypes.c_size_t)]
            L.sknn_join_indexed.argtypes = [_vp, _vp, _i32, _vp, _vp, ctypes.POINTER(Options),
                                            ctypes.POINTER(Stats), _vp]
            L.sknn_level1_bounds.argtypes = [_vp, _vp, _i32, ctypes.POINTER(Options), _vp, _vp]
            L.sknn_index_create.argtypes = [_i64, _i32, _i32, ctypes.POINTER(Options), ctypes.POINTER(_vp)]
            for fn in ("sknn_join", "sknn_join_ex", "sknn_build", "sknn_query", "sknn_merge_partials",
                       "sknn_index_free", "sknn_index_info", "sknn_index_export", "sknn_debug_level1",
                       "sknn_config_decide", "sknn_index_arrays", "sknn_index_create", "sknn_join_indexed",
                       "sknn_level1_bounds"):
                getattr(L, fn).restype = _i32
            _lib = L
    return _lib


def _check(st):
    if st != SKNN_OK:
        raise SknnError(st, lib().sknn_last_error().decode(errors="replace"))


def make_options(**kw) -> Options:
    o = Options()
    lib().sknn_options_default(ctypes.byref(o))
    for key, val in kw.items():
        if val is None:
            continue
        if key == "force_path" and isinstance(val, str):
            val = PATH[val]
        if key == "mapping" and isinstance(val, str):
            val = MAPPING[val]
        if key == "ub_in" and hasattr(val, "data_ptr"):  # a CUDA float32 tensor [mq]
            val = val.data_ptr()
        if not hasattr(o, key):
            raise TypeError("unknown option %r" % key)
        setattr(o, key, val)
    return o


def _stream_ptr(stream, device=None):
    """The stream to enqueue on: `stream`, else torch's current stream of the
    tensors' device (not of the current device: ADVICE r1)."""
    if stream is None:
        import torch
        if torch.cuda.is_available():
            return torch.cuda.current_stream(device).cuda_stream
        return None
    return getattr(stream, "cuda_stream", stream)


class _on_device:
    """Make the tensors' CUDA device current for the C call (the library checks
    pointers against cudaGetDevice()); a no-op for host arrays."""

    def __init__(self, device):
        self.device = device
        self._ctx = None

    def __enter__(self):
        if self.device is not None and getattr(self.device, "type", None) == "cuda":
            import torch
            self._ctx = torch.cuda.device(self.device)
            self._ctx.__enter__()
        return self

    def __exit__(self, *exc):
        if self._ctx is not None:
            self._ctx.__exit__(*exc)
        return False


def _as_points(X):
    """Return (pointer, n, d, keepalive, is_torch_cuda) for a [n, d] fp32 array."""
    try:
        import torch
        if isinstance(X, torch.Tensor):
            if X.dtype != torch.float32 or X.dim() != 2:
                raise ValueError("points must be a 2-D float32 tensor")
            X = X.contiguous()
            return X.data_ptr(), X.shape[0], X.shape[1], X, X.is_cuda
    except ImportError:
        pass
    X = np.ascontiguousarray(X, dtype=np.float32)
    if X.ndim != 2:
        raise ValueError("points must be [n, d]")
    return X.ctypes.data, X.shape[0], X.shape[1], X, False


def _alloc_out(nq, k, on_cuda, device=None):
    if on_cuda:
        import torch
        idx = torch.empty((nq, k), dtype=torch.int32, device=device)
        dist = torch.empty((nq, k), dtype=torch.float32, device=device)
        return idx, dist, idx.data_ptr(), dist.data_ptr()
    idx = np.empty((nq, k), dtype=np.int32)
    dist = np.empty((nq, k), dtype=np.float32)
    return idx, dist, idx.ctypes.data, dist.ctypes.data


def join(Q, T, k: int, *, stream=None, stats: bool = False, with_index: bool = True, out=None, **opts):
    """Exact KNN join (sknn_join_ex). Q: [nq, d], T: [nt, d] float32, torch CUDA
    tensors (stream-ordered, no host sync) or host arrays (staged, synchronous).
    Passing the same object for Q and T runs a self-join. Returns (idx, dist)
    [nq, k] (idx None when with_index=False) and a stats dict when stats=True."""
    qp, nq, d, qkeep, qcuda = _as_points(Q)
    if T is Q:
        tp, nt, dt, tkeep, tcuda = qp, nq, d, qkeep, qcuda
    else:
        tp, nt, dt, tkeep, tcuda = _as_points(T)
    if d != dt:
        raise ValueError("Q and T dimensions differ")
    if out is not None:
        idx, dist = out
        ip = idx.data_ptr() if hasattr(idx, "data_ptr") else (idx.ctypes.data if idx is not None else None)
        dp_ = dist.data_ptr() if hasattr(dist, "data_ptr") else dist.ctypes.data
    else:
        idx, dist, ip, dp_ = _alloc_out(nq, k, qcuda, qkeep.device if qcuda else None)
    if not with_index:
        idx, ip = None, None
    o = make_options(**opts)
    st = Stats()
    st.struct_size = ctypes.sizeof(Stats)
    qdev = qkeep.device if qcuda else None
    with _on_device(qdev):
        _check(lib().sknn_join_ex(qp, nq, tp, nt, d, k, ip, dp_, ctypes.byref(o),
                                  ctypes.byref(st) if stats else None, _stream_ptr(stream, qdev) if qcuda else None))
    if stats:
        return idx, dist, st.to_dict()
    return idx, dist


class Index:
    """Resident target index (sknn_build / sknn_query)."""

    def __init__(self, T, stream=None, **opts):
        tp, nt, d, keep, cuda = _as_points(T)
        self._keep = keep  # the index remembers T's pointer for self-join detection
        self._handle = ctypes.c_void_p()
        o = make_options(**opts)
        tdev = keep.device if cuda else None
        with _on_device(tdev):
            _check(lib().sknn_build(tp, nt, d, ctypes.byref(o), ctypes.byref(self._handle),
                                    _stream_ptr(stream, tdev) if cuda else None))
        self.nt, self.d = nt, d

    @classmethod
    def from_assignment(cls, T, centers, cid, dist, stream=None, **opts):
        """The index sknn_build would return, from a given clustering: centers
        [m, dp] fp32, cid [n] int32, dist [n] fp32 member distances, all CUDA
        (sknn_build_from_assignment; the sharded build of dist.py)."""
        tp, nt, d, keep, cuda = _as_points(T)
        self = cls.__new__(cls)
        self._keep = keep
        self._handle = ctypes.c_void_p()
        o = make_options(**opts)
        with _on_device(keep.device):
            _check(lib().sknn_build_from_assignment(tp, nt, d, ctypes.byref(o), centers.data_ptr(), centers.shape[0],
                                                    cid.data_ptr(), dist.data_ptr(), ctypes.byref(self._handle),
                                                    _stream_ptr(stream, keep.device)))
        self.nt, self.d = nt, d
        return self

    @classmethod
    def create(cls, nt: int, d: int, mt: int, **opts):
        """An index of this geometry with uninitialised device arrays (to be
        filled, e.g. by a broadcast of another rank's index: dist.py)."""
        self = cls.__new__(cls)
        self._keep = None
        self._handle = ctypes.c_void_p()
        o = make_options(**opts)
        _check(lib().sknn_index_create(nt, d, mt, ctypes.byref(o), ctypes.byref(self._handle)))
        self.nt, self.d = nt, d
        return self

    def arrays(self):
        """The index's device arrays as torch uint8 tensors (views, no copy),
        in INDEX_ARRAYS order."""
        import torch
        ptr = (_vp * len(INDEX_ARRAYS))()
        nb = (ctypes.c_size_t * len(INDEX_ARRAYS))()
        _check(lib().sknn_index_arrays(self._handle, ptr, nb))
        dev = torch.cuda.current_device()
        out = []
        for i in range(len(INDEX_ARRAYS)):
            out.append(_device_bytes(ptr[i], nb[i], dev, owner=self))
        return out

    def info(self):
        nt, d, dp, mt, dev = _i64(), _i32(), _i32(), _i32(), _i32()
        _check(lib().sknn_index_info(self._handle, ctypes.byref(nt), ctypes.byref(d), ctypes.byref(dp),
                                     ctypes.byref(mt), ctypes.byref(dev)))
        return dict(nt=nt.value, d=d.value, dp=dp.value, mt=mt.value, device=dev.value)

    def export(self):
        inf = self.info()
        off = np.empty(inf["mt"] + 1, np.int32)
        orig = np.empty(inf["nt"], np.int32)
        dist = np.empty(inf["nt"], np.float32)
        cent = np.empty((inf["mt"], inf["dp"]), np.float32)
        rad = np.empty(inf["mt"], np.float32)
        _check(lib().sknn_index_export(self._handle, off.ctypes.data, orig.ctypes.data, dist.ctypes.data,
                                       cent.ctypes.data, rad.ctypes.data))
        return dict(off=off, orig=orig, dist=dist, centers=cent, radius=rad)

    def query(self, Q, k: int, *, stream=None, stats: bool = False, with_index: bool = True, out=None, **opts):
        qp, nq, d, qkeep, qcuda = _as_points(Q)
        if d != self.d:
            raise ValueError("query dimension differs from the index")
        if out is not None:
            idx, dist = out
            ip = idx.data_ptr() if hasattr(idx, "data_ptr") else idx.ctypes.data
            dp_ = dist.data_ptr() if hasattr(dist, "data_ptr") else dist.ctypes.data
        else:
            idx, dist, ip, dp_ = _alloc_out(nq, k, qcuda, qkeep.device if qcuda else None)
        if not with_index:
            idx, ip = None, None
        o = make_options(**opts) if opts else None
        st = Stats()
        st.struct_size = ctypes.sizeof(Stats)
        qdev = qkeep.device if qcuda else None
        with _on_device(qdev):
            _check(lib().sknn_query(self._handle, qp, nq, k, ip, dp_, ctypes.byref(o) if o is not None else None,
                                    ctypes.byref(st) if stats else None, _stream_ptr(stream, qdev) if qcuda else None))
        if stats:
            return idx, dist, st.to_dict()
        return idx, dist

    def debug_level1(self, Q, k: int, **opts):
        qp, nq, d, qkeep, _ = _as_points(Q)
        inf = self.info()
        mq_cap = min(nq, 16384)
        qcl = np.empty(nq, np.int32)
        ub = np.empty(mq_cap, np.float32)
        cc = np.empty(mq_cap, np.int32)
        cand = np.empty(mq_cap * inf["mt"], np.int32)
        mq = _i32()
        o = make_options(**opts) if opts else None
        _check(lib().sknn_debug_level1(self._handle, qp, nq, k, ctypes.byref(o) if o is not None else None,
                                       ctypes.byref(mq), qcl.ctypes.data, ub.ctypes.data, cc.ctypes.data,
                                       cand.ctypes.data, cand.size))
        m = mq.value
        return dict(mq=m, q_cluster=qcl, ub=ub[:m], cand_count=cc[:m], cand=cand[: m * inf["mt"]].reshape(m, inf["mt"]))

    def close(self):
        if getattr(self, "_handle", None) is not None and self._handle.value:
            lib().sknn_index_free(self._handle)
            self._handle = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class _DevBuf:
    """__cuda_array_interface__ view of library-owned device bytes."""

    def __init__(self, ptr, nbytes, owner):
        self.__cuda_array_interface__ = {"shape": (int(nbytes),), "typestr": "|u1", "data": (int(ptr), False),
                                         "version": 3, "strides": None, "stream": None}
        self._owner = owner


def _device_bytes(ptr, nbytes, device, owner):
    import torch
    return torch.as_tensor(_DevBuf(ptr, nbytes, owner), device=torch.device("cuda", device))


def build(T, **opts) -> Index:
    return Index(T, **opts)


def join_indexed(qindex: Index, tindex: Index, k: int, *, stream=None, stats: bool = False, out=None, **opts):
    """The query index's points against the target index (sknn_join_indexed):
    (idx, dist) [nq, k] on the device, rows in the query set's original order."""
    import torch
    nq = qindex.nt
    dev = torch.device("cuda", torch.cuda.current_device())
    if out is not None:
        idx, dist = out
    else:
        idx = torch.empty((nq, k), dtype=torch.int32, device=dev)
        dist = torch.empty((nq, k), dtype=torch.float32, device=dev)
    o = make_options(**opts)
    st = Stats()
    st.struct_size = ctypes.sizeof(Stats)
    _check(lib().sknn_join_indexed(qindex._handle, tindex._handle, k, idx.data_ptr() if idx is not None else None,
                                   dist.data_ptr(), ctypes.byref(o), ctypes.byref(st) if stats else None,
                                   _stream_ptr(stream, dev)))
    if stats:
        return idx, dist, st.to_dict()
    return idx, dist


def level1_bounds(qindex: Index, tindex: Index, k: int, *, stream=None, **opts):
    """Level-1 calUB of every query cluster of qindex against tindex
    (sknn_level1_bounds): a CUDA float32 tensor [mq]."""
    import torch
    dev = torch.device("cuda", torch.cuda.current_device())
    ub = torch.empty(qindex.info()["mt"], dtype=torch.float32, device=dev)
    o = make_options(**opts)
    _check(lib().sknn_level1_bounds(qindex._handle, tindex._handle, k, ctypes.byref(o), ub.data_ptr(),
                                    _stream_ptr(stream, dev)))
    return ub


def merge_partials(part_idx, part_d2, k: int, *, out_squared: bool = False, stream=None, out=None):
    """Merge [P, nq, k] sorted partial lists (torch CUDA int32 / fp32 squared
    distances, global indices) into the k nearest per query (sknn_merge_partials)."""
    import torch
    P, nq, kk = part_d2.shape
    assert kk == k and part_idx.shape == part_d2.shape
    part_idx = part_idx.contiguous()
    part_d2 = part_d2.contiguous()
    if out is not None:
        idx, dist = out
    else:
        idx = torch.empty((nq, k), dtype=torch.int32, device=part_d2.device)
        dist = torch.empty((nq, k), dtype=torch.float32, device=part_d2.device)
    with _on_device(part_d2.device):
        _check(lib().sknn_merge_partials(part_idx.data_ptr(), part_d2.data_ptr(), P, nq, k,
                                         idx.data_ptr() if idx is not None else None, dist.data_ptr(),
                                         int(out_squared), _stream_ptr(stream, part_d2.device)))
    return idx, dist


def merge_partials_ptrs(idx_ptrs, d2_ptrs, nq_total: int, row_lo: int, nrows: int, k: int, *,
                        out_squared: bool = False, stream=None, out=None, device=None):
    """Merge the rows [row_lo, row_lo + nrows) of P partial-list buffers given
    as device addresses (sknn_merge_partials_ptrs: e.g. symmetric-memory peer
    buffers, each [nq_total, k] int32 indices / fp32 squared distances)."""
    import torch
    P = len(d2_ptrs)
    assert len(idx_ptrs) == P
    dev = torch.device(device) if device is not None else torch.device("cuda", torch.cuda.current_device())
    if out is not None:
        idx, dist = out
    else:
        idx = torch.empty((nrows, k), dtype=torch.int32, device=dev)
        dist = torch.empty((nrows, k), dtype=torch.float32, device=dev)
    ip = (_vp * P)(*[int(x) for x in idx_ptrs])
    dp_ = (_vp * P)(*[int(x) for x in d2_ptrs])
    with _on_device(dev):
        _check(lib().sknn_merge_partials_ptrs(ip, dp_, P, nq_total, row_lo, nrows, k,
                                              idx.data_ptr() if idx is not None else None, dist.data_ptr(),
                                              int(out_squared), _stream_ptr(stream, dev)))
    return idx, dist


def cluster_count(n: int, **opts) -> int:
    """m = the cluster count sknn_build uses for n points (sknn_cluster_count)."""
    o = make_options(**opts)
    return int(lib().sknn_cluster_count(n, ctypes.byref(o)))


def build_assign_shard(T, row_lo: int, row_hi: int, *, out=None, stream=None, **opts):
    """Seeding + Lloyd over all of T and the final assignment of rows
    [row_lo, row_hi) (sknn_build_assign_shard). Returns (centers [m, dp],
    cid [n], dist [n]); rows outside the range are left as given in `out`
    (zeros when allocated here)."""
    import torch
    tp, nt, d, keep, cuda = _as_points(T)
    m = cluster_count(nt, **opts)
    dp = (d + 3) & ~3
    if out is None:
        centers = torch.empty((m, dp), dtype=torch.float32, device=keep.device)
        cid = torch.zeros(nt, dtype=torch.int32, device=keep.device)
        dist = torch.zeros(nt, dtype=torch.float32, device=keep.device)
    else:
        centers, cid, dist = out
    o = make_options(**opts)
    with _on_device(keep.device):
        _check(lib().sknn_build_assign_shard(tp, nt, d, ctypes.byref(o), row_lo, row_hi, centers.data_ptr(),
                                             cid.data_ptr(), dist.data_ptr(), _stream_ptr(stream, keep.device)))
    return centers, cid, dist


def config_decide(nq: int, nt: int, d: int, k: int, props: dict | None = None, r_factor: float = 0.25) -> dict:
    """The adaptive-scheme decisions (Fig. 8) the library takes; pure host arithmetic."""
    c = Config()
    p = None
    if props is not None:
        p = DeviceProps(props["num_sms"], props["max_threads_per_sm"], props["smem_per_sm"],
                        props["max_regs_per_thread"])
    _check(lib().sknn_config_decide(nq, nt, d, k, ctypes.byref(p) if p is not None else None, r_factor,
                                    ctypes.byref(c)))
    return c.to_dict()


def version() -> tuple:
    v = lib().sknn_version()
    return (v >> 16, v & 0xFFFF)
