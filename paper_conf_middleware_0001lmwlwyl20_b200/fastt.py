"""Thin ctypes binding of ``libfastt.so`` (include/fastt.h).

Argument marshalling only: every step of the method runs in the library's
CUDA kernels.  The binding fails loudly when the library is missing or was
built without a device; there is no CPU fallback.  Names mirror the C-ABI.

Arrays: numpy arrays are host buffers; torch CUDA tensors are device buffers
(then FASTT_F_IN_DEVICE / FASTT_F_OUT_DEVICE are set for you).
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("FASTT_LIB") or os.path.join(_HERE, "libfastt.so")

OK, EINVAL, ECYCLE, ENOMEM, ECUDA, ERANGE, EUNSUP = 0, -1, -2, -3, -4, -5, -6
CAND_OK, CAND_INFEASIBLE, CAND_BADSPEC = 0, 1, 2
KIND_BASE, KIND_PIN, KIND_SPLIT = 0, 1, 2
DIM_BATCH, DIM_CHANNEL = 0, 1
F_CP_PIN, F_POLICY_INSERT, F_OUT_DEVICE, F_IN_DEVICE = 1, 2, 4, 8
INT64_MAX = np.iinfo(np.int64).max

CANDIDATE_DTYPE = np.dtype(
    [("kind", "u1"), ("n_pins", "u1"), ("split_dim", "u1"), ("split_n", "u1"),
     ("split_op", "<i4"), ("pin_op", "<i4", (4,)), ("pin_dev", "u1", (4,)), ("dev_mask", "<u4")]
)
assert CANDIDATE_DTYPE.itemsize == 32


class fastt_graph_desc(C.Structure):
    _fields_ = [("n_ops", C.c_int32), ("n_devices", C.c_int32),
                ("succ_off", C.c_void_p), ("succ_dst", C.c_void_p), ("edge_bytes", C.c_void_p),
                ("edge_param", C.c_void_p), ("cost_ns", C.c_void_p), ("mem_bytes", C.c_void_p),
                ("param_bytes", C.c_void_p), ("split_mask", C.c_void_p), ("dev_mem_cap", C.c_void_p),
                ("link_class", C.c_void_p), ("n_link_classes", C.c_int32),
                ("link_alpha_ns", C.c_void_p), ("link_beta_fs_per_byte", C.c_void_p),
                ("split_copy_fs_per_byte", C.c_int64)]


class fastt_gen_params(C.Structure):
    _fields_ = [("seed", C.c_uint64), ("pin_k_min", C.c_uint8), ("pin_k_max", C.c_uint8),
                ("n_pow2_only", C.c_uint8), ("subset_prefixes", C.c_uint8), ("_pad", C.c_uint8 * 4)]


class fastt_opts(C.Structure):
    _fields_ = [("flags", C.c_uint32), ("_pad", C.c_int32), ("cuda_stream", C.c_void_p)]


class fastt_split_result(C.Structure):
    _fields_ = [("n_splits", C.c_int32), ("op", C.POINTER(C.c_int32)), ("dim", C.POINTER(C.c_uint8)),
                ("n", C.POINTER(C.c_uint8)), ("n_ops_final", C.c_int32), ("placement", C.POINTER(C.c_uint8)),
                ("order", C.POINTER(C.c_int32)), ("start_ns", C.POINTER(C.c_int64)), ("makespan", C.c_int64),
                ("status", C.c_uint8)]


class fastt_timing(C.Structure):
    _fields_ = [("launches", C.c_int64), ("candidates", C.c_int64), ("deferred", C.c_int64),
                ("ms_sim", C.c_float), ("ms_prep", C.c_float), ("ms_total", C.c_float), ("topo", C.c_int32),
                ("_pad", C.c_int32), ("warp_steps", C.c_int64), ("lane_steps", C.c_int64)]


SYMBOLS = ["fastt_load_graph", "fastt_free_graph", "fastt_graph_info", "fastt_rank", "fastt_schedule_batch",
           "fastt_stream_info", "fastt_generate_candidates", "fastt_sweep_best", "fastt_split_search",
           "fastt_free_split_result", "fastt_last_timing", "fastt_last_error", "fastt_version",
           "fastt_fit_comm", "fastt_link_model", "fastt_cost_table", "fastt_sync"]
F_TIMING = 16
F_SPLIT_BEST = 32
F_MEM_LIVE = 64
F_SPLIT_MULTI = 128
F_ASYNC = 256  # return once enqueued on the stream; Graph.sync() (or the stream) completes it

_lib = None


def lib():
    """Load libfastt.so (raises if it is missing: no fallback)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise RuntimeError("libfastt.so not built: run __graft_entry__.build() (no CPU fallback exists)")
    L = C.CDLL(LIB_PATH)
    P, i32, i64 = C.c_void_p, C.c_int32, C.c_int64
    L.fastt_load_graph.restype = i32
    L.fastt_load_graph.argtypes = [C.POINTER(fastt_graph_desc), C.c_int, C.POINTER(P)]
    L.fastt_free_graph.argtypes = [P]
    L.fastt_graph_info.restype = i32
    L.fastt_graph_info.argtypes = [P, P, P, P, P]
    L.fastt_rank.restype = i32
    L.fastt_rank.argtypes = [P, P, C.POINTER(fastt_opts), P]
    L.fastt_schedule_batch.restype = i32
    L.fastt_schedule_batch.argtypes = [P, P, i64, C.POINTER(fastt_opts), P, P, P, P, P, P]
    L.fastt_stream_info.restype = i32
    L.fastt_stream_info.argtypes = [P, C.POINTER(fastt_gen_params), C.POINTER(fastt_opts), P]
    L.fastt_generate_candidates.restype = i32
    L.fastt_generate_candidates.argtypes = [P, C.POINTER(fastt_gen_params), C.POINTER(fastt_opts), i64, i64, P]
    L.fastt_sweep_best.restype = i32
    L.fastt_sweep_best.argtypes = [P, C.POINTER(fastt_gen_params), C.POINTER(fastt_opts), i64, i64, i64, P]
    L.fastt_split_search.restype = i32
    L.fastt_split_search.argtypes = [P, C.POINTER(fastt_opts), i32, C.POINTER(fastt_split_result)]
    L.fastt_free_split_result.argtypes = [C.POINTER(fastt_split_result)]
    L.fastt_last_timing.restype = i32
    L.fastt_last_timing.argtypes = [P, C.POINTER(fastt_timing)]
    L.fastt_last_error.restype = C.c_char_p
    L.fastt_version.restype = C.c_char_p
    L.fastt_fit_comm.restype = i32
    L.fastt_fit_comm.argtypes = [i32, i64, P, P, P, P, C.c_int, C.POINTER(fastt_opts), P, P, P]
    L.fastt_link_model.restype = i32
    L.fastt_link_model.argtypes = [i32, P, P, P, P, P, P]
    L.fastt_cost_table.restype = i32
    L.fastt_cost_table.argtypes = [i32, i32, i64, P, P, P, C.c_int, C.POINTER(fastt_opts), P]
    L.fastt_sync.restype = i32
    L.fastt_sync.argtypes = [P, C.POINTER(fastt_opts)]
    _lib = L
    return L


class FasttError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__("fastt status %d: %s" % (code, msg))
        self.code = code


def _check(rc):
    if rc != 0:
        raise FasttError(rc, lib().fastt_last_error().decode(errors="replace"))


def _ptr(a):
    """numpy array -> host pointer; torch tensor -> its data pointer."""
    if a is None:
        return None
    if isinstance(a, np.ndarray):
        return a.ctypes.data_as(C.c_void_p)
    return C.c_void_p(int(a.data_ptr()))


def _is_dev(a):
    return a is not None and not isinstance(a, np.ndarray) and getattr(a, "is_cuda", False)


def _opts(flags=0, stream=None):
    o = fastt_opts()
    o.flags = int(flags)
    if stream is None:
        o.cuda_stream = None
    elif isinstance(stream, int):
        o.cuda_stream = stream
    else:
        o.cuda_stream = int(stream.cuda_stream)
    return o


def gen_params(seed, pin_k_min=1, pin_k_max=4, n_pow2_only=False, subset_prefixes=False):
    g = fastt_gen_params()
    g.seed = int(seed) & 0xFFFFFFFFFFFFFFFF
    g.pin_k_min = pin_k_min
    g.pin_k_max = pin_k_max
    g.n_pow2_only = 1 if n_pow2_only else 0
    g.subset_prefixes = 1 if subset_prefixes else 0
    return g


def make_candidate(kind=KIND_BASE, pins=(), split=None, dev_mask=0):
    c = np.zeros(1, CANDIDATE_DTYPE)[0]
    c["kind"] = kind
    c["split_op"] = -1
    c["pin_op"] = [-1, -1, -1, -1]
    for q, (o, d) in enumerate(pins):
        c["pin_op"][q] = o
        c["pin_dev"][q] = d
    c["n_pins"] = len(pins)
    if split is not None:
        c["split_op"], c["split_dim"], c["split_n"] = split
    c["dev_mask"] = dev_mask
    return c


class Graph:
    """fastt_load_graph(desc, cuda_device) -- desc is a synth.GraphDesc (or any
    object with the same arrays: an edge list + per-op tables)."""

    def __init__(self, desc, device=0):
        L = lib()
        V = int(desc.n_ops)
        src = np.asarray(desc.src, np.int64)
        order = np.argsort(src, kind="stable")
        counts = np.bincount(src, minlength=V) if len(src) else np.zeros(V, np.int64)
        off = np.zeros(V + 1, np.int32)
        off[1:] = np.cumsum(counts)
        keep = [off,
                np.ascontiguousarray(np.asarray(desc.dst, np.int32)[order]),
                np.ascontiguousarray(np.asarray(desc.bytes, np.int64)[order]),
                np.ascontiguousarray(np.asarray(desc.eparam, np.uint8)[order]),
                np.ascontiguousarray(np.asarray(desc.cost, np.int64).reshape(-1)),
                np.ascontiguousarray(np.asarray(desc.mem, np.int64)),
                np.ascontiguousarray(np.asarray(desc.param, np.int64)),
                np.ascontiguousarray(np.asarray(desc.split_mask, np.uint8)),
                np.ascontiguousarray(np.asarray(desc.cap, np.int64)),
                np.ascontiguousarray(np.asarray(desc.link_class, np.uint8).reshape(-1)),
                np.ascontiguousarray(np.asarray(desc.alpha, np.int64)),
                np.ascontiguousarray(np.asarray(desc.beta, np.int64))]
        d = fastt_graph_desc()
        d.n_ops = V
        d.n_devices = int(desc.n_devices)
        (d.succ_off, d.succ_dst, d.edge_bytes, d.edge_param, d.cost_ns, d.mem_bytes, d.param_bytes, d.split_mask,
         d.dev_mem_cap, d.link_class) = [a.ctypes.data for a in keep[:10]]
        d.n_link_classes = int(len(keep[10]))
        d.link_alpha_ns = keep[10].ctypes.data
        d.link_beta_fs_per_byte = keep[11].ctypes.data
        d.split_copy_fs_per_byte = int(desc.copy_fs)
        h = C.c_void_p()
        _check(L.fastt_load_graph(C.byref(d), int(device), C.byref(h)))
        self.h = h
        self.device = int(device)
        self.G = int(desc.n_devices)
        info = self.info()
        self.V, self.v_max, self.cp_len, self.time_bits = info

    def __del__(self):
        if getattr(self, "h", None) and _lib is not None:
            _lib.fastt_free_graph(self.h)
            self.h = None

    def info(self):
        a = [C.c_int32() for _ in range(4)]
        _check(lib().fastt_graph_info(self.h, *[C.byref(x) for x in a]))
        return tuple(int(x.value) for x in a)

    def rank(self, cand=None, flags=0, stream=None):
        out = np.zeros(self.v_max, np.int64)
        cp = None
        if cand is not None:
            ca = np.ascontiguousarray(np.asarray(cand, CANDIDATE_DTYPE).reshape(1))
            cp = ca.ctypes.data_as(C.c_void_p)
        o = _opts(flags, stream)
        _check(lib().fastt_rank(self.h, cp, C.byref(o), _ptr(out)))
        return out

    def schedule_batch(self, cands, flags=0, stream=None, peak=True, placement=False, order=False, start=False,
                       out=None):
        """DPOS of a batch.  cands: numpy structured array (host) or a torch
        CUDA uint8 tensor [n, 32] (device).  Returns a dict of outputs (numpy
        unless `out` supplies torch CUDA tensors)."""
        n = int(len(cands))
        fl = int(flags)
        if _is_dev(cands):
            fl |= F_IN_DEVICE
            cptr = _ptr(cands)
        else:
            cands = np.ascontiguousarray(np.asarray(cands, CANDIDATE_DTYPE))
            cptr = _ptr(cands)
        res = out
        if res is None:
            res = {"makespan": np.zeros(n, np.int64), "status": np.zeros(n, np.uint8)}
            if peak:
                res["peak_mem"] = np.zeros(n * self.G, np.int64)
            if placement:
                res["placement"] = np.zeros(n * self.v_max, np.uint8)
            if order:
                res["order"] = np.zeros(n * self.v_max, np.int32)
            if start:
                res["start"] = np.zeros(n * self.v_max, np.int64)
        if _is_dev(res["makespan"]):
            fl |= F_OUT_DEVICE
        o = _opts(fl, stream)
        _check(lib().fastt_schedule_batch(self.h, cptr, n, C.byref(o), _ptr(res["makespan"]), _ptr(res.get("peak_mem")),
                                          _ptr(res["status"]), _ptr(res.get("placement")), _ptr(res.get("order")),
                                          _ptr(res.get("start"))))
        if out is None:
            for k in ("placement", "order", "start"):
                if k in res:
                    res[k] = res[k].reshape(n, self.v_max)
            if "peak_mem" in res:
                res["peak_mem"] = res["peak_mem"].reshape(n, self.G)
        return res

    def stream_info(self, gen, flags=0, stream=None):
        ns = C.c_int64()
        o = _opts(flags, stream)
        _check(lib().fastt_stream_info(self.h, C.byref(gen), C.byref(o), C.byref(ns)))
        return int(ns.value)

    def generate_candidates(self, gen, first, n, flags=0, stream=None, out=None):
        """The stream's candidates [first, first + n): numpy records, or into
        `out` (a torch CUDA uint8 tensor [n, 32]) on the device."""
        fl = int(flags)
        if out is None:
            out = np.zeros(n, CANDIDATE_DTYPE)
        elif _is_dev(out):
            fl |= F_OUT_DEVICE
        o = _opts(fl, stream)
        _check(lib().fastt_generate_candidates(self.h, C.byref(gen), C.byref(o), int(first), int(n), _ptr(out)))
        return out

    def sync(self, stream=None):
        """fastt_sync: completes every asynchronous call on this graph and
        reports a deferred device-side error."""
        o = _opts(0, stream)
        _check(lib().fastt_sync(self.h, C.byref(o)))

    def sweep_best(self, gen, first, n, stride=1, flags=0, stream=None, out=None):
        """Returns (best makespan, best index); with `out` (a torch CUDA int64
        tensor of 2) the result stays on the device."""
        fl = int(flags)
        buf = out if out is not None else np.zeros(2, np.int64)
        if _is_dev(buf):
            fl |= F_OUT_DEVICE
        o = _opts(fl, stream)
        _check(lib().fastt_sweep_best(self.h, C.byref(gen), C.byref(o), int(first), int(n), int(stride), _ptr(buf)))
        if out is not None:
            return out
        return int(buf[0]), int(buf[1])

    def last_timing(self):
        t = fastt_timing()
        _check(lib().fastt_last_timing(self.h, C.byref(t)))
        return {"launches": int(t.launches), "candidates": int(t.candidates), "deferred": int(t.deferred),
                "ms_sim": float(t.ms_sim), "ms_prep": float(t.ms_prep), "ms_total": float(t.ms_total),
                "topo": int(t.topo), "warp_steps": int(t.warp_steps), "lane_steps": int(t.lane_steps)}

    def split_search(self, flags=0, n_pow2_only=False, stream=None, best_improvement=False, multi=False):
        r = fastt_split_result()
        o = _opts(flags | (F_SPLIT_BEST if best_improvement else 0) | (F_SPLIT_MULTI if multi else 0), stream)
        _check(lib().fastt_split_search(self.h, C.byref(o), 1 if n_pow2_only else 0, C.byref(r)))
        try:
            n = r.n_splits
            nf = r.n_ops_final
            res = {"sp": [(int(r.op[q]), int(r.dim[q]), int(r.n[q])) for q in range(n)], "n_ops_final": nf,
                   "placement": np.ctypeslib.as_array(r.placement, (nf,)).copy() if nf else np.zeros(0, np.uint8),
                   "order": np.ctypeslib.as_array(r.order, (nf,)).copy() if nf else np.zeros(0, np.int32),
                   "start": np.ctypeslib.as_array(r.start_ns, (nf,)).copy() if nf else np.zeros(0, np.int64),
                   "makespan": int(r.makespan), "status": int(r.status)}
        finally:
            lib().fastt_free_split_result(C.byref(r))
        return res


def fit_comm(n_devices, src, dst, nbytes, time_ns, device=0, stream=None):
    """fastt_fit_comm: per ordered device pair the non-negative least-squares
    line time = alpha + beta * bytes (R26).  Returns (alpha_ns, beta_fs, count)
    as G x G int64 arrays."""
    G = int(n_devices)
    src = np.ascontiguousarray(np.asarray(src, np.uint8))
    dst = np.ascontiguousarray(np.asarray(dst, np.uint8))
    nb = np.ascontiguousarray(np.asarray(nbytes, np.int64))
    tn = np.ascontiguousarray(np.asarray(time_ns, np.int64))
    n = len(src)
    if not (len(dst) == len(nb) == len(tn) == n):
        raise ValueError("sample arrays differ in length")
    a = np.zeros(G * G, np.int64)
    b = np.zeros(G * G, np.int64)
    c = np.zeros(G * G, np.int64)
    o = _opts(0, stream)
    _check(lib().fastt_fit_comm(G, n, _ptr(src), _ptr(dst), _ptr(nb), _ptr(tn), int(device), C.byref(o), _ptr(a),
                                _ptr(b), _ptr(c)))
    return a.reshape(G, G), b.reshape(G, G), c.reshape(G, G)


def cost_table(n_ops, n_devices, op, dev, time_ns, device=0, stream=None):
    """fastt_cost_table: per (op, device) the mean sample time, nearest ns
    (halves up), 0 where no sample exists."""
    V, G = int(n_ops), int(n_devices)
    op = np.ascontiguousarray(np.asarray(op, np.int32))
    dv = np.ascontiguousarray(np.asarray(dev, np.uint8))
    tn = np.ascontiguousarray(np.asarray(time_ns, np.int64))
    n = len(op)
    if not (len(dv) == len(tn) == n):
        raise ValueError("sample arrays differ in length")
    out = np.zeros(V * G, np.int64)
    o = _opts(0, stream)
    _check(lib().fastt_cost_table(V, G, n, _ptr(op), _ptr(dv), _ptr(tn), int(device), C.byref(o), _ptr(out)))
    return out.reshape(V, G)


def link_model(alpha_ns, beta_fs):
    """fastt_link_model: per-pair parameters -> (link_class[G][G], alpha[K], beta[K])."""
    a = np.ascontiguousarray(np.asarray(alpha_ns, np.int64))
    b = np.ascontiguousarray(np.asarray(beta_fs, np.int64))
    G = a.shape[0]
    lc = np.zeros((G, G), np.uint8)
    k = np.zeros(1, np.int32)
    ka = np.zeros(16, np.int64)
    kb = np.zeros(16, np.int64)
    _check(lib().fastt_link_model(G, _ptr(a), _ptr(b), _ptr(lc), _ptr(k), _ptr(ka), _ptr(kb)))
    K = int(k[0])
    return lc, ka[:K].copy(), kb[:K].copy()


def load_graph(desc, device=0):
    return Graph(desc, device)


def version():
    return lib().fastt_version().decode()
