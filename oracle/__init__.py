"""ctypes binding of the plain C oracle (``oracle/fastt_oracle.c``).

TEST INFRASTRUCTURE ONLY: imported by ``tests/``, ``__graft_entry__.smoke()``
and ``bench.py``'s cpu_baseline / ``--impl reference`` legs.  Nothing in the
product package imports this module, and this module imports nothing from the
product package (the seeded input generators live in their own module and hold
none of the method's arithmetic).

Parity status of each oracle function is listed in DESIGN.md ("Oracle pins").
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "fastt_oracle.c")
_LIB = os.path.join(_HERE, "liboracle_fastt.so")
# tools/oracle_mutants.py points this at a mutated copy of the source (built
# into /tmp) to show that the pins catch each mutation
if os.environ.get("FASTT_ORACLE_SRC"):
    _SRC = os.path.abspath(os.environ["FASTT_ORACLE_SRC"])
    _LIB = "/tmp/liboracle_%s.so" % os.path.basename(_SRC).replace(".c", "")

INF = np.iinfo(np.int64).max
CAND_OK, CAND_INFEASIBLE, CAND_BADSPEC = 0, 1, 2
KIND_BASE, KIND_PIN, KIND_SPLIT = 0, 1, 2
DIM_BATCH, DIM_CHANNEL = 0, 1
F_CP_PIN = 1
F_POLICY_INSERT = 2
F_MEM_LIVE = 64
F_SPLIT_MULTI = 128  # best-improvement split search with multi-split candidates (R27)
GEN_POW2, GEN_SUBSETS = 1, 2

CAND_DTYPE = np.dtype(
    [("kind", "u1"), ("n_pins", "u1"), ("split_dim", "u1"), ("split_n", "u1"),
     ("split_op", "<i4"), ("pin_op", "<i4", (4,)), ("pin_dev", "u1", (4,)), ("dev_mask", "<u4")]
)
assert CAND_DTYPE.itemsize == 32


def build(force: bool = False) -> str:
    """Compile the oracle with plain gcc -O2 (no vectorisation claims)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + ".tmp%d" % os.getpid()
        subprocess.check_call(["gcc", "-O2", "-std=gnu11", "-shared", "-fPIC", "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        _lib = C.CDLL(build())
        P = C.c_void_p
        i32, i64, u32, u64 = C.c_int32, C.c_int64, C.c_uint32, C.c_uint64
        _lib.fastt_ref_load.restype = i32
        _lib.fastt_ref_load.argtypes = [i32, i64, i32, P, P, P, P, P, P, P, P, P, P, i32, P, P, i64, C.POINTER(P)]
        _lib.fastt_ref_free.argtypes = [P]
        _lib.fastt_ref_v_max.restype = i32
        _lib.fastt_ref_v_max.argtypes = [P]
        _lib.fastt_ref_num_ops.restype = i32
        _lib.fastt_ref_num_ops.argtypes = [P]
        _lib.fastt_ref_num_edges.restype = i64
        _lib.fastt_ref_num_edges.argtypes = [P]
        _lib.fastt_ref_schedule.restype = i32
        _lib.fastt_ref_schedule.argtypes = [P, i32, i32, P, P, i32, i32, i32, u32, u32, P, P, P, P, P, P, P, P]
        _lib.fastt_ref_split_export.restype = i64
        _lib.fastt_ref_split_export.argtypes = [P, i32, i32, i32, P, P, P, P, P, P, P, P, P]
        _lib.fastt_ref_rank.restype = i32
        _lib.fastt_ref_rank.argtypes = [P, i32, i32, P, P, i32, i32, i32, u32, P]
        _lib.fastt_ref_split_search.restype = i32
        _lib.fastt_ref_split_search.argtypes = [P, u32, i32, i32, P, P, P, P, i32, P, P, P, P, P, P]
        _lib.fastt_ref_split_search_bi.restype = i32
        _lib.fastt_ref_split_search_bi.argtypes = [P, u32, i32, i32, P, P, P, P, i32, P, P, P, P, P, P]
        _lib.fastt_ref_stream_info.restype = i32
        _lib.fastt_ref_stream_info.argtypes = [P, u32, i32, P, P]
        _lib.fastt_ref_generate.restype = i32
        _lib.fastt_ref_generate.argtypes = [P, u32, u64, i32, i32, i32, i64, i64, P]
        _lib.fastt_ref_sweep.restype = i32
        _lib.fastt_ref_sweep.argtypes = [P, u32, u64, i32, i32, i32, i64, i64, i64, P, P, P]
        _lib.fastt_ref_splitmix64_next.restype = u64
        _lib.fastt_ref_splitmix64_next.argtypes = [C.POINTER(u64)]
        _lib.fastt_ref_cp.restype = i32
        _lib.fastt_ref_cp.argtypes = [P, P]
    return _lib


def _p(a):
    return a.ctypes.data_as(C.c_void_p) if a is not None else None


def splitmix64_next(state: int):
    s = C.c_uint64(state)
    v = lib().fastt_ref_splitmix64_next(C.byref(s))
    return int(v), int(s.value)


class OracleError(RuntimeError):
    def __init__(self, code):
        super().__init__("oracle status %d" % code)
        self.code = code


class OracleGraph:
    """A graph loaded into the oracle.  ``desc`` is a synth.GraphDesc (or any
    object with the same array attributes)."""

    def __init__(self, desc):
        L = lib()
        self._keep = []

        def arr(x, dt):
            a = np.ascontiguousarray(np.asarray(x, dtype=dt))
            self._keep.append(a)
            return a

        src = arr(desc.src, np.int32)
        dst = arr(desc.dst, np.int32)
        byt = arr(desc.bytes, np.int64)
        epr = arr(desc.eparam, np.uint8)
        cost = arr(desc.cost, np.int64).reshape(-1)
        mem = arr(desc.mem, np.int64)
        prm = arr(desc.param, np.int64)
        sm = arr(desc.split_mask, np.uint8)
        cap = arr(desc.cap, np.int64)
        lc = arr(desc.link_class, np.uint8).reshape(-1)
        al = arr(desc.alpha, np.int64)
        be = arr(desc.beta, np.int64)
        h = C.c_void_p()
        rc = L.fastt_ref_load(int(desc.n_ops), int(len(src)), int(desc.n_devices), _p(src), _p(dst), _p(byt),
                              _p(epr), _p(cost), _p(mem), _p(prm), _p(sm), _p(cap), _p(lc), int(len(al)), _p(al),
                              _p(be), int(desc.copy_fs), C.byref(h))
        self._keep = []
        if rc != 0:
            raise OracleError(rc)
        self.h = h
        self.G = int(desc.n_devices)
        self.V = int(L.fastt_ref_num_ops(h))
        self.E = int(L.fastt_ref_num_edges(h))
        self.v_max = int(L.fastt_ref_v_max(h))

    def __del__(self):
        if getattr(self, "h", None):
            lib().fastt_ref_free(self.h)
            self.h = None

    @staticmethod
    def _cand_args(cand):
        if cand is None:
            return KIND_BASE, 0, None, None, -1, 0, 0, 0
        c = cand
        pin_op = np.ascontiguousarray(np.asarray(c["pin_op"], dtype=np.int32).reshape(4))
        pin_dev = np.ascontiguousarray(np.asarray(c["pin_dev"], dtype=np.uint8).reshape(4))
        return (int(c["kind"]), int(c["n_pins"]), pin_op, pin_dev, int(c["split_op"]), int(c["split_dim"]),
                int(c["split_n"]), int(c["dev_mask"]))

    def schedule(self, cand=None, flags=0, outputs=True):
        """One candidate through DPOS.  Returns a dict."""
        kind, npins, po, pd, so, sd, sn, dm = self._cand_args(cand)
        ms = np.zeros(1, np.int64)
        st = np.zeros(1, np.uint8)
        peak = np.zeros(self.G, np.int64)
        vm = self.v_max
        place = np.zeros(vm, np.uint8) if outputs else None
        order = np.zeros(vm, np.int32) if outputs else None
        start = np.zeros(vm, np.int64) if outputs else None
        rank = np.zeros(vm, np.int64) if outputs else None
        deq = np.zeros(vm, np.int32) if outputs else None
        rc = lib().fastt_ref_schedule(self.h, kind, npins, _p(po), _p(pd), so, sd, sn, dm, flags, _p(ms), _p(peak),
                                      _p(st), _p(place), _p(order), _p(start), _p(rank), _p(deq))
        if rc != 0:
            raise OracleError(rc)
        out = {"makespan": int(ms[0]), "status": int(st[0]), "peak_mem": peak}
        if outputs:
            out.update(placement=place, order=order, start=start, rank=rank, dequeue=deq)
        return out

    def rank(self, cand=None):
        kind, npins, po, pd, so, sd, sn, dm = self._cand_args(cand)
        r = np.zeros(self.v_max, np.int64)
        rc = lib().fastt_ref_rank(self.h, kind, npins, _p(po), _p(pd), so, sd, sn, dm, _p(r))
        if rc != 0:
            raise OracleError(rc)
        return r

    def split_export(self, op, dim, n):
        """The materialised SplitOperation graph of a SPLIT candidate (R13)."""
        vm = self.v_max
        emax = self.E + vm * (self.G + 2) * 2 + 16
        Vo = np.zeros(1, np.int32)
        src = np.zeros(emax, np.int32)
        dst = np.zeros(emax, np.int32)
        byt = np.zeros(emax, np.int64)
        epr = np.zeros(emax, np.uint8)
        cost = np.zeros(vm * self.G, np.int64)
        mem = np.zeros(vm, np.int64)
        prm = np.zeros(vm, np.int64)
        alive = np.zeros(vm, np.uint8)
        E = lib().fastt_ref_split_export(self.h, op, dim, n, _p(Vo), _p(src), _p(dst), _p(byt), _p(epr), _p(cost),
                                         _p(mem), _p(prm), _p(alive))
        if E < 0:
            raise OracleError(int(E))
        V = int(Vo[0])
        return {"V": V, "src": src[:E], "dst": dst[:E], "bytes": byt[:E], "eparam": epr[:E],
                "cost": cost[: V * self.G].reshape(V, self.G), "mem": mem[:V], "param": prm[:V], "alive": alive[:V]}

    def critical_path(self):
        cp = np.zeros(self.V + 1, np.int32)
        n = lib().fastt_ref_cp(self.h, _p(cp))
        return cp[:n]

    def split_search(self, flags=0, pow2_only=False, out_cap=None, best_improvement=False, multi=False):
        cap = out_cap or (self.V + 64 * (self.G + 64) + 1024)
        sp_n = np.zeros(1, np.int32)
        spc = 4096
        sp_op = np.zeros(spc, np.int32)
        sp_dim = np.zeros(spc, np.uint8)
        sp_cnt = np.zeros(spc, np.uint8)
        nfin = np.zeros(1, np.int32)
        place = np.zeros(cap, np.uint8)
        order = np.zeros(cap, np.int32)
        start = np.zeros(cap, np.int64)
        ms = np.zeros(1, np.int64)
        st = np.zeros(1, np.uint8)
        fn = lib().fastt_ref_split_search_bi if (best_improvement or multi) else lib().fastt_ref_split_search
        rc = fn(self.h, flags | (F_SPLIT_MULTI if multi else 0), int(bool(pow2_only)), spc, _p(sp_n), _p(sp_op), _p(sp_dim),
                _p(sp_cnt), cap, _p(nfin), _p(place), _p(order), _p(start), _p(ms), _p(st))
        if rc != 0:
            raise OracleError(rc)
        n = int(sp_n[0])
        nf = int(nfin[0])
        if nf > cap:
            return self.split_search(flags, pow2_only, out_cap=nf + 16, best_improvement=best_improvement, multi=multi)
        return {"sp": [(int(sp_op[q]), int(sp_dim[q]), int(sp_cnt[q])) for q in range(n)], "n_ops_final": nf,
                "placement": place[:nf], "order": order[:nf], "start": start[:nf], "makespan": int(ms[0]),
                "status": int(st[0])}

    @staticmethod
    def _gen_opts(pow2_only, subsets):
        return (GEN_POW2 if pow2_only else 0) | (GEN_SUBSETS if subsets else 0)

    def stream_info(self, flags=0, pow2_only=False, subsets=False):
        ns = np.zeros(1, np.int64)
        bp = np.zeros(max(self.V, 1), np.uint8)
        lib().fastt_ref_stream_info(self.h, flags, self._gen_opts(pow2_only, subsets), _p(ns), _p(bp))
        return int(ns[0]), bp[: self.V]

    def generate(self, seed, first, n, kmin=1, kmax=4, flags=0, pow2_only=False, subsets=False):
        out = np.zeros(n, CAND_DTYPE)
        rc = lib().fastt_ref_generate(self.h, flags, seed, kmin, kmax, self._gen_opts(pow2_only, subsets), first, n,
                                      _p(out))
        if rc != 0:
            raise OracleError(rc)
        return out

    def sweep(self, seed, first, n, stride=1, kmin=1, kmax=4, flags=0, pow2_only=False, per_candidate=False,
              subsets=False):
        bm = np.zeros(1, np.int64)
        bi = np.zeros(1, np.int64)
        mss = np.zeros(n, np.int64) if per_candidate else None
        rc = lib().fastt_ref_sweep(self.h, flags, seed, kmin, kmax, self._gen_opts(pow2_only, subsets), first, n,
                                   stride, _p(bm), _p(bi), _p(mss))
        if rc != 0:
            raise OracleError(rc)
        res = {"makespan": int(bm[0]), "index": int(bi[0])}
        if per_candidate:
            res["makespans"] = mss
        return res


def make_cand(kind=KIND_BASE, pins=(), split=None, dev_mask=0):
    """Build one candidate record: pins = [(op, dev), ...]; split = (op, dim, n);
    dev_mask = the candidate's device subset (R25, 0 = all devices)."""
    c = np.zeros(1, CAND_DTYPE)[0]
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
