"""Cost-model ingestion (host side).

The paper bootstraps its cost models from profiled training steps
(RunMetadata of the TensorFlow profiler): "The computation cost
model provides the execution time of a (sub-)operation on a device, using the
operation's name and device as the key.  The communication cost model provides
the tensor transfer time between adjacent operations assigned to two different
devices, according to tensor size and device pair", with a linear
regression per device pair.  The B200 analogue reads a Chrome
trace as exported by ``torch.profiler`` (``prof.export_chrome_trace``):

* complete events (``"ph": "X"``) of category ``kernel`` / ``cpu_op`` /
  ``gpu_op`` whose ``name`` is a graph op name give computation samples,
  keyed by (name, ``args["device"]``); ``dur`` is in microseconds;
* events of category ``gpu_memcpy`` with ``args["bytes"]``,
  ``args["src_device"]`` and ``args["dst_device"]`` (or ``args["device"]``
  as the source) give transfer samples.

``cost_table`` averages the computation samples into the int64-ns table of
``fastt_graph_desc`` (unknown entries are 0); ``fit_link_model``
fits the transfer samples on the GPU (``fastt_fit_comm``, reading R26) and
groups the pairs into link classes (``fastt_link_model``).  Everything here is
argument marshalling around the C-ABI; the arithmetic of the fit runs in
``k_fit.cu``.
"""
from __future__ import annotations

import json
from fractions import Fraction

import numpy as np

from . import fastt as F

_COMPUTE_CATS = ("kernel", "cpu_op", "gpu_op", "operator")


def load_trace(path_or_obj):
    """A Chrome trace (path, JSON string, dict or event list) -> event list."""
    obj = path_or_obj
    if isinstance(obj, str):
        obj = json.loads(obj) if obj.lstrip().startswith(("{", "[")) else json.load(open(obj))
    if isinstance(obj, dict):
        obj = obj.get("traceEvents", [])
    return list(obj)


def _ns(dur_us):
    """Microseconds (trace float) -> integer ns, nearest with halves up."""
    q = Fraction(str(dur_us)) * 1000
    return int((q.numerator * 2 + q.denominator) // (2 * q.denominator))


def compute_samples(events, op_index):
    """(op id, device, ns) for every compute event whose name is a graph op."""
    out = []
    for e in events:
        if e.get("ph") != "X" or e.get("cat") not in _COMPUTE_CATS:
            continue
        op = op_index.get(e.get("name"))
        dev = (e.get("args") or {}).get("device")
        if op is None or dev is None or "dur" not in e:
            continue
        out.append((int(op), int(dev), _ns(e["dur"])))
    return out


def comm_samples(events):
    """(src device, dst device, bytes, ns) for every device-to-device copy."""
    out = []
    for e in events:
        if e.get("ph") != "X" or e.get("cat") != "gpu_memcpy":
            continue
        a = e.get("args") or {}
        s = a.get("src_device", a.get("device"))
        d = a.get("dst_device")
        b = a.get("bytes")
        if s is None or d is None or b is None or int(s) == int(d) or "dur" not in e:
            continue
        out.append((int(s), int(d), int(b), _ns(e["dur"])))
    return out


def cost_table(events, op_index, n_ops, n_devices):
    """cost_ns[op][device] = mean of the op's samples on the device (nearest
    integer ns, halves up); 0 where no sample exists."""
    acc = {}
    for op, dev, t in compute_samples(events, op_index):
        if 0 <= op < n_ops and 0 <= dev < n_devices:
            s = acc.setdefault((op, dev), [0, 0])
            s[0] += t
            s[1] += 1
    cost = np.zeros((n_ops, n_devices), np.int64)
    for (op, dev), (tot, cnt) in acc.items():
        cost[op, dev] = (2 * tot + cnt) // (2 * cnt)
    return cost


def fit_link_model(events, n_devices, device=0):
    """Transfer samples -> per-pair fit on the GPU -> link classes.
    Returns dict(link_class, alpha, beta, pair_alpha, pair_beta, count)."""
    smp = comm_samples(events)
    if smp:
        s, d, b, t = (np.asarray(x) for x in zip(*smp))
    else:
        s = d = b = t = np.zeros(0, np.int64)
    pa, pb, cnt = F.fit_comm(n_devices, s, d, b, t, device=device)
    lc, ka, kb = F.link_model(pa, pb)
    return {"link_class": lc, "alpha": ka, "beta": kb, "pair_alpha": pa, "pair_beta": pb, "count": cnt}
