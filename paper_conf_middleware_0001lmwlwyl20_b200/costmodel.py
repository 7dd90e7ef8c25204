"""Cost-model ingestion (host side).

The paper bootstraps its cost models from profiled training steps
(RunMetadata of the TensorFlow profiler): "The computation cost
model provides the execution time of a (sub-)operation on a device, using the
operation's name and device as the key.  The communication cost model provides
the tensor transfer time between adjacent operations assigned to two different
devices, according to tensor size and device pair", with a linear
regression per device pair.  The B200 analogue reads a Chrome
trace as exported by ``torch.profiler`` (``prof.export_chrome_trace``, the
Kineto format; ``tests/golden/trace_b200_mlp2.json`` is a trimmed capture
from a B200, ``tools/capture_trace.py``):

* computation samples: complete events (``"ph": "X"``) whose ``name`` is a
  graph op name -- the GPU-side spans of ``record_function(op_name)``
  (category ``gpu_user_annotation``, one per annotated op execution on the
  device in ``args["device"]``), or ``kernel`` / ``cpu_op`` / ``gpu_op``
  events named after graph ops; ``dur`` is in microseconds;
* transfer samples: ``gpu_memcpy`` events with ``args["bytes"]``.  The
  device pair comes from ``args["src_device"]`` / ``args["dst_device"]`` when
  present (peer copies), else from the copy kind in the name: ``HtoD`` is
  host -> ``args["device"]``, ``DtoH`` the reverse, with the host mapped to
  device index ``host_device`` (transfers over the host link are skipped when
  it is None); same-device copies are not transfers.

``cost_table`` averages the computation samples into the int64-ns table of
``fastt_graph_desc`` on the GPU (``fastt_cost_table``: unknown entries are 0,
P:472-477); ``fit_link_model`` fits the transfer samples on the GPU
(``fastt_fit_comm``, reading R26) and groups the pairs into link classes
(``fastt_link_model``).  Everything here is trace parsing and argument
marshalling around the C-ABI; the arithmetic runs in ``k_fit.cu``.
"""
from __future__ import annotations

import json
from fractions import Fraction

import numpy as np

from . import fastt as F

_COMPUTE_CATS = ("gpu_user_annotation", "kernel", "cpu_op", "gpu_op", "operator")


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


def _device(e):
    """the device of an event: args.device, else (device-side Kineto events,
    whose pid is the GPU index) pid"""
    a = e.get("args") or {}
    if a.get("device") is not None:
        return a["device"]
    if str(e.get("cat", "")).startswith("gpu_") or e.get("cat") == "kernel":
        return e.get("pid")
    return None


def compute_samples(events, op_index):
    """(op id, device, ns) for every compute event whose name is a graph op."""
    out = []
    for e in events:
        if e.get("ph") != "X" or e.get("cat") not in _COMPUTE_CATS:
            continue
        op = op_index.get(e.get("name"))
        dev = _device(e)
        if op is None or dev is None or "dur" not in e:
            continue
        out.append((int(op), int(dev), _ns(e["dur"])))
    return out


def _copy_pair(e, host_device):
    """(src, dst) devices of a gpu_memcpy event, None if not a transfer"""
    a = e.get("args") or {}
    if "src_device" in a and "dst_device" in a:
        return int(a["src_device"]), int(a["dst_device"])
    name = e.get("name", "")
    dev = _device(e)
    if dev is None:
        return None
    if "HtoD" in name:
        return (None if host_device is None else (int(host_device), int(dev)))
    if "DtoH" in name:
        return (None if host_device is None else (int(dev), int(host_device)))
    if "dst_device" in a:
        return int(dev), int(a["dst_device"])
    return None  # DtoD / DtoH without a host index / memset: no device pair


def comm_samples(events, host_device=None):
    """(src device, dst device, bytes, ns) for every copy between two devices
    (the host counts as device host_device when given)."""
    out = []
    for e in events:
        if e.get("ph") != "X" or e.get("cat") != "gpu_memcpy" or "dur" not in e:
            continue
        b = (e.get("args") or {}).get("bytes")
        pr = _copy_pair(e, host_device)
        if pr is None or b is None or pr[0] == pr[1]:
            continue
        out.append((pr[0], pr[1], int(b), _ns(e["dur"])))
    return out


def cost_table(events, op_index, n_ops, n_devices, device=0):
    """cost_ns[op][device] = mean of the op's samples on the device (nearest
    integer ns, halves up); 0 where no sample exists.  The
    averaging runs in the library (fastt_cost_table)."""
    smp = [(op, dev, t) for op, dev, t in compute_samples(events, op_index) if 0 <= op < n_ops and 0 <= dev < n_devices]
    if smp:
        op, dv, t = (np.asarray(x) for x in zip(*smp))
    else:
        op = dv = t = np.zeros(0, np.int64)
    return F.cost_table(n_ops, n_devices, op, dv, t, device=device)


def fit_link_model(events, n_devices, device=0, host_device=None):
    """Transfer samples -> per-pair fit on the GPU -> link classes.
    Returns dict(link_class, alpha, beta, pair_alpha, pair_beta, count).
    With host_device, n_devices counts the host as one more device."""
    smp = comm_samples(events, host_device)
    if smp:
        s, d, b, t = (np.asarray(x) for x in zip(*smp))
    else:
        s = d = b = t = np.zeros(0, np.int64)
    pa, pb, cnt = F.fit_comm(n_devices, s, d, b, t, device=device)
    lc, ka, kb = F.link_model(pa, pb)
    return {"link_class": lc, "alpha": ka, "beta": kb, "pair_alpha": pa, "pair_beta": pb, "count": cnt}
