"""Capture a real torch.profiler (Kineto) Chrome trace on the GPU box for the
cost-model ingestion tests (P:459-465 profiled cost models):
the C1 MLP training graph's ops (synth.config("C1")) are executed as torch
CUDA ops, each under record_function("<op id>:<op type>") so the trace
carries one GPU-side span per op execution, plus host<->device copies of
several sizes (the only device pair one GPU has).  The trace is trimmed to
the events the cost model reads and written to tests/golden/trace_b200_mlp2.json;
the untrimmed export goes to gpurun_out/.

usage (on the box): python tools/capture_trace.py
       (here)         python tools/capture_trace.py --trim gpurun_out/trace_b200_mlp2_full.json "<gpu, torch>"
"""
import json
import os
import sys

import torch
from torch.profiler import ProfilerActivity, profile, record_function

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_middleware_0001lmwlwyl20_b200 import synth  # noqa: E402

OUT = os.path.join(ROOT, "tests", "golden", "trace_b200_mlp2.json")


def main():
    desc = synth.config("C1")
    V = desc.n_ops
    names = ["%d:%s" % (i, desc.op_type[i] if desc.op_type else "op") for i in range(V)]
    out_bytes = [0] * V
    for s, b in zip(desc.src, desc.bytes):
        out_bytes[int(s)] = max(out_bytes[int(s)], int(b))
    dev = torch.device("cuda", 0)
    x = torch.randn(64, 784, device=dev)
    w = torch.randn(784, 256, device=dev)
    bufs = [torch.randn(max(1, out_bytes[i] // 4), device=dev) for i in range(V)]
    hosts = [torch.empty(1 << k, dtype=torch.uint8).pin_memory() for k in range(10, 25, 2)]
    devs = [torch.empty(1 << k, dtype=torch.uint8, device=dev) for k in range(10, 25, 2)]
    torch.cuda.synchronize()

    def step():
        for i in range(V):
            t = desc.op_type[i] if desc.op_type else ""
            with record_function(names[i]):
                if "MatMul" in t:
                    torch.mm(x, w)
                else:
                    bufs[i].mul_(1.0001).add_(1e-6)
        for h, d in zip(hosts, devs):
            d.copy_(h, non_blocking=True)
            h.copy_(d, non_blocking=True)

    for _ in range(2):
        step()
    torch.cuda.synchronize()
    with profile(activities=[ProfilerActivity.CPU, ProfilerActivity.CUDA]) as prof:
        for _ in range(3):
            step()
        torch.cuda.synchronize()
    os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
    full = os.path.join(ROOT, "gpurun_out", "trace_b200_mlp2_full.json")
    prof.export_chrome_trace(full)
    trim(full, names, OUT, "%s, torch %s" % (torch.cuda.get_device_name(0), torch.__version__))


def trim(full, names, out, where):
    """keep the events the cost model reads: the GPU-side record_function
    spans of the graph ops and the memcpy events (Kineto puts the GPU index
    of device-side events in pid; args.device where it exists)"""
    tr = json.load(open(full))
    keep = []
    cats = {}
    for e in tr.get("traceEvents", []):
        cats[e.get("cat")] = cats.get(e.get("cat"), 0) + 1
        if e.get("ph") != "X":
            continue
        c = e.get("cat")
        a = e.get("args") or {}
        if c == "gpu_user_annotation" and e.get("name") in names:
            keep.append({"ph": "X", "cat": c, "name": e["name"], "pid": e.get("pid"), "ts": e.get("ts"), "dur": e["dur"],
                         "args": {k: a[k] for k in ("device",) if k in a}})
        elif c == "gpu_memcpy":
            keep.append({"ph": "X", "cat": c, "name": e["name"], "pid": e.get("pid"), "ts": e.get("ts"), "dur": e["dur"],
                         "args": {k: a[k] for k in ("device", "bytes", "src_device", "dst_device") if k in a}})
    res = {"fastt_note": "torch.profiler (Kineto) trace captured by tools/capture_trace.py on %s; trimmed to the "
                         "gpu_user_annotation spans of the C1 ops and the gpu_memcpy events" % where,
           "fastt_op_names": names, "fastt_event_categories": cats, "traceEvents": keep}
    with open(out, "w") as f:
        json.dump(res, f, indent=0)
    print("kept %d of %d events; categories %s" % (len(keep), sum(cats.values()), cats))


if __name__ == "__main__":
    if len(sys.argv) > 2 and sys.argv[1] == "--trim":  # re-trim an untrimmed export: --trim full.json [where]
        d = synth.config("C1")
        trim(sys.argv[2], ["%d:%s" % (i, d.op_type[i]) for i in range(d.n_ops)], OUT,
             sys.argv[3] if len(sys.argv) > 3 else "NVIDIA B200")
    else:
        main()
