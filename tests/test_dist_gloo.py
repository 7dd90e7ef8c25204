"""Multi-rank argmin logic over torch.distributed with the
gloo backend on CPU, world_size 2 and 4: the two-pass all_reduce(MIN) of
combine_best equals the lexicographic min over all ranks, ties go to the
smallest global index, and all-infeasible stays (INT64_MAX, -1)."""
import os
import socket

import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_middleware_0001lmwlwyl20_b200.dist import INT64_MAX, combine_best

CASES = [
    [(50, 7), (40, 3), (40, 1), (60, 0)],
    [(40, 9), (40, 2), (40, 6), (40, 4)],
    [(INT64_MAX, -1), (INT64_MAX, -1), (INT64_MAX, -1), (INT64_MAX, -1)],
    [(INT64_MAX, -1), (77, 5), (INT64_MAX, -1), (78, 1)],
    [((1 << 62) + 5, (1 << 40) + 3), ((1 << 62) + 5, (1 << 40) + 1), ((1 << 62) + 6, 0), (INT64_MAX, -1)],
]


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    out = []
    for case in CASES:
        b = torch.tensor(list(case[rank]), dtype=torch.int64)
        combine_best(b)
        out.append(tuple(b.tolist()))
    q.put((rank, out))
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 4])
def test_combine_best_gloo(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in ps:
        p.start()
    res = dict(q.get(timeout=120) for _ in range(world))
    for p in ps:
        p.join(timeout=60)
    for k, case in enumerate(CASES):
        sub = case[:world]
        feas = [c for c in sub if c[1] >= 0]
        want = min(feas) if feas else (INT64_MAX, -1)
        for r in range(world):
            assert res[r][k] == want, (k, r, res[r][k], want)
