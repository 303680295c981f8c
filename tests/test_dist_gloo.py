"""World-size-2 tests of the N>1 host path on CPU (gloo): unique-id rendezvous,
max-over-ranks timing, and the slice-then-sum exchange (a11) with the oracle standing in
for the per-rank GPU partials.  The work-balanced bounds rule is restated here
(w(u) = d~(u) + Σ_{v∈N+(u)} d~(v), or Σ min(d~(u), d~(v)) under the shorter-list schedule;
bound g = first u with prefix >= g·W/world) and checked against the GPU implementation in
tests/test_gpu_configs.py."""
import os
import socket

import numpy as np
import pytest
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def work_bounds(offs, col, world, bucket_off=None, shorter=False):
    n = len(offs) - 1
    od = np.diff(offs.astype(np.int64))
    w = od.copy()
    for u in range(n):
        dv = od[col[offs[u]:offs[u + 1]]]
        w[u] += np.minimum(dv, od[u]).sum() if shorter else dv.sum()
    pre = np.concatenate([[0], np.cumsum(w)])
    W = pre[-1]
    b = [0]
    for g in range(1, world):
        b.append(int(np.searchsorted(pre[:n + 1], (W * g) // world, side="left")))
    b.append(n)
    if bucket_off is not None and len(bucket_off):
        for g in range(1, world):
            i = np.searchsorted(bucket_off, b[g], side="left")
            b[g] = int(bucket_off[i]) if i < len(bucket_off) else n
            b[g] = max(b[g], b[g - 1])
    return b


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import graphgen
        import oracle
        from paper_conf_sigmod_hu0l21_b200 import dist as tdist

        # rendezvous of the NCCL unique id (128 opaque bytes) as done before tc_nccl_comm_init
        uid = tdist.broadcast_bytes(bytes(range(128)) if rank == 0 else None)
        assert uid == bytes(range(128))
        # timing reduction: max over ranks
        assert tdist.max_over_ranks(1.5 + rank) == 1.5 + world - 1
        # a11 exchange: every rank counts its slice, one sum-allreduce gives T
        spec = graphgen.rmat_spec(11, 16, 42)
        src, dst = graphgen.generate_cpu(spec)
        for d, r in (("degree", "none"), ("paper", "paper")):
            res = oracle.run(src, dst, spec.n, d, r)
            b = work_bounds(res["offs"], res["col"], world, res["bucket_off"])
            part = oracle.count_forward(res["offs"], res["col"], b[rank], b[rank + 1])
            total = tdist.sum_over_ranks_u64(part)
            assert total == res["T"], (d, r, total, res["T"])
        q.put((rank, "ok"))
    except Exception as e:  # pragma: no cover - surfaced through the queue
        q.put((rank, repr(e)))
    finally:
        dist.destroy_process_group()


def test_gloo_world2_slices_sum_to_total():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    results = dict(q.get(timeout=300) for _ in procs)
    for p in procs:
        p.join(timeout=60)
    assert results == {0: "ok", 1: "ok"}, results


def test_bounds_rule_properties():
    import graphgen
    import oracle
    spec = graphgen.rmat_spec(10, 16, 7)
    src, dst = graphgen.generate_cpu(spec)
    res = oracle.run(src, dst, spec.n, "degree", "none")
    for world, shorter in ((1, False), (2, True), (3, False), (8, True)):
        b = work_bounds(res["offs"], res["col"], world, shorter=shorter)
        assert b[0] == 0 and b[-1] == spec.n and all(x <= y for x, y in zip(b, b[1:]))
        parts = [oracle.count_forward(res["offs"], res["col"], b[i], b[i + 1]) for i in range(world)]
        assert sum(parts) == res["T"]
