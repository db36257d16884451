"""Multi-rank host path on CPU (gloo, world size 2): the §8(e) sharding and the
exact partial-aggregate merge that bench.py runs over NCCL on GPUs.

* each rank generates its order-key shard of lineitem+orders (dimensions
  replicated); per-rank oracle partials merged over the collective equal the
  oracle on the whole database (co-partitioned orders make this exact);
* int128 partial vectors all-gathered over gloo and reduced by
  gpl_merge_partials in fixed rank order equal the Python-integer sum.
"""
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


def _worker(rank, world, port, q, ret):
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    sys.path.insert(0, root)
    import torch

    import oracle
    import tpchgen
    from paper_conf_sigmod_paulhh16_b200 import gpl

    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        sf, seed = 0.02, 17
        shard = tpchgen.generate(sf, seed=seed, rank=rank, world=world)
        local = oracle.run(q, shard).as_dict()
        gathered = [None] * world
        dist.all_gather_object(gathered, local)
        merged = {}
        for part in gathered:
            for k, v in part.items():
                merged[k] = [a + b for a, b in zip(merged.get(k, [0] * len(v)), v)]
        whole = oracle.run(q, tpchgen.generate(sf, seed=seed)).as_dict()
        merged = {k: v for k, v in merged.items() if v[0] > 0 or k == ()}
        ok_shard = merged == whole

        # int128 partial vectors through the collective + gpl_merge_partials
        rng = np.random.default_rng(100 + rank)
        vals = [int(x) * (1 << 40) + int(y) for x, y in zip(rng.integers(-2**40, 2**40, 16), rng.integers(0, 2**40, 16))]
        buf = np.zeros((16, 2), dtype=np.uint64)
        for i, v in enumerate(vals):
            u = v & ((1 << 128) - 1)
            buf[i, 0], buf[i, 1] = u & ((1 << 64) - 1), u >> 64
        t = torch.from_numpy(buf.view(np.int64).reshape(-1).copy())
        out = torch.empty(world * t.numel(), dtype=torch.int64)
        dist.all_gather_into_tensor(out, t)
        merged128 = gpl.merge_partials(out.numpy().view(np.uint64), world).reshape(16, 2)
        all_vals = [None] * world
        dist.all_gather_object(all_vals, vals)
        ok_merge = True
        for i in range(16):
            got = (int(merged128[i, 1]) << 64) | int(merged128[i, 0])
            if got >= 1 << 127:
                got -= 1 << 128
            ok_merge &= got == sum(v[i] for v in all_vals)
        ret[rank] = bool(ok_shard and ok_merge)
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("q", ["Q5", "Q9"])
def test_sharded_merge_world2(q):
    ctx = mp.get_context("spawn")
    mgr = ctx.Manager()
    ret = mgr.dict()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q, ret)) for r in range(2)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(timeout=300)
    assert all(p.exitcode == 0 for p in procs)
    assert ret.get(0) and ret.get(1)
