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


def _q3_rows(res):
    """oracle Q3 result -> hash group-by rows as the device emits them: [(l_orderkey << 32) | o_orderdate, count, sum]."""
    import numpy as np
    rows = np.zeros((len(res.keys), 3), dtype=np.int64)
    for i, (k, a) in enumerate(zip(res.keys, res.aggs)):
        rows[i] = [(int(k[0]) << 32) | (int(k[1]) & 0xFFFFFFFF), a[0], a[1]]
    return rows


def _worker_hash(rank, world, port, ret):
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    sys.path.insert(0, root)
    import numpy as np

    import oracle
    import tpchgen
    from paper_conf_sigmod_paulhh16_b200 import gpl, queries

    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        sf, seed = 0.05, 29
        whole_db = tpchgen.generate(sf, seed=seed)
        whole = oracle.run("Q3", whole_db)
        seg = queries.segments(queries.plan_text("Q3", whole_db))[-1]
        full_seg = "\n".join(ln for ln in seg.splitlines() if not ln.startswith(("order", "limit")))
        ctx = gpl.Context(device=-1)
        ok = True
        # (1) order-key shards (§8(e) layout): groups are disjoint; each rank ships its top-10 rows only
        shard = tpchgen.generate(sf, seed=seed, rank=rank, world=world)
        local_top = _q3_rows(oracle.order_limit("Q3", oracle.run("Q3", shard)))
        parts = [None] * world
        dist.all_gather_object(parts, local_top)
        r = ctx.merge_groups(seg, np.concatenate(parts))
        want = oracle.order_limit("Q3", whole)
        ok &= r.keys == want.keys and r.aggs == want.aggs
        # (2) lineitem split NOT on order boundaries: groups overlap across ranks, every group shipped
        n = whole_db.nrows("lineitem")
        # cut inside a qualifying order with >= 2 qualifying lineitems, so that group has rows on both ranks
        k = next(k for k, a in zip(whole.keys, whole.aggs) if a[0] >= 2)[0]
        first = int(np.nonzero(whole_db.tables["lineitem"]["l_orderkey"] == k)[0][0])
        mid = first + 1
        while not (whole_db.tables["lineitem"]["l_shipdate"][first:mid] > 19950315).any():
            mid += 1
        cut = [0, mid, n][rank:rank + 2]
        local_all = _q3_rows(oracle.run("Q3", whole_db, None, tuple(cut)))
        parts = [None] * world
        dist.all_gather_object(parts, local_all)
        rows = np.concatenate(parts)
        overlap = len({int(x) for x in parts[0][:, 0]} & {int(x) for x in parts[1][:, 0]}) if world == 2 else 0
        r = ctx.merge_groups(seg, rows)
        ok &= r.keys == want.keys and r.aggs == want.aggs and overlap > 0
        r = ctx.merge_groups(full_seg, rows)
        ok &= r.keys == whole.keys and r.aggs == whole.aggs and r.stats["groups_total"] == len(whole.keys)
        ret[rank] = bool(ok)
    finally:
        dist.destroy_process_group()


def test_hash_groupby_merge_world2():
    """NEXT-4 across ranks (§8(e)): hash group-by rows all-gathered over gloo and merged exactly by
    gpl_merge_groups (int128 sums per key, then ORDER BY/LIMIT) equal the oracle on the whole database —
    for order-key shards (disjoint groups: the ranks' top-10s suffice) and for an arbitrary lineitem split
    (overlapping groups: all groups shipped)."""
    ctx = mp.get_context("spawn")
    mgr = ctx.Manager()
    ret = mgr.dict()
    port = _free_port()
    procs = [ctx.Process(target=_worker_hash, args=(r, 2, port, ret)) for r in range(2)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(timeout=300)
    assert all(p.exitcode == 0 for p in procs)
    assert ret.get(0) and ret.get(1)
