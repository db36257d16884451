"""Generator properties (input recipe): determinism under
sharding, FK integrity, value ranges, physical clustering."""
import numpy as np
import pytest

import tpchgen


@pytest.fixture(scope="module")
def db():
    return tpchgen.generate(0.01, seed=7)


def test_sizes_scale():
    s = tpchgen.sizes(1.0)
    assert s == {"part": 200000, "supplier": 10000, "partsupp": 800000, "customer": 150000,
                 "orders": 1500000}
    assert tpchgen.sizes(0.0005)["supplier"] >= 4


def test_deterministic_and_shard_invariant():
    a = tpchgen.generate(0.01, seed=11)
    b = tpchgen.generate(0.01, seed=11)
    for t in a.tables:
        for c in a.tables[t]:
            assert np.array_equal(a.tables[t][c], b.tables[t][c])
    shards = [tpchgen.generate(0.01, seed=11, rank=r, world=3, tables=["orders", "lineitem"])
              for r in range(3)]
    for t in ("orders", "lineitem"):
        for c in a.tables[t]:
            cat = np.concatenate([s.tables[t][c] for s in shards])
            assert np.array_equal(cat, a.tables[t][c]), (t, c)
    c = tpchgen.generate(0.01, seed=12)
    assert not np.array_equal(c.tables["lineitem"]["l_partkey"], a.tables["lineitem"]["l_partkey"])


def test_fk_integrity(db):
    li, o, ps = db.tables["lineitem"], db.tables["orders"], db.tables["partsupp"]
    assert np.isin(li["l_orderkey"], o["o_orderkey"]).all()
    assert np.isin(li["l_partkey"], db.tables["part"]["p_partkey"]).all()
    assert np.isin(li["l_suppkey"], db.tables["supplier"]["s_suppkey"]).all()
    assert np.isin(o["o_custkey"], db.tables["customer"]["c_custkey"]).all()
    assert (o["o_custkey"] % 3 != 0).all()
    pairs = set(zip(ps["ps_partkey"].tolist(), ps["ps_suppkey"].tolist()))
    assert len(pairs) == len(ps["ps_partkey"])  # composite PK unique
    assert all((p, s) in pairs for p, s in zip(li["l_partkey"].tolist(), li["l_suppkey"].tolist()))
    for t, k in (("part", "p_partkey"), ("supplier", "s_suppkey"), ("customer", "c_custkey"),
                 ("orders", "o_orderkey")):
        assert len(np.unique(db.tables[t][k])) == len(db.tables[t][k])


def test_value_ranges(db):
    li = db.tables["lineitem"]
    assert li["l_discount"].min() >= 0 and li["l_discount"].max() <= 10
    assert li["l_tax"].min() >= 0 and li["l_tax"].max() <= 8
    q = li["l_quantity"] // 100
    assert q.min() >= 1 and q.max() <= 50 and (li["l_quantity"] % 100 == 0).all()
    price = dict(zip(db.tables["part"]["p_partkey"].tolist(), db.tables["part"]["p_retailprice"].tolist()))
    assert all(ep == qq * price[pk] for ep, qq, pk in
               zip(li["l_extendedprice"][:500].tolist(), q[:500].tolist(), li["l_partkey"][:500].tolist()))
    od = db.tables["orders"]["o_orderdate"]
    assert od.min() >= 19920101 and od.max() <= 19980802
    assert li["l_shipdate"].min() > 19920101 and li["l_shipdate"].max() <= 19981231
    m, d = (li["l_shipdate"] // 100) % 100, li["l_shipdate"] % 100
    assert m.min() >= 1 and m.max() <= 12 and d.min() >= 1 and d.max() <= 31
    assert db.tables["supplier"]["s_nationkey"].max() <= 24
    assert db.tables["part"]["p_type"].max() < 150
    ps = db.tables["partsupp"]["ps_supplycost"]
    assert ps.min() >= 100 and ps.max() <= 100000


def test_clustered_by_orderkey(db):
    ok = db.tables["lineitem"]["l_orderkey"]
    assert (np.diff(ok) >= 0).all()
    assert (np.diff(db.tables["orders"]["o_orderkey"]) > 0).all()


def test_dictionaries():
    pt = tpchgen.P_TYPES
    assert len(pt) == 150 and pt == sorted(pt)
    promo = [i for i, s in enumerate(pt) if s.startswith("PROMO")]
    assert promo == list(range(promo[0], promo[0] + 25))  # contiguous code range
    assert "ECONOMY ANODIZED STEEL" in pt
    asia = [i for i, (n, r) in enumerate(tpchgen.NATIONS) if tpchgen.REGIONS[r] == "ASIA"]
    assert asia == [8, 9, 12, 18, 21]


def test_date_add_days():
    assert tpchgen.date_add_days(19951231, 1) == 19960101
    assert tpchgen.date_add_days(19960228, 1) == 19960229
    assert tpchgen.date_add_days(19970228, 1) == 19970301
    assert tpchgen.date_add_days(19950901, 30) == 19951001
