"""Build tiny tpchgen-shaped databases from the hand-written fixtures in tests/golden/."""
import json
import os

import numpy as np

import tpchgen

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")

_COLS = {
    "region": [("r_regionkey", np.int32), ("r_name", np.int32)],
    "nation": [("n_nationkey", np.int32), ("n_name", np.int32), ("n_regionkey", np.int32)],
    "supplier": [("s_suppkey", np.int32), ("s_nationkey", np.int32)],
    "customer": [("c_custkey", np.int32), ("c_nationkey", np.int32), ("c_mktsegment", np.int32)],
    "part": [("p_partkey", np.int32), ("p_type", np.int32), ("p_retailprice", np.int64)],
    "partsupp": [("ps_partkey", np.int32), ("ps_suppkey", np.int32), ("ps_supplycost", np.int64)],
    "orders": [("o_orderkey", np.int32), ("o_custkey", np.int32), ("o_orderdate", np.int32)],
    "lineitem": [(c, t) for c, t in zip(tpchgen.LINEITEM_COLS, tpchgen._LI_TYPES)],
}
_DICT_COLS = {"r_name": "r_name", "n_name": "n_name", "p_type": "p_type", "c_mktsegment": "c_mktsegment"}


def load(name):
    with open(os.path.join(GOLDEN, name)) as f:
        return json.load(f)


def build_db(fx):
    """Database whose dictionary columns are codes into per-fixture dictionaries."""
    db = tpchgen.Database(sf=0.0, seed=0)
    dicts = {"r_name": [], "n_name": [], "p_type": [], "c_mktsegment": []}
    for tname, spec in fx["tables"].items():
        for c in spec["columns"]:
            if c in dicts:
                j = spec["columns"].index(c)
                for row in spec["rows"]:
                    if row[j] not in dicts[c]:
                        dicts[c].append(row[j])
    for d in dicts.values():
        d.sort()
    db.r_name, db.n_name, db.p_type = dicts["r_name"], dicts["n_name"], dicts["p_type"]
    db.c_mktsegment = dicts["c_mktsegment"] or list(tpchgen.SEGMENTS)
    for tname, cols in _COLS.items():
        spec = fx["tables"].get(tname, {"columns": [], "rows": []})
        n = len(spec["rows"])
        t = {}
        for c, ty in cols:
            if c in spec["columns"]:
                j = spec["columns"].index(c)
                vals = [r[j] for r in spec["rows"]]
                if c in dicts:
                    vals = [dicts[c].index(v) for v in vals]
                t[c] = np.array(vals, dtype=ty)
            else:
                t[c] = np.zeros(n, dtype=ty)
        db.tables[tname] = t
    return db


def expected_keys_as_codes(fx, db):
    """Map expected string keys (nation names) to the fixture's dictionary codes."""
    out = []
    for k in fx["expected"]["keys"]:
        out.append(tuple(db.n_name.index(v) if isinstance(v, str) else v for v in k))
    return out
