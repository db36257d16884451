"""Seeded, shardable TPC-H-shaped input generator (ctypes over libtpchgen.so).

Input generation only: this module holds none of the method's arithmetic, so
both the CPU oracle (``oracle/``) and the CUDA path may consume its output
(task rule ③: "only the seeded input generators serve both").

Shapes: SURVEY.md Appendix B. The paper evaluated dbgen TPC-H data at SF 10
(§5.1) and SF 0.1-10 (§5.4); the GPU box has no network,
so data is generated in-repo with a counter-based RNG (identical bytes under
any thread count or shard).

Encodings: keys/dates/dictionary codes int32 (dates yyyymmdd); decimals int64
scaled by 100 (discount/tax in per cent).
"""
from __future__ import annotations

import ctypes
import itertools
import os
from dataclasses import dataclass, field

import numpy as np

DEFAULT_SEED = 20160626

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "libtpchgen.so")
_lib = None

# TPC-H fixed nation/region lists (TPC-H spec §4.2.3) [EXT]
REGIONS = ["AFRICA", "AMERICA", "ASIA", "EUROPE", "MIDDLE EAST"]
NATIONS = [
    ("ALGERIA", 0), ("ARGENTINA", 1), ("BRAZIL", 1), ("CANADA", 1), ("EGYPT", 4),
    ("ETHIOPIA", 0), ("FRANCE", 3), ("GERMANY", 3), ("INDIA", 2), ("INDONESIA", 2),
    ("IRAN", 4), ("IRAQ", 4), ("JAPAN", 2), ("JORDAN", 4), ("KENYA", 0),
    ("MOROCCO", 0), ("MOZAMBIQUE", 0), ("PERU", 1), ("CHINA", 2), ("ROMANIA", 3),
    ("SAUDI ARABIA", 4), ("VIETNAM", 2), ("RUSSIA", 3), ("UNITED KINGDOM", 3),
    ("UNITED STATES", 1),
]
_SYL1 = ["STANDARD", "SMALL", "MEDIUM", "LARGE", "ECONOMY", "PROMO"]
_SYL2 = ["ANODIZED", "BURNISHED", "PLATED", "POLISHED", "BRUSHED"]
_SYL3 = ["TIN", "NICKEL", "BRASS", "STEEL", "COPPER"]
# p_type dictionary: sorted, so 'PROMO%' is a contiguous code range.
P_TYPES = sorted(" ".join(t) for t in itertools.product(_SYL1, _SYL2, _SYL3))
# c_mktsegment dictionary (TPC-H spec §4.2.2.13) [EXT], sorted
SEGMENTS = ["AUTOMOBILE", "BUILDING", "FURNITURE", "HOUSEHOLD", "MACHINERY"]


def _load():
    global _lib
    if _lib is None:
        if not os.path.exists(_LIB_PATH):
            raise RuntimeError(f"{_LIB_PATH} missing: run `make` (or __graft_entry__.build())")
        lib = ctypes.CDLL(_LIB_PATH)
        d, u64, i64 = ctypes.c_double, ctypes.c_uint64, ctypes.c_int64
        P = ctypes.c_void_p
        lib.tg_sizes.argtypes = [d, P]
        lib.tg_gen_part.argtypes = [d, u64, P, P, P]
        lib.tg_gen_supplier.argtypes = [d, u64, P, P]
        lib.tg_gen_customer.argtypes = [d, u64, P, P, P]
        lib.tg_gen_partsupp.argtypes = [d, u64, P, P, P]
        lib.tg_gen_orders.argtypes = [d, u64, i64, i64, P, P, P]
        lib.tg_lineitem_count.argtypes = [d, u64, i64, i64]
        lib.tg_lineitem_count.restype = i64
        lib.tg_gen_lineitem.argtypes = [d, u64, i64, i64] + [P] * 8
        lib.tg_date_add_days.argtypes = [ctypes.c_int32, ctypes.c_int32]
        lib.tg_date_add_days.restype = ctypes.c_int32
        _lib = lib
    return _lib


def _ptr(a: np.ndarray):
    return ctypes.c_void_p(a.ctypes.data)


def sizes(sf: float) -> dict:
    out = np.zeros(5, dtype=np.int64)
    _load().tg_sizes(sf, _ptr(out))
    return dict(zip(["part", "supplier", "partsupp", "customer", "orders"], map(int, out)))


def date_add_days(yyyymmdd: int, ndays: int) -> int:
    return int(_load().tg_date_add_days(yyyymmdd, ndays))


def order_range(sf: float, rank: int = 0, world: int = 1) -> tuple[int, int]:
    """Contiguous order-index shard [b, e) of rank `rank` out of `world`."""
    o = sizes(sf)["orders"]
    return o * rank // world, o * (rank + 1) // world


@dataclass
class Database:
    sf: float
    seed: int
    rank: int = 0
    world: int = 1
    tables: dict = field(default_factory=dict)  # table -> {column -> np.ndarray}

    # string dictionaries (code -> string)
    n_name = [n for n, _ in NATIONS]
    r_name = REGIONS
    p_type = P_TYPES
    c_mktsegment = SEGMENTS

    def nrows(self, table: str) -> int:
        cols = self.tables[table]
        return len(next(iter(cols.values())))


LINEITEM_COLS = ["l_orderkey", "l_partkey", "l_suppkey", "l_quantity", "l_extendedprice",
                 "l_discount", "l_tax", "l_shipdate"]
_LI_TYPES = [np.int32, np.int32, np.int32, np.int64, np.int64, np.int64, np.int64, np.int32]


def generate(sf: float, seed: int = DEFAULT_SEED, rank: int = 0, world: int = 1,
             tables=None, lineitem_cols=None) -> Database:
    """Generate a TPC-H-shaped database.

    Dimension tables (region, nation, supplier, customer, part, partsupp) are
    generated whole; orders and lineitem only for this rank's contiguous
    order-key shard: lineitem is generated per order, so the
    shard boundary falls on order boundaries and the orders shard holds every
    order its lineitems reference.
    """
    lib = _load()
    sz = sizes(sf)
    want = set(tables) if tables else {"region", "nation", "supplier", "customer", "part",
                                       "partsupp", "orders", "lineitem"}
    db = Database(sf=sf, seed=seed, rank=rank, world=world)
    if "region" in want:
        db.tables["region"] = {"r_regionkey": np.arange(5, dtype=np.int32),
                               "r_name": np.arange(5, dtype=np.int32)}
    if "nation" in want:
        db.tables["nation"] = {"n_nationkey": np.arange(25, dtype=np.int32),
                               "n_name": np.arange(25, dtype=np.int32),
                               "n_regionkey": np.array([r for _, r in NATIONS], dtype=np.int32)}
    if "part" in want:
        n = sz["part"]
        a, b, c = np.empty(n, np.int32), np.empty(n, np.int32), np.empty(n, np.int64)
        lib.tg_gen_part(sf, seed, _ptr(a), _ptr(b), _ptr(c))
        db.tables["part"] = {"p_partkey": a, "p_type": b, "p_retailprice": c}
    if "supplier" in want:
        n = sz["supplier"]
        a, b = np.empty(n, np.int32), np.empty(n, np.int32)
        lib.tg_gen_supplier(sf, seed, _ptr(a), _ptr(b))
        db.tables["supplier"] = {"s_suppkey": a, "s_nationkey": b}
    if "customer" in want:
        n = sz["customer"]
        a, b, c = np.empty(n, np.int32), np.empty(n, np.int32), np.empty(n, np.int32)
        lib.tg_gen_customer(sf, seed, _ptr(a), _ptr(b), _ptr(c))
        db.tables["customer"] = {"c_custkey": a, "c_nationkey": b, "c_mktsegment": c}
    if "partsupp" in want:
        n = sz["partsupp"]
        a, b, c = np.empty(n, np.int32), np.empty(n, np.int32), np.empty(n, np.int64)
        lib.tg_gen_partsupp(sf, seed, _ptr(a), _ptr(b), _ptr(c))
        db.tables["partsupp"] = {"ps_partkey": a, "ps_suppkey": b, "ps_supplycost": c}
    ob, oe = order_range(sf, rank, world)
    if "orders" in want:
        n = oe - ob
        a, b, c = np.empty(n, np.int32), np.empty(n, np.int32), np.empty(n, np.int32)
        lib.tg_gen_orders(sf, seed, ob, oe, _ptr(a), _ptr(b), _ptr(c))
        db.tables["orders"] = {"o_orderkey": a, "o_custkey": b, "o_orderdate": c}
    if "lineitem" in want:
        n = int(lib.tg_lineitem_count(sf, seed, ob, oe))
        cols = lineitem_cols or LINEITEM_COLS
        arrs = {}
        ptrs = []
        for name, t in zip(LINEITEM_COLS, _LI_TYPES):
            if name in cols:
                arrs[name] = np.empty(n, t)
                ptrs.append(_ptr(arrs[name]))
            else:
                ptrs.append(ctypes.c_void_p(0))
        lib.tg_gen_lineitem(sf, seed, ob, oe, *ptrs)
        db.tables["lineitem"] = arrs
    return db
