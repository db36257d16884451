/*
 * tpchgen.c — seeded, shardable TPC-H-shaped data generator.
 *
 * This module is INPUT GENERATION ONLY. It holds none of the method's
 * arithmetic (no filters, joins, hashing or aggregation) and is shared by the
 * CPU oracle (oracle/), the tests and bench.py, which is the one thing the task
 * allows the oracle and the CUDA path to share.
 *
 * Shapes follow SURVEY.md Appendix B (TPC-H spec shapes; exact dbgen
 * compatibility is not required because parity is oracle-vs-GPU on the same
 * bytes). The paper ran dbgen data at SF 0.1-10 (§5.1; P:424,
 * §5.4); there is no network, so the data is generated here.
 *
 * Every value is a pure function of (seed, stream, counter): a counter-based
 * splitmix64 RNG. Output is therefore identical under any thread count and
 * any sharding of the order range ("rank r of R generates orders
 * [O*r/R, O*(r+1)/R) and exactly their lineitems").
 *
 * Column encodings (SURVEY.md §8 conventions):
 *   keys, dict codes, dates -> int32 (dates as yyyymmdd)
 *   decimals               -> int64 scaled by 100 (price, cost, quantity,
 *                             discount and tax in per cent: 0.05 -> 5)
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#define TG_API __attribute__((visibility("default")))

/* RNG streams (one per generated attribute). */
enum {
  S_PTYPE = 1, S_SNAT, S_CNAT, S_PSCOST, S_OCUST, S_ODATE,
  S_LCNT, S_LPART, S_LSUPP, S_LQTY, S_LDISC, S_LTAX, S_LSHIP,
  S_CSEG /* appended: earlier streams (and their bytes) are unchanged */
};

static inline uint64_t sm64(uint64_t x) {
  x += 0x9E3779B97F4A7C15ull;
  x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
  x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
  return x ^ (x >> 31);
}
static inline uint64_t rnd(uint64_t seed, uint32_t stream, uint64_t ctr) {
  return sm64(sm64(seed * 0xD1B54A32D192ED03ull + stream) ^ ctr);
}
/* uniform integer in [0, n) */
static inline uint32_t uni(uint64_t seed, uint32_t stream, uint64_t ctr, uint32_t n) {
  return (uint32_t)(((rnd(seed, stream, ctr) >> 32) * (uint64_t)n) >> 32);
}

/* ---- calendar (civil date <-> day number), data encoding only ---- */
static int64_t days_from_civil(int64_t y, unsigned m, unsigned d) {
  y -= m <= 2;
  const int64_t era = (y >= 0 ? y : y - 399) / 400;
  const unsigned yoe = (unsigned)(y - era * 400);
  const unsigned doy = (153 * (m + (m > 2 ? -3 : 9)) + 2) / 5 + d - 1;
  const unsigned doe = yoe * 365 + yoe / 4 - yoe / 100 + doy;
  return era * 146097 + (int64_t)doe - 719468;
}
static int32_t yyyymmdd_from_days(int64_t z) {
  z += 719468;
  const int64_t era = (z >= 0 ? z : z - 146096) / 146097;
  const unsigned doe = (unsigned)(z - era * 146097);
  const unsigned yoe = (doe - doe / 1460 + doe / 36524 - doe / 146096) / 365;
  int64_t y = (int64_t)yoe + era * 400;
  const unsigned doy = doe - (365 * yoe + yoe / 4 - yoe / 100);
  const unsigned mp = (5 * doy + 2) / 153;
  const unsigned d = doy - (153 * mp + 2) / 5 + 1;
  const unsigned m = mp < 10 ? mp + 3 : mp - 9;
  y += (m <= 2);
  return (int32_t)(y * 10000 + m * 100 + d);
}

TG_API int32_t tg_date_add_days(int32_t yyyymmdd, int32_t ndays) {
  int64_t dn = days_from_civil(yyyymmdd / 10000, (yyyymmdd / 100) % 100, yyyymmdd % 100);
  return yyyymmdd_from_days(dn + ndays);
}

/* ---- cardinalities ---- */
static int64_t scaled(double sf, double base, int64_t minimum) {
  int64_t n = (int64_t)(sf * base + 0.5);
  return n < minimum ? minimum : n;
}
/* out[0..4] = part, supplier, partsupp, customer, orders */
TG_API void tg_sizes(double sf, int64_t* out) {
  out[0] = scaled(sf, 200000.0, 1);
  out[1] = scaled(sf, 10000.0, 4); /* >= 4 so the 4 partsupp suppliers are distinct */
  out[2] = out[0] * 4;
  out[3] = scaled(sf, 150000.0, 3);
  out[4] = scaled(sf, 1500000.0, 1);
}

/* p_retailprice in cents (TPC-H formula). */
static inline int64_t retailprice(int64_t pk) {
  return 90000 + ((pk / 10) % 20001) + 100 * (pk % 1000);
}
/* supplier j (0..3) of part pk: distinct for S >= 4. */
static inline int32_t ps_supp(int64_t pk, int j, int64_t S) {
  return (int32_t)(((pk - 1) + (int64_t)j * (S / 4)) % S + 1);
}

TG_API void tg_gen_part(double sf, uint64_t seed, int32_t* p_partkey, int32_t* p_type,
                        int64_t* p_retailprice) {
  int64_t sz[5];
  tg_sizes(sf, sz);
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < sz[0]; i++) {
    int64_t pk = i + 1;
    p_partkey[i] = (int32_t)pk;
    p_type[i] = (int32_t)uni(seed, S_PTYPE, (uint64_t)i, 150);
    p_retailprice[i] = retailprice(pk);
  }
}

TG_API void tg_gen_supplier(double sf, uint64_t seed, int32_t* s_suppkey, int32_t* s_nationkey) {
  int64_t sz[5];
  tg_sizes(sf, sz);
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < sz[1]; i++) {
    s_suppkey[i] = (int32_t)(i + 1);
    s_nationkey[i] = (int32_t)uni(seed, S_SNAT, (uint64_t)i, 25);
  }
}

/* c_mktsegment: uniform over the 5 TPC-H market segments (dictionary codes of
 * the sorted segment names); NULL = not generated. */
TG_API void tg_gen_customer(double sf, uint64_t seed, int32_t* c_custkey, int32_t* c_nationkey,
                            int32_t* c_mktsegment) {
  int64_t sz[5];
  tg_sizes(sf, sz);
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < sz[3]; i++) {
    c_custkey[i] = (int32_t)(i + 1);
    c_nationkey[i] = (int32_t)uni(seed, S_CNAT, (uint64_t)i, 25);
    if (c_mktsegment) c_mktsegment[i] = (int32_t)uni(seed, S_CSEG, (uint64_t)i, 5);
  }
}

TG_API void tg_gen_partsupp(double sf, uint64_t seed, int32_t* ps_partkey, int32_t* ps_suppkey,
                            int64_t* ps_supplycost) {
  int64_t sz[5];
  tg_sizes(sf, sz);
  const int64_t S = sz[1];
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < sz[2]; i++) {
    int64_t pk = i / 4 + 1;
    int j = (int)(i % 4);
    ps_partkey[i] = (int32_t)pk;
    ps_suppkey[i] = ps_supp(pk, j, S);
    ps_supplycost[i] = 100 + (int64_t)uni(seed, S_PSCOST, (uint64_t)i, 99901);
  }
}

/* Order index i -> o_orderkey: sparse, "first 8 of every 32" (TPC-H). */
static inline int32_t orderkey_of(int64_t i) { return (int32_t)((i / 8) * 32 + (i % 8) + 1); }

static int32_t orderdate_of(uint64_t seed, int64_t i) {
  static const int64_t lo_days = 8035; /* days_from_civil(1992,1,1) */
  /* [1992-01-01, 1998-12-31 - 151 days] */
  const int64_t hi_days = 10591 - 151; /* days_from_civil(1998,12,31) = 10591 */
  int64_t d = lo_days + uni(seed, S_ODATE, (uint64_t)i, (uint32_t)(hi_days - lo_days + 1));
  return yyyymmdd_from_days(d);
}

TG_API void tg_gen_orders(double sf, uint64_t seed, int64_t o_begin, int64_t o_end,
                          int32_t* o_orderkey, int32_t* o_custkey, int32_t* o_orderdate) {
  int64_t sz[5];
  tg_sizes(sf, sz);
  const int64_t C = sz[3];
  const int64_t n_valid = C - C / 3; /* customers with custkey % 3 != 0 */
#pragma omp parallel for schedule(static)
  for (int64_t i = o_begin; i < o_end; i++) {
    int64_t k = i - o_begin;
    o_orderkey[k] = orderkey_of(i);
    int64_t m = uni(seed, S_OCUST, (uint64_t)i, (uint32_t)n_valid);
    o_custkey[k] = (int32_t)((m / 2) * 3 + (m % 2) + 1);
    o_orderdate[k] = orderdate_of(seed, i);
  }
}

static inline int lines_of(uint64_t seed, int64_t i) { return 1 + (int)uni(seed, S_LCNT, (uint64_t)i, 7); }

/* Number of lineitem rows generated for orders [o_begin, o_end). */
TG_API int64_t tg_lineitem_count(double sf, uint64_t seed, int64_t o_begin, int64_t o_end) {
  (void)sf;
  int64_t total = 0;
#pragma omp parallel for reduction(+ : total) schedule(static)
  for (int64_t i = o_begin; i < o_end; i++) total += lines_of(seed, i);
  return total;
}

/* Lineitem rows of orders [o_begin, o_end), clustered by orderkey (generated
 * per order).  Any column pointer may be NULL to skip it. */
TG_API void tg_gen_lineitem(double sf, uint64_t seed, int64_t o_begin, int64_t o_end,
                            int32_t* l_orderkey, int32_t* l_partkey, int32_t* l_suppkey,
                            int64_t* l_quantity, int64_t* l_extendedprice, int64_t* l_discount,
                            int64_t* l_tax, int32_t* l_shipdate) {
  int64_t sz[5];
  tg_sizes(sf, sz);
  const int64_t P = sz[0], S = sz[1];
  const int64_t n = o_end - o_begin;
  if (n <= 0) return;
  int64_t* off = (int64_t*)malloc(sizeof(int64_t) * (size_t)(n + 1));
  /* blocked prefix sum of per-order line counts */
  int nt = 1;
#ifdef _OPENMP
  nt = omp_get_max_threads();
#endif
  int64_t* part = (int64_t*)calloc((size_t)nt + 1, sizeof(int64_t));
#pragma omp parallel num_threads(nt)
  {
    int t = 0;
#ifdef _OPENMP
    t = omp_get_thread_num();
#endif
    int64_t b = n * t / nt, e = n * (t + 1) / nt, s = 0;
    for (int64_t k = b; k < e; k++) { off[k] = s; s += lines_of(seed, o_begin + k); }
    part[t + 1] = s;
#pragma omp barrier
#pragma omp single
    for (int u = 0; u < nt; u++) part[u + 1] += part[u];
    for (int64_t k = b; k < e; k++) off[k] += part[t];
  }
  off[n] = part[nt];
  free(part);

#pragma omp parallel for schedule(static)
  for (int64_t k = 0; k < n; k++) {
    const int64_t i = o_begin + k;
    const int32_t okey = orderkey_of(i);
    const int32_t odate = orderdate_of(seed, i);
    const int64_t cnt = off[k + 1] - off[k];
    for (int64_t j = 0; j < cnt; j++) {
      const int64_t r = off[k] + j;
      const uint64_t c = (uint64_t)i * 8 + (uint64_t)j;
      const int64_t pk = 1 + uni(seed, S_LPART, c, (uint32_t)P);
      const int64_t qty = 1 + uni(seed, S_LQTY, c, 50);
      if (l_orderkey) l_orderkey[r] = okey;
      if (l_partkey) l_partkey[r] = (int32_t)pk;
      if (l_suppkey) l_suppkey[r] = ps_supp(pk, (int)uni(seed, S_LSUPP, c, 4), S);
      if (l_quantity) l_quantity[r] = qty * 100;
      if (l_extendedprice) l_extendedprice[r] = qty * retailprice(pk);
      if (l_discount) l_discount[r] = uni(seed, S_LDISC, c, 11);
      if (l_tax) l_tax[r] = uni(seed, S_LTAX, c, 9);
      if (l_shipdate) l_shipdate[r] = tg_date_add_days(odate, 1 + (int32_t)uni(seed, S_LSHIP, c, 121));
    }
  }
  free(off);
}
