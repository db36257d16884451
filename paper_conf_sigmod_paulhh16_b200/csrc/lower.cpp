// lower.cpp — semantic validation of parsed segments and lowering to the
// device descriptors (BuildDesc / PipeDesc). Host only.
#include "lower.h"

#include "kernels.h"

#include <algorithm>
#include <cmath>
#include <map>
#include <set>

namespace gpl {
namespace {

bool is_int32(const Column& c) { return c.width == 4; }

struct Range {
  long double lo, hi;
};
Range mul(Range a, Range b) {
  long double c[4] = {a.lo * b.lo, a.lo * b.hi, a.hi * b.lo, a.hi * b.hi};
  return {*std::min_element(c, c + 4), *std::max_element(c, c + 4)};
}

// Zone restriction (SURVEY §7 "zone maps for build scans"): a range filter on
// a column that is sorted (non-decreasing, recorded at load: partsupp by
// ps_partkey, part by p_partkey, orders by o_orderkey, lineitem by l_orderkey)
// selects one contiguous row range, so only that range is scanned. The bounds
// are two binary searches (device, one small synchronous read-back at plan
// preparation; host-only contexts search their host copy). Filters still run
// on every scanned row, so the result does not depend on the restriction.
gpl_status sorted_range(gpl_ctx* ctx, const Table& T, const std::vector<FilterIR>& filters, int64_t* r0, int64_t* r1,
                        std::string* err) {
  *r0 = 0;
  *r1 = T.nrows;
  if (ctx->opt.zone_restrict == 0) return GPL_OK;
  for (const FilterIR& F : filters) {
    const Column* c = T.find(F.col);
    if (!c || !c->sorted || F.kind != F_RANGE || T.nrows == 0) continue;
    if (F.lo <= c->vmin && F.hi >= c->vmax) continue;  // passes every row
    long long b[2] = {0, T.nrows};
    if (ctx->host_only) {
      auto v = [&](int64_t i) {
        return c->width == 4 ? (long long)((const int32_t*)c->host.data())[i] : ((const int64_t*)c->host.data())[i];
      };
      int64_t a = 0, e = T.nrows;
      while (a < e) { const int64_t m = (a + e) / 2; if (v(m) < F.lo) a = m + 1; else e = m; }
      b[0] = a;
      e = T.nrows;
      while (a < e) { const int64_t m = (a + e) / 2; if (v(m) <= F.hi) a = m + 1; else e = m; }
      b[1] = a;
    } else {
      if (!ctx->d_bounds) {
        if (cudaMalloc(&ctx->d_bounds, 16) != cudaSuccess) { *err = "bounds scratch"; return GPL_E_NOMEM; }
      }
      cudaError_t e = launch_sorted_bounds(c->dev, c->width, T.nrows, F.lo, F.hi, ctx->d_bounds, ctx->stream);
      if (e == cudaSuccess) e = cudaMemcpyAsync(b, ctx->d_bounds, 16, cudaMemcpyDeviceToHost, ctx->stream);
      if (e == cudaSuccess) e = cudaStreamSynchronize(ctx->stream);
      if (e != cudaSuccess) { *err = std::string("zone bounds: ") + cudaGetErrorString(e); return GPL_E_CUDA; }
    }
    *r0 = std::max<int64_t>(*r0, b[0]);
    *r1 = std::min<int64_t>(*r1, b[1]);
  }
  *r0 &= ~(int64_t)3;  // 4-row aligned: 16-B aligned TMA sources for every column width
  if (*r1 < *r0) *r1 = *r0;
  return GPL_OK;
}

}  // namespace

int64_t next_pow2(int64_t x) {
  int64_t p = 1;
  while (p < x) p <<= 1;
  return p;
}

HTHeader trivial_header(int64_t count, long long kmin, long long kmax, int64_t cap_slots, int load_pct) {
  HTHeader h{};
  uint64_t need = ((uint64_t)count * 100ull + (uint64_t)load_pct - 1) / (uint64_t)load_pct;
  uint32_t log2 = 4;
  while ((1ull << log2) < need) log2++;
  while ((1ll << log2) > cap_slots && log2 > 4) log2--;
  uint64_t nslots = 1ull << log2;
  if (count == 0) kmin = kmax = 0;
  uint64_t range = (uint64_t)(kmax - kmin) + 1ull;
  h.count = (unsigned long long)count;
  h.kmin = kmin;
  h.kmax = kmax;
  h.mult = (nslots << 32) / range;
  h.log2 = log2;
  h.mask = (uint32_t)(nslots - 1);
  h.acc_count = 0;
  h.acc_kmin = INT64_MAX;
  h.acc_kmax = INT64_MIN;
  h.done = 0;
  return h;
}

gpl_status lower_build(gpl_ctx* ctx, const Segment& s, BuildDesc* d, HashTable* shape, bool* trivial,
                       std::string* err) {
  *d = BuildDesc{};
  auto tit = ctx->tables.find(s.table);
  if (tit == ctx->tables.end()) { *err = "unknown table '" + s.table + "'"; return GPL_E_STATE; }
  const Table& T = tit->second;
  std::vector<const Column*> cols;
  std::map<std::string, int> cidx;
  std::map<std::string, int> slot_of;  // slot name -> probe index
  for (size_t p = 0; p < s.probes.size(); p++)
    if (!s.probes[p].out.empty()) {
      if (T.find(s.probes[p].out)) { *err = "slot '" + s.probes[p].out + "' shadows a column"; return GPL_E_PLAN; }
      if (slot_of.count(s.probes[p].out)) { *err = "slot '" + s.probes[p].out + "' defined twice"; return GPL_E_PLAN; }
      slot_of[s.probes[p].out] = (int)p;
    }
  auto col = [&](const std::string& n, int* out) -> gpl_status {
    auto it = cidx.find(n);
    if (it != cidx.end()) { *out = it->second; return GPL_OK; }
    const Column* c = T.find(n);
    if (!c) { *err = "unknown column '" + n + "' in table " + T.name; return GPL_E_STATE; }
    if ((int)cols.size() >= MAXC) { *err = "too many columns"; return GPL_E_PLAN; }
    cidx[n] = (int)cols.size();
    cols.push_back(c);
    *out = cidx[n];
    return GPL_OK;
  };
  gpl_status st;
  d->nfilt = (int)s.filters.size();
  for (int f = 0; f < d->nfilt; f++) {
    const FilterIR& F = s.filters[f];
    int ci;
    if ((st = col(F.col, &ci))) return st;
    d->filt[f] = Filt{F.kind, ci, F.lo, F.hi, F.mask};
  }
  std::map<int, int> ht_slot;  // ht id -> index in d->src
  d->nprobe = (int)s.probes.size();
  std::vector<const HashTable*> src_ht(d->nprobe);
  for (int p = 0; p < d->nprobe; p++) {
    const ProbeIR& P = s.probes[p];
    auto hit = ctx->ht_by_name.find(P.ht);
    if (hit == ctx->ht_by_name.end()) { *err = "unknown hash table '" + P.ht + "'"; return GPL_E_STATE; }
    const HashTable& H = ctx->hts[hit->second];
    if (!H.valid) { *err = "hash table '" + P.ht + "' is stale (its table was reloaded)"; return GPL_E_STATE; }
    if (P.kind == P_MARK) { *err = "'mark' is not allowed in a build segment"; return GPL_E_PLAN; }
    if (H.kind == HT_MULTI) { *err = "a 'multi' table is probed by an inner 'probe' of a probe segment"; return GPL_E_PLAN; }
    if (H.kind == HT_PART) { *err = "'" + P.ht + "' is a partitioned table (scan it with 'run')"; return GPL_E_PLAN; }
    if ((int)P.keys.size() != H.key_arity) { *err = "key arity mismatch probing " + P.ht; return GPL_E_PLAN; }
    if (!P.out.empty() && !H.has_payload) { *err = P.ht + " has no payload to bind to '" + P.out + "'"; return GPL_E_PLAN; }
    int k1, k2 = -1;
    if ((st = col(P.keys[0], &k1))) return st;
    if (P.keys.size() == 2 && (st = col(P.keys[1], &k2))) return st;
    if (!is_int32(*cols[k1]) || (k2 >= 0 && !is_int32(*cols[k2]))) { *err = "probe keys must be 32-bit columns"; return GPL_E_PLAN; }
    if (!ht_slot.count(H.id)) {
      int i = (int)ht_slot.size();
      ht_slot[H.id] = i;
      d->src[i] = H.ref();
    }
    d->probe[p] = Probe{ht_slot[H.id], P.kind, k1, k2, p};
    src_ht[p] = &H;
  }
  d->nht = (int)ht_slot.size();
  if (s.key.size() > 2) { *err = "at most 2 key columns"; return GPL_E_PLAN; }
  if ((st = col(s.key[0], &d->k1))) return st;
  d->k2 = -1;
  if (s.key.size() == 2 && (st = col(s.key[1], &d->k2))) return st;
  if (!is_int32(*cols[d->k1]) || (d->k2 >= 0 && !is_int32(*cols[d->k2]))) { *err = "build keys must be 32-bit columns"; return GPL_E_PLAN; }
  shape->key_arity = (int)s.key.size();
  shape->has_payload = s.payload.kind != RefIR::CONST;
  shape->pay_min = shape->pay_max = 1;
  d->pay_kind = PAY_NONE;
  if (shape->has_payload) {
    if (s.payload.kind == RefIR::YEARCOL) {
      if ((st = col(s.payload.name, &d->pay_ref))) return st;
      if (!is_int32(*cols[d->pay_ref])) { *err = "year() needs a 32-bit date column"; return GPL_E_PLAN; }
      d->pay_kind = PAY_YEARCOL;
      shape->pay_min = cols[d->pay_ref]->vmin / 10000;
      shape->pay_max = cols[d->pay_ref]->vmax / 10000;
    } else if (slot_of.count(s.payload.name)) {
      int p = slot_of[s.payload.name];
      d->pay_kind = PAY_SLOT;
      d->pay_ref = p;
      shape->pay_min = src_ht[p]->pay_min;
      shape->pay_max = src_ht[p]->pay_max;
    } else {
      if ((st = col(s.payload.name, &d->pay_ref))) return st;
      d->pay_kind = PAY_COL;
      shape->pay_min = cols[d->pay_ref]->vmin;
      shape->pay_max = cols[d->pay_ref]->vmax;
    }
    // the segment's filters on the payload's column bound the inserted values
    // (Q5: c_nationkey in the nations of ASIA -> [8, 21], so 4-bit cells)
    if (d->pay_kind == PAY_COL || d->pay_kind == PAY_YEARCOL)
      for (const FilterIR& F : s.filters) {
        if (F.col != s.payload.name) continue;
        long long lo = F.lo, hi = F.hi;
        if (F.kind == F_MASK) {
          if (!F.mask) continue;
          lo = __builtin_ctzll(F.mask);
          hi = 63 - __builtin_clzll(F.mask);
        } else if (F.kind != F_RANGE) {
          continue;
        }
        if (d->pay_kind == PAY_YEARCOL) {  // yyyymmdd dates -> years
          lo = lo == INT64_MIN ? lo : lo / 10000;
          hi = hi == INT64_MAX ? hi : hi / 10000;
        }
        if (std::max<long long>(lo, shape->pay_min) <= std::min<long long>(hi, shape->pay_max)) {
          shape->pay_min = std::max<long long>(lo, shape->pay_min);
          shape->pay_max = std::min<long long>(hi, shape->pay_max);
        }
      }
  }
  int load = ctx->opt.hash_load_pct > 0 ? (int)ctx->opt.hash_load_pct : s.load_pct;
  if (shape->key_arity == 2) shape->kind = HT_MAP64;
  else shape->kind = shape->has_payload ? HT_MAP32 : HT_SET32;
  if (!s.multi && shape->kind == HT_MAP32 && (shape->pay_min < INT32_MIN || shape->pay_max > INT32_MAX)) {
    *err = "payload range does not fit the 32-bit payload of a single-key table";
    return GPL_E_OVERFLOW;
  }
  shape->hash = shape->kind == HT_MAP64 ? H_MULT : std::max(s.hash, 0);
  if (s.multi) {
    // non-unique key (NEXT-4 fan-out join): CSR over the key column's dense
    // domain — offsets[nslots + 1] + an int32 payload per qualifying row
    if (shape->key_arity != 1) { *err = "'multi' tables take a single key column"; return GPL_E_PLAN; }
    if (shape->has_payload && (shape->pay_min < INT32_MIN || shape->pay_max > INT32_MAX)) {
      *err = "a 'multi' payload must fit 32 bits";
      return GPL_E_OVERFLOW;
    }
    const Column* kc = cols[d->k1];
    const long long kmin = T.nrows ? kc->vmin : 0, kmax = T.nrows ? kc->vmax : 0;
    const unsigned long long range = (unsigned long long)(kmax - kmin) + 1ull;
    if (range > (1ull << 31) || T.nrows >= (1ll << 32)) { *err = "'multi' key domain too large"; return GPL_E_PLAN; }
    shape->kind = HT_MULTI;
    shape->hash = 0;
    shape->width = 4;
    shape->dkmin = kmin;
    shape->dnslots = range;
    shape->pay_base = 0;
    if (!shape->has_payload) shape->pay_min = shape->pay_max = 1;
  }

  // DIRECT (collision-free) addressing over a dense key domain: single int32
  // key, domain [min, max] of the key column, cells just wide enough for the
  // payload range. Chosen when its size is modest or within 2x of the hashed
  // table's upper-bound size (explicit 'hash mult|ordered' keeps hashing).
  if (!s.multi && shape->key_arity == 1 && (s.hash == -1 || s.hash == 2)) {
    const Column* kc = cols[d->k1];
    long long kmin = T.nrows ? kc->vmin : 0, kmax = T.nrows ? kc->vmax : 0;
    // a range filter on the key column itself bounds the inserted keys: the
    // domain shrinks to it (Q9: p_partkey < 1000 -> a 1000-bit set instead of
    // one bit per part), so the table can live in shared memory
    for (const FilterIR& F : s.filters)
      if (F.col == s.key[0] && F.kind == F_RANGE && T.nrows) {
        kmin = std::max<long long>(kmin, F.lo);
        kmax = std::min<long long>(kmax, F.hi);
      }
    if (kmax < kmin) kmax = kmin;
    const unsigned long long range = (unsigned long long)(kmax - kmin) + 1ull;
    int width = -1;
    if (!shape->has_payload) width = 0;
    else {
      // cell values 1..(pay_max - pay_min + 1), 0 = empty: 4-bit cells when they
      // fit (nation keys of a region, years), else the narrowest byte width
      const unsigned long long prange = (unsigned long long)(shape->pay_max - shape->pay_min) + 2ull;
      width = prange <= 0x10ull && ctx->opt.nibble_cells != 0 ? W_NIBBLE
              : prange <= 0xFFull ? 1 : prange <= 0xFFFFull ? 2 : prange <= 0xFFFFFFFFull ? 4 : -1;
    }
    if (width >= 0 && range <= (1ull << 31)) {
      const unsigned long long dbytes = width == 0 ? (range + 31) / 32 * 4 : width == W_NIBBLE ? (range + 1) / 2 : range * width;
      const unsigned long long hbytes = (unsigned long long)std::max<int64_t>(16, next_pow2((T.nrows * 100 + load - 1) / load)) *
                                        (shape->has_payload ? 8ull : 4ull);
      if (s.hash == 2 || dbytes <= (64ull << 20) || dbytes <= 2 * hbytes) {
        shape->kind = HT_DIRECT;
        shape->width = width;
        shape->dkmin = kmin;
        shape->dnslots = range;
        shape->pay_base = shape->has_payload ? shape->pay_min : 0;
      }
    }
    if (s.hash == 2 && shape->kind != HT_DIRECT) { *err = "'hash direct' needs a single key and a bounded payload range"; return GPL_E_PLAN; }
  }
  d->ncols = (int)cols.size();
  for (int c = 0; c < d->ncols; c++) {
    d->col[c] = cols[c]->dev;
    d->colw[c] = cols[c]->width;
  }
  d->nrows = T.nrows;
  {  // scan only the row range the sorted filter columns allow
    int64_t r0, r1;
    if ((st = sorted_range(ctx, T, s.filters, &r0, &r1, err))) return st;
    for (int c = 0; c < d->ncols; c++) d->col[c] += r0 * d->colw[c];
    d->nrows = r1 - r0;
  }
  d->kind = shape->kind;
  d->hash = shape->hash;
  d->load_pct = load;
  d->width = shape->width;
  d->kmin = shape->dkmin;
  d->nslots = shape->dnslots;
  d->pay_base = shape->pay_base;
  d->cap_slots = std::max<int64_t>(16, next_pow2((T.nrows * 100 + load - 1) / load));
  shape->cap_slots = d->cap_slots;
  shape->src_table = T.name;
  shape->src_version = T.version;
  *trivial = s.filters.empty() && s.probes.empty();
  return GPL_OK;
}

gpl_status lower_probe(gpl_ctx* ctx, const Segment& s, int split, PipeDesc* d, LowerInfo* li, std::string* err,
                       const HashTable* ins) {
  *d = PipeDesc{};
  *li = LowerInfo{};
  li->table = s.table;
  const bool part = s.is_build && s.is_partition;  // partition phase (NEXT-4 partitioned hash join)
  if (s.is_build && !ins && !part) { *err = "expected a probe segment ('run TABLE')"; return GPL_E_PLAN; }
  if (part && (!s.wheres.empty() || (int)s.probes.size() > MAXSP))
    { *err = "a partition segment takes filters and at most 2 probes"; return GPL_E_PLAN; }
  d->cl_probe = d->cl_col = -1;
  d->fan_probe = -1;
  if (ins && (!s.is_build || ins->kind != HT_DIRECT || s.key.size() != 1)) {
    *err = "pipelined build needs a single-key DIRECT build segment";
    return GPL_E_PLAN;
  }
  auto tit = ctx->tables.find(s.table);
  if (tit == ctx->tables.end()) { *err = "unknown table '" + s.table + "'"; return GPL_E_STATE; }
  const Table& T = tit->second;
  const int np = (int)s.probes.size();

  // slots
  std::map<std::string, int> slot_of;
  for (int p = 0; p < np; p++)
    if (!s.probes[p].out.empty()) {
      const std::string& o = s.probes[p].out;
      if (T.find(o)) { *err = "slot '" + o + "' shadows a column"; return GPL_E_PLAN; }
      if (slot_of.count(o)) { *err = "slot '" + o + "' defined twice"; return GPL_E_PLAN; }
      slot_of[o] = p;
    }
  // hash tables
  std::vector<const HashTable*> pht(np);
  std::map<int, int> ht_slot;
  for (int p = 0; p < np; p++) {
    const ProbeIR& P = s.probes[p];
    auto hit = ctx->ht_by_name.find(P.ht);
    if (hit == ctx->ht_by_name.end()) { *err = "unknown hash table '" + P.ht + "'"; return GPL_E_STATE; }
    const HashTable& H = ctx->hts[hit->second];
    if (!H.valid) { *err = "hash table '" + P.ht + "' is stale (its table was reloaded)"; return GPL_E_STATE; }
    if (H.kind == HT_PART) { *err = "'" + P.ht + "' is a partitioned table (scan it with 'run')"; return GPL_E_PLAN; }
    if ((int)P.keys.size() != H.key_arity) { *err = "key arity mismatch probing " + P.ht; return GPL_E_PLAN; }
    if (P.kind == P_INNER && !P.out.empty() && !H.has_payload) {
      *err = P.ht + " has no payload to bind to '" + P.out + "' (use semi or mark)";
      return GPL_E_PLAN;
    }
    if (H.kind == HT_MULTI) {  // non-unique build key: a fan-out inner join (NEXT-4)
      if (P.kind != P_INNER || ins) { *err = "a 'multi' table is probed by an inner 'probe' of a probe segment"; return GPL_E_PLAN; }
      if (d->fan_probe >= 0) { *err = "at most one fan-out probe (into a 'multi' table) per segment"; return GPL_E_PLAN; }
      d->fan_probe = p;
    }
    pht[p] = &H;
    if (!ht_slot.count(H.id)) {
      int i = (int)ht_slot.size();
      if (i >= MAXHT) { *err = "too many hash tables"; return GPL_E_PLAN; }
      ht_slot[H.id] = i;
      d->ht[i] = H.ref();
      li->ht_bytes.push_back((int64_t)(H.kind == HT_DIRECT ? H.bytes() : H.bytes() / 2));
      li->ht_ids.push_back(H.id);
    }
    li->probe_ht.push_back(ht_slot[H.id]);
  }
  d->nht = (int)ht_slot.size();
  // small DIRECT tables live in shared memory for the kernel's lifetime
  // (offsets relative to the tables region; apply_config makes them absolute)
  {
    int off = 0;
    for (int i = 0; i < MAXHT; i++) d->ht_smem_off[i] = -1, d->ht_smem_bytes[i] = 0;
    for (int i = 0; i < d->nht; i++) {
      const HashTable& H = ctx->hts[li->ht_ids[i]];
      const int b = (int)((H.bytes() + 15) / 16 * 16);
      if (H.kind == HT_DIRECT && b <= kSmemTableMax && off + b <= kSmemTablesTotal) {
        d->ht_smem_off[i] = off;
        d->ht_smem_bytes[i] = b;
        off += b;
      }
    }
    d->smem_tables_bytes = off;
  }

  // staged columns
  std::vector<const Column*> cols;
  std::map<std::string, int> cidx;
  // a partitioned (derived) table holds its key and the source row id; any other
  // column of the source table is *indirect*: gathered through the row id (lazy)
  const Table* src = nullptr;
  if (T.derived) {
    auto si = ctx->tables.find(T.src_table);
    if (si == ctx->tables.end()) { *err = "the source table of '" + T.name + "' is not loaded"; return GPL_E_STATE; }
    src = &si->second;
  }
  std::set<int> ind_col;  // indices (in cols) of indirect columns
  auto stage = [&](const std::string& n, int* out) -> gpl_status {
    auto it = cidx.find(n);
    if (it != cidx.end()) { *out = it->second; return GPL_OK; }
    const Column* c = T.find(n);
    bool ind = false;
    if (!c && src && (c = src->find(n))) ind = true;
    if (!c) { *err = "unknown column or slot '" + n + "'"; return GPL_E_STATE; }
    if ((int)cols.size() >= MAXC) { *err = "too many columns (max 8)"; return GPL_E_PLAN; }
    cidx[n] = (int)cols.size();
    if (ind) ind_col.insert((int)cols.size());
    cols.push_back(c);
    *out = cidx[n];
    return GPL_OK;
  };
  gpl_status st;
  int tmp;
  for (auto& f : s.filters) {
    if ((st = stage(f.col, &tmp))) return st;
    if (ind_col.count(tmp)) { *err = "filter on '" + f.col + "': filter the source in the partition segment"; return GPL_E_PLAN; }
  }
  // probes keyed by an earlier probe's slot (a chained join, e.g. partsupp ->
  // supplier) run in the queue phase, where slots are queue fields
  int first_queue_only = np;
  for (int p = 0; p < np; p++)
    for (auto& k : s.probes[p].keys) {
      if (slot_of.count(k)) {
        if (slot_of[k] >= p || s.probes[slot_of[k]].kind == P_MARK || pht[slot_of[k]]->kind == HT_MAP64) {
          *err = "probe key slot '" + k + "' must be a 32-bit payload of an earlier probe";
          return GPL_E_PLAN;
        }
        first_queue_only = std::min(first_queue_only, p);
        continue;
      }
      if ((st = stage(k, &tmp))) return st;
      if (!is_int32(*cols[tmp])) { *err = "probe key '" + k + "' must be a 32-bit column"; return GPL_E_PLAN; }
      if (ind_col.count(tmp)) first_queue_only = std::min(first_queue_only, p);  // gathered in the drain
    }
  if (d->fan_probe >= 0) first_queue_only = std::min(first_queue_only, d->fan_probe);
  if (ins && first_queue_only < np) { *err = "a pipelined build cannot probe by a slot"; return GPL_E_PLAN; }
  for (auto& g : s.groups)
    if (!slot_of.count(g.ref.name)) {
      if ((st = stage(g.ref.name, &tmp))) return st;
      if (g.ref.kind == RefIR::YEARCOL && !is_int32(*cols[tmp])) { *err = "year() needs a 32-bit date column"; return GPL_E_PLAN; }
    } else if (g.ref.kind == RefIR::YEARCOL) {
      *err = "year() takes a column";
      return GPL_E_PLAN;
    }
  for (auto& t : s.value)
    for (auto& f : t.f)
      if (f.x.kind != RefIR::CONST && !slot_of.count(f.x.name))
        if ((st = stage(f.x.name, &tmp))) return st;
  for (auto& w : s.wheres) {
    if (!slot_of.count(w.a) || (w.kind == R_EQ || w.kind == R_PAIRS ? !slot_of.count(w.b) : false)) {
      *err = "where refers to an unknown slot";
      return GPL_E_PLAN;
    }
  }
  for (auto& a : s.aggs)
    if (a.kind >= A_SUMIF && !slot_of.count(a.slot)) { *err = "agg condition refers to unknown slot '" + a.slot + "'"; return GPL_E_PLAN; }
  const bool pay_slot = ins && ins->has_payload && slot_of.count(s.payload.name);
  if (part) {  // the partition key is staged
    if ((st = stage(s.key[0], &tmp))) return st;
    if (!is_int32(*cols[tmp])) { *err = "partition keys must be 32-bit columns"; return GPL_E_PLAN; }
  }
  if (ins) {  // build key and payload columns are staged too
    if ((st = stage(s.key[0], &tmp))) return st;
    if (!is_int32(*cols[tmp])) { *err = "build keys must be 32-bit columns"; return GPL_E_PLAN; }
    if (ins->has_payload && !pay_slot && (st = stage(s.payload.name, &tmp))) return st;
  }

  // split (probes run before the survivor queue)
  int sp = split;
  if (sp < 0 && s.split_hint >= -1) sp = s.split_hint;
  if (sp < 0) sp = s.filters.empty() ? std::min(1, np) : 0;
  sp = std::min(std::min(std::min(sp, np), MAXSP), first_queue_only);

  // Late materialisation (the paper's k_reduce fetches
  // LINEITEM only for the satisfied tuples). A column used only after
  // selective operators is *lazy*: not TMA-staged; the survivor queue carries
  // the row id and the drain gathers the column from HBM for its (up to) 128
  // queued rows at once. It pays one 32-B sector per surviving row instead of
  // its width per scanned row, so it is chosen when (rows reaching the queue /
  // rows) * 64 <= width, from the previous run's pass fractions λ. In auto mode
  // a stage-phase probe whose key column qualifies moves to the queue phase.
  std::set<std::string> lazy;
  std::map<std::string, int> lazy_at;  // lazy column -> queue probe it is gathered before (np: the tail)
  const int nf0 = (int)s.filters.size();
  // (not in build segments: measured on B200, SF 100 Q5 HT_O, a late-gathered
  // build key costs a dependent gather per packet for the dense zero fill's
  // boundary keys, 0.45 -> 0.62 ms)
  if (!ins && !part && !T.derived && ctx->opt.lazy_columns != 0 && T.nrows < (1ll << 31)) {
    auto lit = ctx->lambda.find(s.text);
    const std::vector<double>* lam =
        lit != ctx->lambda.end() && (int)lit->second.size() >= nf0 + np ? &lit->second : nullptr;
    const bool force = ctx->opt.lazy_columns > 0;
    std::set<std::string> filter_cols;
    for (auto& f : s.filters) filter_cols.insert(f.col);
    auto worthy = [&](const std::string& c, int op) {
      if (filter_cols.count(c) || op < 0) return false;
      if (force) return true;
      return lam && (*lam)[op] * 64.0 <= (double)cols[cidx[c]]->width;
    };
    if (!force)
      for (int p = 0; p < sp; p++) {
        bool moved = false;
        for (auto& k : s.probes[p].keys) moved |= worthy(k, nf0 + p - 1);
        if (moved) {
          sp = p;
          break;
        }
      }
    std::set<std::string> stage_cols;  // read in the stage phase (filters, stage-probe keys)
    for (auto& f : s.filters) stage_cols.insert(f.col);
    for (int p = 0; p < sp; p++)
      for (auto& k : s.probes[p].keys) stage_cols.insert(k);
    // a lazy column is gathered right before its first use in the queue phase
    // (a queue probe's key, else the group-by / value after every probe and
    // residual), for the rows alive there: its cost is one sector per row
    // reaching that point (the pass count of the op before it)
    const int nops_all = nf0 + np + (int)s.wheres.size();
    auto reach_op = [&](int at) { return at < np ? nf0 + at - 1 : nops_all - 1; };
    std::map<std::string, int> first_use;  // queue-phase column -> its first use point
    auto use = [&](const std::string& c, int at) {
      if (slot_of.count(c) || stage_cols.count(c)) return;
      auto it = first_use.find(c);
      if (it == first_use.end() || at < it->second) first_use[c] = at;
    };
    for (int p = sp; p < np; p++)
      for (auto& k : s.probes[p].keys) use(k, p);
    for (auto& g : s.groups) use(g.ref.name, np);
    for (auto& t : s.value)
      for (auto& f : t.f)
        if (f.x.kind != RefIR::CONST) use(f.x.name, np);
    for (auto& [c, at] : first_use)
      if (worthy(c, reach_op(at))) {
        lazy.insert(c);
        lazy_at[c] = at;
      }
    for (auto& c : lazy) {
      li->lazy_w.push_back(cols[cidx[c]]->width);
      li->lazy_reach.push_back(reach_op(lazy_at[c]));
    }
  }

  if (src) {  // every indirect column is gathered by row id right before its first use
    const int nops_all = nf0 + np + (int)s.wheres.size();
    auto first = [&](const std::string& c) {
      int at = np;
      for (int p = sp; p < np; p++)
        for (auto& k : s.probes[p].keys)
          if (k == c) at = std::min(at, p);
      return at;
    };
    for (int c : ind_col) {
      std::string name;
      for (auto& kv : cidx)
        if (kv.second == c) name = kv.first;
      lazy.insert(name);
      lazy_at[name] = first(name);
      li->lazy_w.push_back(cols[c]->width);
      const int at = lazy_at[name];
      li->lazy_reach.push_back(at < np ? nf0 + at - 1 : nops_all - 1);
    }
  }
  // Expression pushdown: a value term whose factors are all columns, constants
  // or stage-phase slots is computed before the queue and carried as one field
  // (not when a factor is a lazy column: the drain computes it after the gather).
  auto stage_avail = [&](const std::string& n) {
    return !lazy.count(n) && (!slot_of.count(n) || slot_of[n] < sp);
  };
  std::vector<bool> term_push(s.value.size(), false);
  for (size_t t = 0; t < s.value.size(); t++) {
    bool ok = true;
    for (auto& f : s.value[t].f)
      if (f.x.kind != RefIR::CONST && !stage_avail(f.x.name)) ok = false;
    term_push[t] = ok;
  }
  // queue fields: columns used in the queue phase, stage-probe slots, pushed
  // terms, then queue-probe slots (written in the queue phase)
  std::vector<std::string> qcols;
  auto need_col = [&](const std::string& n) {
    if (std::find(qcols.begin(), qcols.end(), n) == qcols.end()) qcols.push_back(n);
  };
  for (int p = sp; p < np; p++)
    for (auto& k : s.probes[p].keys)
      if (!slot_of.count(k)) need_col(k);
  for (auto& g : s.groups)
    if (!slot_of.count(g.ref.name)) need_col(g.ref.name);
  for (size_t t = 0; t < s.value.size(); t++)
    if (!term_push[t])
      for (auto& f : s.value[t].f)
        if (f.x.kind != RefIR::CONST && !slot_of.count(f.x.name)) need_col(f.x.name);
  std::set<std::string> used_slots;
  for (auto& w : s.wheres) {
    used_slots.insert(w.a);
    if (w.kind == R_EQ || w.kind == R_PAIRS) used_slots.insert(w.b);
  }
  for (auto& g : s.groups)
    if (slot_of.count(g.ref.name)) used_slots.insert(g.ref.name);
  for (size_t t = 0; t < s.value.size(); t++)
    if (!term_push[t])
      for (auto& f : s.value[t].f)
        if (f.x.kind != RefIR::CONST && slot_of.count(f.x.name)) used_slots.insert(f.x.name);
  for (auto& a : s.aggs)
    if (a.kind >= A_SUMIF) used_slots.insert(a.slot);
  for (auto& pr : s.probes)
    for (auto& k : pr.keys)
      if (slot_of.count(k)) used_slots.insert(k);
  if (ins) {
    need_col(s.key[0]);
    if (ins->has_payload) {
      if (pay_slot) used_slots.insert(s.payload.name);
      else need_col(s.payload.name);
    }
  }

  auto slot_width = [&](int p) { return (s.probes[p].kind != P_MARK && pht[p]->kind == HT_MAP64) ? 8 : 4; };
  std::map<std::string, int> field;
  std::vector<int> fw;
  int nf = 0;
  for (int f = 0; f < MAXQ; f++) d->qlazy[f] = -1, d->qlazy_at[f] = np;
  d->rowid_field = -1;
  for (auto& c : qcols) {
    if (lazy.count(c)) continue;
    d->push[nf] = Push{PUSH_COL, cidx[c]};
    fw.push_back(cols[cidx[c]]->width);
    field[c] = nf++;
  }
  for (int p = 0; p < sp; p++) {
    const std::string& o = s.probes[p].out;
    if (!o.empty() && used_slots.count(o)) {
      if (nf >= MAXQ) { *err = "too many queue fields"; return GPL_E_PLAN; }
      d->push[nf] = Push{PUSH_SREG, p};
      fw.push_back(slot_width(p));
      field[o] = nf++;
    }
  }
  for (int t = 0; t < MAXTERM; t++) d->term_field[t] = -1;
  for (size_t t = 0; t < s.value.size(); t++)
    if (term_push[t]) {
      if (nf >= MAXQ) { *err = "too many queue fields"; return GPL_E_PLAN; }
      d->push[nf] = Push{PUSH_TERM, (int)t};
      d->term_field[t] = nf;
      fw.push_back(8);
      nf++;
    }
  if (!lazy.empty()) {  // the row id the drain gathers lazy columns by
    if (nf >= MAXQ) { *err = "too many queue fields"; return GPL_E_PLAN; }
    if (src) {  // a derived table: the source row id is a staged column
      int rc;
      if ((st = stage(T.rowid_col, &rc))) return st;
      d->push[nf] = Push{PUSH_COL, rc};
    } else {
      d->push[nf] = Push{PUSH_ROWID, 0};
    }
    fw.push_back(4);
    d->rowid_field = nf++;
  }
  d->npush = nf;
  for (auto& c : qcols) {  // lazy columns: queue fields filled by the drain's gather
    if (!lazy.count(c)) continue;
    if (nf >= MAXQ) { *err = "too many queue fields"; return GPL_E_PLAN; }
    d->qlazy[nf] = cidx[c];
    d->qlazy_at[nf] = lazy_at.count(c) ? lazy_at[c] : np;
    fw.push_back(cols[cidx[c]]->width);
    field[c] = nf++;
  }
  for (int p = sp; p < np; p++) {
    const std::string& o = s.probes[p].out;
    if (!o.empty() && used_slots.count(o)) {
      if (nf >= MAXQ) { *err = "too many queue fields"; return GPL_E_PLAN; }
      fw.push_back(slot_width(p));
      field[o] = nf++;
    }
  }
  if (nf > MAXQ) { *err = "too many queue fields"; return GPL_E_PLAN; }
  d->nfield = std::max(nf, 1);
  // the plan-specialised kernel keeps the fields the drain produces in
  // registers; only the pushed fields need warp-queue space (shared memory
  // then goes to a deeper ring / more CTAs per SM)
  d->reg_fields = ctx->opt.jit != 0 && ctx->opt.reg_fields != 0 && jit_available() ? 1 : 0;
  {
    int off = 0;
    for (int f = 0; f < nf; f++) {
      d->qoff[f] = off;
      d->qw[f] = fw[f];
      if (!d->reg_fields || f < d->npush) off += fw[f] * QCAP;
    }
    d->qbytes = std::max(off, 16);
  }

  if (part) {
    // partition phase: every probe in the stage phase, the sink reads the staged key
    if (sp != np) { *err = "partition segment probes must all run in the stage phase"; return GPL_E_PLAN; }
    auto hit = ctx->ht_by_name.find(s.by_ht);
    if (hit == ctx->ht_by_name.end()) { *err = "partition by unknown hash table '" + s.by_ht + "'"; return GPL_E_STATE; }
    const HashTable& PH = ctx->hts[hit->second];
    if (PH.kind != HT_DIRECT) { *err = "partition by a DIRECT (dense key domain) table"; return GPL_E_PLAN; }
    d->sink = SINK_PCOUNT;
    d->ins_kcol = cidx[s.key[0]];
    d->ins_pcol = d->ins_psreg = -1;
    d->nparts = s.nparts;
    int sh = 0;
    while (((unsigned long long)s.nparts << sh) < PH.dnslots) sh++;
    d->part_shift = sh;
    d->part_kmin = PH.dkmin;
    d->static_tiles = 1;
  }
  if (ins) {
    d->sink = SINK_INSERT;
    d->ins_kfield = field[s.key[0]];
    d->ins_pfield = ins->has_payload ? field[s.payload.name] : -1;
    d->ins_ptransform = ins->has_payload && s.payload.kind == RefIR::YEARCOL ? G_YEAR : G_ID;
    d->ins_width = ins->width;
    d->ins_kmin = ins->dkmin;
    d->ins_nslots = ins->dnslots;
    d->ins_pay_base = ins->pay_base;
    d->ins_pcol = d->ins_psreg = -1;
    d->ins_kcol = cidx[s.key[0]];  // staged (a dense build's zero fill reads it in the stage phase)
    d->ins_q = 1;
    if (sp == np && s.wheres.empty()) {  // every probe in the stage phase: insert from the staged tile
      d->ins_q = 0;
      if (ins->has_payload) {
        if (pay_slot) d->ins_psreg = slot_of[s.payload.name];
        else d->ins_pcol = cidx[s.payload.name];
      }
    }
  }
  // slot value ranges (validator)
  auto slot_range = [&](const std::string& n) -> Range {
    int p = slot_of[n];
    if (s.probes[p].kind == P_MARK) return {0, 1};
    return {(long double)pht[p]->pay_min, (long double)pht[p]->pay_max};
  };
  auto ref_range = [&](const std::string& n) -> Range {
    if (slot_of.count(n)) return slot_range(n);
    const Column* c = cols[cidx[n]];
    return {(long double)c->vmin, (long double)c->vmax};
  };

  // filters (stage columns)
  d->nfilt = (int)s.filters.size();
  for (int f = 0; f < d->nfilt; f++) {
    const FilterIR& F = s.filters[f];
    d->filt[f] = Filt{F.kind, cidx[F.col], F.lo, F.hi, F.mask};
    li->op_names.push_back("filter " + F.col);
  }
  // probes
  d->nprobe = np;
  d->nsprobe = sp;
  for (int p = 0; p < np; p++) {
    const ProbeIR& P = s.probes[p];
    Probe& D = d->probe[p];
    D.ht = li->probe_ht[p];
    D.kind = P.kind;
    if (p < sp) {
      D.k1 = cidx[P.keys[0]];
      D.k2 = P.keys.size() == 2 ? cidx[P.keys[1]] : -1;
      D.out = -1;
    } else {
      D.k1 = field[P.keys[0]];
      D.k2 = P.keys.size() == 2 ? field[P.keys[1]] : -1;
      D.out = (!P.out.empty() && field.count(P.out)) ? field[P.out] : -1;
    }
    li->op_names.push_back(std::string(P.kind == P_INNER ? "probe " : P.kind == P_SEMI ? "semi " : "mark ") + P.ht);
  }
  // Clustered probe: the first stage-phase probe reads a DIRECT table (not
  // already in shared memory) by one key column that is sorted in the fact
  // table (lineitem.l_orderkey: lineitem is generated per order) -> the
  // producer stages each stage's cell range with the columns.
  if (!ins && sp >= 1 && ctx->opt.clustered != 0) {
    const Probe& P0 = d->probe[0];
    const HashTable& H0 = *pht[0];
    if (H0.kind == HT_DIRECT && P0.k2 < 0 && cols[P0.k1]->sorted && cols[P0.k1]->width == 4 &&
        d->ht_smem_off[P0.ht] < 0 && H0.bytes() < (1ull << 31)) {
      d->cl_probe = 0;
      d->cl_col = P0.k1;
      // cell buffer per slot: twice the column's average key span per row
      // (lineitem: ~1 order key per row), 1..4 keys per row; a stage whose
      // range is wider probes the table in memory instead (correct, slower)
      const Column& kc = *cols[P0.k1];
      const double kpr = T.nrows > 0 ? (double)(kc.vmax - kc.vmin + 1) / (double)T.nrows : 1.0;
      d->cl_kpr = (int)std::min(4.0, std::max(1.0, std::ceil(2.0 * kpr)));
      li->cl_bytes = (double)H0.bytes();  // the producer streams the table's cells once (bytes per launch)
    }
  }
  // where residuals
  d->nresid = (int)s.wheres.size();
  for (int r = 0; r < d->nresid; r++) {
    const WhereIR& W = s.wheres[r];
    Resid& R = d->resid[r];
    R = Resid{};
    R.kind = W.kind;
    R.a = field[W.a];
    R.b = (W.kind == R_EQ || W.kind == R_PAIRS) ? field[W.b] : -1;
    R.npairs = (int)W.pairs.size();
    for (int i = 0; i < R.npairs; i++) {
      R.pa[i] = (int32_t)W.pairs[i].first;
      R.pb[i] = (int32_t)W.pairs[i].second;
    }
    R.lo = W.lo;
    R.hi = W.hi;
    R.mask = W.mask;
    li->op_names.push_back("where " + W.a);
  }
  // group-by
  d->ngroup = (int)s.groups.size();
  int64_t G = 1;
  if (s.hash_group) {  // unbounded keys (NEXT-4): packed int32 fields, no domain
    for (int g = 0; g < d->ngroup; g++) {
      const GroupIR& Gi = s.groups[g];
      GroupDim& D = d->gdim[g];
      D.field = field[Gi.ref.name];
      D.transform = Gi.ref.kind == RefIR::YEARCOL ? G_YEAR : G_ID;
      D.lo = D.size = D.stride = 0;
      if (Gi.ref.kind != RefIR::YEARCOL) {
        const Range r = ref_range(Gi.ref.name);
        if (r.lo < INT32_MIN || r.hi > INT32_MAX) { *err = "group hash keys must be 32-bit values"; return GPL_E_PLAN; }
      }
    }
    li->hash_group = true;
  }
  // the result step (A10): ORDER BY / LIMIT (on the device for a hash
  // group-by, on the host at fetch for dense groups), key decodes, ratios
  li->limit = s.limit;
  li->norder = (int)s.order.size();
  for (int i = 0; i < li->norder; i++) {
    li->ord_is_agg[i] = s.order[i].is_agg;
    li->ord_idx[i] = s.order[i].idx;
    li->ord_desc[i] = s.order[i].desc;
  }
  for (const DecodeIR& dc : s.decodes) {
    auto dt = ctx->tables.find(dc.table);
    if (dt == ctx->tables.end()) { *err = "decode: unknown table " + dc.table; return GPL_E_STATE; }
    const Column* kc = dt->second.find(dc.keycol);
    const Column* oc = dt->second.find(dc.outcol);
    if (!kc || !oc) { *err = "decode: unknown column of " + dc.table; return GPL_E_STATE; }
    if (kc->width != 4 || oc->width != 4) { *err = "decode: columns must be 32-bit"; return GPL_E_PLAN; }
    if (dt->second.nrows > (1 << 20)) { *err = "decode: table larger than 2^20 rows"; return GPL_E_PLAN; }
  }
  li->decodes = s.decodes;
  li->ratios = s.ratios;
  for (int g = s.hash_group ? -1 : d->ngroup - 1; g >= 0; g--) {
    const GroupIR& Gi = s.groups[g];
    GroupDim& D = d->gdim[g];
    D.field = field[Gi.ref.name];
    D.transform = Gi.ref.kind == RefIR::YEARCOL ? G_YEAR : G_ID;
    D.lo = (int32_t)Gi.lo;
    D.size = (int32_t)(Gi.hi - Gi.lo);
    D.stride = (int32_t)G;
    G *= D.size;
    if (G > (1 << 16)) { *err = "group domain too large (max 65536 groups)"; return GPL_E_PLAN; }
    li->glo[g] = D.lo;
    li->gsize[g] = D.size;
    li->gstride[g] = D.stride;
  }
  d->ngroups_total = (int)G;
  li->ngroups_total = (int)G;
  li->ngroup_dims = d->ngroup;
  li->has_groups = d->ngroup > 0;
  // value
  d->nterm = (int)s.value.size();
  Range vr{0, 0};
  for (int t = 0; t < d->nterm; t++) {
    const TermIR& Ti = s.value[t];
    Term& D = d->term[t];
    Term& SD = d->sterm[t];
    D.sign = SD.sign = Ti.sign;
    D.nfact = SD.nfact = (int)Ti.f.size();
    Range tr{1, 1};
    for (int f = 0; f < D.nfact; f++) {
      const FactorIR& F = Ti.f[f];
      Factor& X = D.f[f];
      Factor& SX = SD.f[f];
      X.a = SX.a = F.a;
      X.b = SX.b = F.b;
      Range fr;
      if (F.x.kind == RefIR::CONST) {
        X.field = SX.field = SREF_CONST;
        X.b = SX.b = 0;
        fr = {(long double)F.a, (long double)F.a};
      } else {
        if (term_push[t]) {
          X.field = -1;
          SX.field = slot_of.count(F.x.name) ? -(slot_of[F.x.name] + 2) : cidx[F.x.name];
        } else {
          X.field = field[F.x.name];
          SX.field = SREF_CONST;
        }
        Range xr = ref_range(F.x.name);
        long double e1 = F.a + F.b * xr.lo, e2 = F.a + F.b * xr.hi;
        fr = {std::min(e1, e2), std::max(e1, e2)};
      }
      tr = mul(tr, fr);
    }
    if (Ti.sign < 0) tr = {-tr.hi, -tr.lo};
    vr = {vr.lo + tr.lo, vr.hi + tr.hi};
  }
  li->maxabs = std::max(std::fabs((double)vr.lo), std::fabs((double)vr.hi));
  if (li->maxabs >= 4.0e18L) {
    *err = "value expression may exceed exact int64 arithmetic per row (bound " + std::to_string((double)li->maxabs) + ")";
    return GPL_E_OVERFLOW;
  }
  // aggregates (agg 0 = COUNT)
  d->nagg = (int)s.aggs.size();
  for (int a = 0; a < d->nagg; a++) {
    const AggIR& A = s.aggs[a];
    d->agg[a] = Agg{A.kind, A.kind >= A_SUMIF ? field[A.slot] : -1, A.c};
  }
  li->nagg = d->nagg;
  // staged columns
  d->ncols = (int)cols.size();
  int bpr = 0, bpr_all = 0;
  for (int c = 0; c < d->ncols; c++) {
    d->col[c] = cols[c]->dev;
    d->colw[c] = cols[c]->width;
    d->lazy[c] = 0;
    bpr_all += cols[c]->width;
  }
  for (auto& c : lazy) d->lazy[cidx[c]] = 1;
  for (int c = 0; c < d->ncols; c++)
    if (!d->lazy[c]) bpr += cols[c]->width;
  li->bytes_per_row = bpr;
  li->bytes_per_row_all = bpr_all;
  d->nrows = T.nrows;
  // a partitioned (derived) table: its row count is written on the device by the partition phase
  d->nrows_dev = T.derived ? T.nrows_dev : nullptr;
  {  // scan only the row range the sorted filter columns allow (zone restriction)
    int64_t r0, r1;
    if ((st = sorted_range(ctx, T, s.filters, &r0, &r1, err))) return st;
    for (int c = 0; c < d->ncols; c++)
      if (!ind_col.count(c)) d->col[c] += r0 * d->colw[c];
    d->nrows = r1 - r0;
    d->part_row0 = r0;  // partition phase: row ids are absolute rows of the scanned table
    // clustered (dense) build: a DIRECT build whose key column is sorted and
    // fully scanned, with the domain exactly [min, max] of that column, writes
    // every cell of the domain exactly once (rows' cells + the gaps)
    d->ins_dense = 0;
    if (ins && d->ins_kcol >= 0 && ins->kind == HT_DIRECT && ins->width >= 1 && ctx->opt.dense_build != 0 &&
        T.nrows > 0 && r0 == 0 && r1 == T.nrows) {
      const Column& kc = *cols[d->ins_kcol];
      // strictly increasing: no duplicate key can exist, each row owns one cell
      if (kc.strict && ins->dkmin == kc.vmin && ins->dkmin + (long long)ins->dnslots - 1 == kc.vmax) d->ins_dense = 1;
    }
  }
  li->nfilt = d->nfilt;
  li->nprobe = np;
  li->nops = d->nfilt + np + d->nresid;
  // aggregation mode (exactness): per-row |value| <= maxabs, so any int64
  // accumulator covering <= R rows is exact when R * maxabs < 2^62.
  const long double lim = 4.6e18L;
  const long double total = (long double)std::max<int64_t>(T.nrows, 1) * std::max<long double>(li->maxabs, 1);
  if (s.hash_group) {  // one exact int64 accumulator per group and aggregate
    if (total >= lim) {
      *err = "hash group-by sums are int64: rows x max|value| may exceed 2^62";
      return GPL_E_OVERFLOW;
    }
    d->agg_mode = AGG_HASH;
    d->flush_each_tile = 0;
  } else if (d->ngroups_total == 1) {
    // a lane's register accumulator receives 4 rows of each 128-row packet (stage
    // phase) or of each 128-entry drain, so at most nrows / 32 + 8 rows over the
    // run; the warp's flush sums the lanes in 128 bits
    d->agg_mode = AGG_REG;
    const long double lane_total = ((long double)std::max<int64_t>(T.nrows, 1) / 32.0L + 8.0L) * std::max<long double>(li->maxabs, 1);
    d->flush_each_tile = lane_total >= lim ? 1 : 0;
  } else {
    d->agg_mode = (total < lim && (int64_t)d->ngroups_total * d->nagg * 8 <= 48 * 1024) ? AGG_SMEM : AGG_GLOBAL;
    d->flush_each_tile = 0;
  }
  // lane-private copies of a small shared-memory table (<= 16 KB for all 32):
  // lanes of a warp never collide on a word, only the same lane of other warps
  d->agg_lanes = d->agg_mode == AGG_SMEM && (int64_t)d->ngroups_total * d->nagg * 8 * 32 <= 16 * 1024 ? 32 : 1;
  // forced accumulator placement (tests): global int128 atomics are exact for
  // every plan; registers / the smem table only where the bound above allows
  if (!s.hash_group && ctx->opt.agg_mode == AGG_GLOBAL) {
    d->agg_mode = AGG_GLOBAL;
    d->flush_each_tile = 0;
  }
  if (part) {  // the per-CTA partition counts / cursors live in the shared table region
    d->agg_mode = AGG_SMEM;
    d->ngroups_total = li->ngroups_total = (s.nparts + 1) / 2;  // u64 words holding nparts u32
    d->nagg = li->nagg = 1;
    d->flush_each_tile = 0;
    d->agg_lanes = 1;
  }
  return GPL_OK;
}

}  // namespace gpl
