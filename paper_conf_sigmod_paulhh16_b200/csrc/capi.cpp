// capi.cpp — the extern "C" boundary (include/gpl.h). Argument checking,
// column store (A0), build/run orchestration on the ctx stream, result decode
// (A10). No exception crosses the ABI.
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <climits>
#include <cstring>
#include <new>
#include <limits>
#include <map>
#include <set>
#include <string>

#include "costmodel.h"
#include "ctx.h"
#include "gpl.h"
#include "kernels.h"
#include "lower.h"
#include "plan.h"

#define GPL_API extern "C" __attribute__((visibility("default")))

using namespace gpl;

namespace {

std::string g_create_error;

gpl_status fail(gpl_ctx* ctx, gpl_status st, const std::string& msg) {
  if (ctx) ctx->err = msg;
  else g_create_error = msg;
  return st;
}

#define CK(call)                                                                            \
  do {                                                                                      \
    cudaError_t e_ = (call);                                                                \
    if (e_ != cudaSuccess) return fail(ctx, GPL_E_CUDA, std::string(#call) + ": " + cudaGetErrorString(e_)); \
  } while (0)

int type_width(int t) {
  switch (t) {
    case GPL_I32: case GPL_DATE32: case GPL_DICT32: return 4;
    case GPL_I64: case GPL_DEC64: return 8;
    default: return 0;
  }
}

// Device scratch, one allocation so a run's outputs come back in ONE D2H copy:
//   word 0          error bits (u32), latched until fetched
//   word 1          tile counter (zeroed per run)
//   words 2..17     op_pass[MAXOPS]  (zeroed per run)
//   words 18..      int128 partials [groups][aggs] (zeroed per run)
// After a fused run a one-CTA kernel copies words [0, head + partials) into
// mapped pinned host memory (h_stage), so fetching needs no D2H copy node.
constexpr int kScratchHead = 2 + MAXOPS;
constexpr int kMinmaxSlots = 4096;  // column slots for pending loads' min/max
constexpr size_t kMaxPartialBytes = (size_t)(1 << 16) * MAXA * 16;
constexpr size_t kScratchBytes = kScratchHead * 8 + kMaxPartialBytes + MAXOPS * 8;  // + build op counters

unsigned int* err_ptr(gpl_ctx* ctx) { return (unsigned int*)ctx->d_scratch; }
unsigned long long* counter_ptr(gpl_ctx* ctx) { return ctx->d_scratch + 1; }
unsigned long long* op_pass_ptr(gpl_ctx* ctx) { return ctx->d_scratch + 2; }
// bytes of the per-run zeroed region (tile counter .. partials)
size_t run_clear_bytes(size_t pbytes) { return (1 + MAXOPS) * sizeof(unsigned long long) + pbytes; }
// the plan has a RunProfile taken on the current contents of its fact table
bool profile_current(const gpl_ctx* ctx, const std::string& text, const std::string& table) {
  auto it = ctx->profile.find(text);
  if (it == ctx->profile.end()) return false;
  auto ti = ctx->tables.find(table);
  return ti != ctx->tables.end() && ti->second.version == it->second.table_version && it->second.runs >= 2;
}

// per-run result bytes after the head: dense int128 partials, or for a hash
// group-by [distinct groups, rows out, LIMIT rows of (1 + nagg) words]
size_t run_pbytes(const LowerInfo& li) {
  if (li.hash_group) return ((size_t)(2 + li.limit * (1 + li.nagg)) * 8 + 15) / 16 * 16;
  return (size_t)li.ngroups_total * li.nagg * 16;
}
// words the result copy-out moves (error bits, counters, partials)
int result_words(size_t pbytes) { return kScratchHead + (int)(pbytes / 8); }
unsigned long long* partials_ptr(gpl_ctx* ctx) { return ctx->d_scratch + kScratchHead; }
// op counters of pipelined builds (written, never read)
unsigned long long* build_ops_ptr(gpl_ctx* ctx) { return ctx->d_scratch + kScratchHead + kMaxPartialBytes / 8; }
// a DIRECT table's pipelined build keeps its tile counter right after the
// cells, so the one memset that clears the table also resets the counter
size_t direct_counter_off(size_t bytes) { return (bytes + 15) / 16 * 16; }

gpl_status check_dev(gpl_ctx* ctx) {
  if (!ctx) return GPL_E_ARG;
  if (ctx->host_only) return fail(ctx, GPL_E_NODEV, "host-only context (device -1)");
  CK(cudaSetDevice(ctx->device));
  return GPL_OK;
}

void free_column(gpl_ctx* ctx, Column& c) {
  if (c.owned && c.dev && !ctx->host_only) cudaFree(c.dev);
  c.dev = nullptr;
}

// Read latched device error bits (syncs) and clear them.
gpl_status take_device_errors(gpl_ctx* ctx) {
  // pinned destination: a pageable D2H costs ~10 us more than the copy itself
  CK(cudaMemcpyAsync(ctx->h_err, err_ptr(ctx), sizeof(unsigned int), cudaMemcpyDeviceToHost, ctx->stream));
  CK(cudaStreamSynchronize(ctx->stream));
  const unsigned int bits = *ctx->h_err;
  if (bits) {
    CK(cudaMemsetAsync(err_ptr(ctx), 0, sizeof(unsigned int), ctx->stream));
    if (bits & ERR_DUPKEY) return fail(ctx, GPL_E_DUPKEY, "duplicate build key (joins must be FK->PK)");
    if (bits & ERR_RESERVED_KEY) return fail(ctx, GPL_E_ARG, "a build key equals the reserved empty-slot value");
    if (bits & ERR_DOMAIN) return fail(ctx, GPL_E_DOMAIN, "a group value fell outside its declared domain");
    return fail(ctx, GPL_E_CAPACITY, "device capacity error");
  }
  return GPL_OK;
}

// A10: the key -> output map of a 'decode' statement, read from the loaded
// table (one small D2H per table version; nation: 25 rows).
gpl_status decode_map(gpl_ctx* ctx, const DecodeIR& dc, const std::map<int32_t, int32_t>** out) {
  auto ti = ctx->tables.find(dc.table);
  if (ti == ctx->tables.end()) return fail(ctx, GPL_E_STATE, "decode: table " + dc.table + " is not loaded");
  const Table& T = ti->second;
  const std::string id = dc.table + "." + dc.keycol + "->" + dc.outcol;
  auto it = ctx->decode_maps.find(id);
  if (it != ctx->decode_maps.end() && it->second.first == T.version) {
    *out = &it->second.second;
    return GPL_OK;
  }
  const Column* kc = T.find(dc.keycol);
  const Column* oc = T.find(dc.outcol);
  if (!kc || !oc || kc->width != 4 || oc->width != 4) return fail(ctx, GPL_E_STATE, "decode: bad columns of " + dc.table);
  std::vector<int32_t> k(T.nrows), v(T.nrows);
  if (T.nrows) {
    if (ctx->host_only) {
      std::memcpy(k.data(), kc->host.data(), T.nrows * 4);
      std::memcpy(v.data(), oc->host.data(), T.nrows * 4);
    } else {
      CK(cudaMemcpyAsync(k.data(), kc->dev, T.nrows * 4, cudaMemcpyDeviceToHost, ctx->stream));
      CK(cudaMemcpyAsync(v.data(), oc->dev, T.nrows * 4, cudaMemcpyDeviceToHost, ctx->stream));
      CK(cudaStreamSynchronize(ctx->stream));
    }
  }
  std::map<int32_t, int32_t> m;
  for (int64_t i = 0; i < T.nrows; i++)
    if (!m.emplace(k[i], v[i]).second)
      return fail(ctx, GPL_E_DUPKEY, "decode: duplicate key in " + dc.table + "." + dc.keycol);
  auto& slot = ctx->decode_maps[id];
  slot.first = T.version;
  slot.second.swap(m);
  *out = &slot.second;
  return GPL_OK;
}

// A10 ratio columns: scale * double(num) / double(den), den = 0 -> NaN (SQL
// NULL); the IEEE sequence of reading R12, from the exact int128 sums.
void fill_ratios(const std::vector<RatioIR>& ratios, gpl_result* out, int rows) {
  out->n_ratios = (int32_t)ratios.size();
  if (!out->ratios) return;
  const int A = out->n_aggs;
  for (int r = 0; r < rows; r++)
    for (size_t j = 0; j < ratios.size(); j++) {
      auto get = [&](int a) {
        const unsigned __int128 u = ((unsigned __int128)(uint64_t)out->aggs[(r * A + a) * 2 + 1] << 64) |
                                    (uint64_t)out->aggs[(r * A + a) * 2];
        return (__int128)u;
      };
      const __int128 num = get(ratios[j].num), den = get(ratios[j].den);
      out->ratios[r * ratios.size() + j] =
          den == 0 ? std::numeric_limits<double>::quiet_NaN() : ratios[j].scale * (double)num / (double)den;
    }
}

// Dense partials -> result rows (A10 finalize, "ORDER BY is blocking";
// SURVEY §8(a) A10): drop empty groups, decode group ids to key values and
// through the plan's 'decode' tables, ORDER BY (ties: the decoded key tuple
// ascending, reading R8) else key order, LIMIT, ratio columns.
}  // namespace

// Read back the min/max/sortedness of every pending load (one event wait for
// the whole batch) and decide each reloaded table's version: unchanged shape
// (same rows, buffers and value ranges) keeps the old version.
gpl_status resolve_pending(gpl_ctx* ctx) {
  if (ctx->pending.empty()) return GPL_OK;
  CK(cudaEventSynchronize(ctx->mm_ev));
  for (PendingLoad& pl : ctx->pending) {
    auto it = ctx->tables.find(pl.table);
    if (it == ctx->tables.end()) continue;
    Table& t = it->second;
    const long long* mm = ctx->h_minmax + 4 * pl.slot0;
    for (int i = 0; i < pl.ncols && i < (int)t.cols.size(); i++) {
      t.cols[i].vmin = t.nrows ? mm[4 * i] : 0;
      t.cols[i].vmax = t.nrows ? mm[4 * i + 1] : 0;
      t.cols[i].sorted = mm[4 * i + 2] == 0;                        // no descent between consecutive rows
      t.cols[i].strict = t.cols[i].sorted && mm[4 * i + 3] == 0;   // ... and no two equal consecutive rows
    }
    if (pl.has_old) {
      const Table& o = pl.old_meta;
      bool same = o.nrows == t.nrows && o.cols.size() == t.cols.size();
      for (size_t i = 0; same && i < t.cols.size(); i++) {
        const Column& a = o.cols[i];
        const Column& b = t.cols[i];
        same = a.name == b.name && a.type == b.type && a.width == b.width && a.dev == b.dev && a.vmin == b.vmin &&
               a.vmax == b.vmax && a.cap_rows == b.cap_rows && a.sorted == b.sorted && a.strict == b.strict;
      }
      if (same) t.version = o.version;
    }
  }
  ctx->pending.clear();
  ctx->mm_next = 0;
  return GPL_OK;
}

namespace {

gpl_status decode(gpl_ctx* ctx, const unsigned long long* part, gpl_result* out) {
  const LowerInfo& li = ctx->last.run->li;
  const int G = li.ngroups_total, A = li.nagg, NK = li.ngroup_dims;
  out->n_keys = NK;
  out->n_aggs = A;
  out->n_ratios = (int32_t)li.ratios.size();
  struct Row {
    int32_t key[MAXG];
    int g;
  };
  std::vector<Row> rows;
  for (int g = 0; g < G; g++) {
    const bool nonempty = part[2 * (g * A)] != 0 || part[2 * (g * A) + 1] != 0;
    if (!nonempty && li.has_groups) continue;
    Row r{};
    r.g = g;
    for (int k = 0; k < NK; k++) r.key[k] = li.glo[k] + (g / li.gstride[k]) % li.gsize[k];
    rows.push_back(r);
  }
  for (const DecodeIR& dc : li.decodes) {
    const std::map<int32_t, int32_t>* m = nullptr;
    gpl_status st = decode_map(ctx, dc, &m);
    if (st) return st;
    for (Row& r : rows) {
      auto it = m->find(r.key[dc.key]);
      if (it == m->end())
        return fail(ctx, GPL_E_STATE, "decode: group key " + std::to_string(r.key[dc.key]) + " not in " + dc.table);
      r.key[dc.key] = it->second;
    }
  }
  auto agg = [&](const Row& r, int a) {
    return (__int128)(((unsigned __int128)part[2 * (r.g * A + a) + 1] << 64) | part[2 * (r.g * A + a)]);
  };
  std::sort(rows.begin(), rows.end(), [&](const Row& x, const Row& y) {
    for (int i = 0; i < li.norder; i++) {
      const __int128 a = li.ord_is_agg[i] ? agg(x, li.ord_idx[i]) : (__int128)x.key[li.ord_idx[i]];
      const __int128 b = li.ord_is_agg[i] ? agg(y, li.ord_idx[i]) : (__int128)y.key[li.ord_idx[i]];
      if (a != b) return li.ord_desc[i] ? a > b : a < b;
    }
    for (int k = 0; k < NK; k++)
      if (x.key[k] != y.key[k]) return x.key[k] < y.key[k];
    return false;
  });
  if (li.limit > 0 && (int)rows.size() > li.limit) rows.resize(li.limit);
  const int n = (int)rows.size();
  out->n_groups = n;
  if (n > out->cap_groups) return fail(ctx, GPL_E_CAPACITY, "result capacity too small");
  if (n && (!out->aggs || (NK && !out->keys))) return fail(ctx, GPL_E_ARG, "NULL result arrays");
  for (int r = 0; r < n; r++) {
    for (int k = 0; k < NK; k++) out->keys[r * NK + k] = rows[r].key[k];
    for (int a = 0; a < A; a++) {
      out->aggs[(r * A + a) * 2] = (int64_t)part[2 * (rows[r].g * A + a)];
      out->aggs[(r * A + a) * 2 + 1] = (int64_t)part[2 * (rows[r].g * A + a) + 1];
    }
  }
  fill_ratios(li.ratios, out, n);
  return GPL_OK;
}

// Hash group-by result (NEXT-4): LIMIT rows come back with the counters in
// ORDER BY order; without a LIMIT every group is copied from the device row
// buffer and ordered by key on the host (as the dense decode orders gids).
gpl_status decode_hash(gpl_ctx* ctx, const unsigned long long* part, gpl_result* out) {
  const LowerInfo& li = ctx->last.run->li;
  const int A = li.nagg, NK = li.ngroup_dims, W = 1 + A;
  const uint64_t nrows = part[1];
  out->n_keys = NK;
  out->n_aggs = A;
  out->n_ratios = (int32_t)li.ratios.size();
  out->n_groups = (int32_t)std::min<uint64_t>(nrows, INT32_MAX);
  if (nrows > (uint64_t)std::max(out->cap_groups, 0)) return fail(ctx, GPL_E_CAPACITY, "result capacity too small");
  if (nrows && (!out->aggs || !out->keys)) return fail(ctx, GPL_E_ARG, "NULL result arrays");
  std::vector<unsigned long long> rows;
  const unsigned long long* src = part + 2;
  if (li.limit == 0 && nrows) {
    // every group: the full ORDER BY (else key order) as a device sort of the
    // compacted rows (ORDER BY is blocking), then one D2H
    const size_t tb = sort_hagg_tmp_bytes(nrows);
    const size_t need = tb + ((size_t)nrows * W * 8 + 255) / 256 * 256;
    if (ctx->sort_alloc < need) {
      CK(cudaStreamSynchronize(ctx->stream));
      if (ctx->d_sort) cudaFree(ctx->d_sort);
      ctx->d_sort = nullptr;
      ctx->sort_alloc = 0;
      cudaError_t e = cudaMalloc(&ctx->d_sort, need);
      if (e != cudaSuccess) return fail(ctx, GPL_E_NOMEM, std::string("sort buffers: ") + cudaGetErrorString(e));
      ctx->sort_alloc = need;
    }
    unsigned long long* sorted = (unsigned long long*)((char*)ctx->d_sort + tb);
    CK(sort_hagg_rows(ctx->last.run->hres, ctx->last.run->hres.rows, nrows, sorted, ctx->d_sort, ctx->sms, ctx->stream));
    rows.resize((size_t)nrows * W);
    CK(cudaMemcpyAsync(rows.data(), sorted, rows.size() * 8, cudaMemcpyDeviceToHost, ctx->stream));
    CK(cudaStreamSynchronize(ctx->stream));
    src = rows.data();
  }
  for (uint64_t r = 0; r < nrows; r++) {
    const unsigned long long key = src[r * W];
    for (int k = 0; k < NK; k++)
      out->keys[r * NK + k] = NK == 2 ? (int32_t)(uint32_t)(k == 0 ? key >> 32 : key) : (int32_t)(uint32_t)key;
    for (int a = 0; a < A; a++) {
      const long long v = (long long)src[r * W + 1 + a];
      out->aggs[(r * A + a) * 2] = v;
      out->aggs[(r * A + a) * 2 + 1] = v < 0 ? -1 : 0;
    }
  }
  fill_ratios(li.ratios, out, (int)nrows);
  return GPL_OK;
}

}  // namespace

GPL_API const char* gpl_version(void) { return "gpl-b200 0.1 sm_100a"; }

GPL_API const char* gpl_last_error(const gpl_ctx* ctx) { return ctx ? ctx->err.c_str() : g_create_error.c_str(); }

GPL_API gpl_status gpl_create(int device, void* cuda_stream, gpl_ctx** out) {
  gpl_ctx* ctx = nullptr;
  if (!out) return fail(nullptr, GPL_E_ARG, "out is NULL");
  *out = nullptr;
  ctx = new (std::nothrow) gpl_ctx();
  if (!ctx) return fail(nullptr, GPL_E_NOMEM, "host allocation failed");
  if (device < 0) {
    ctx->host_only = true;
    *out = ctx;
    return GPL_OK;
  }
  ctx->host_only = false;
  ctx->device = device;
  auto bad = [&](cudaError_t e, const char* what) {
    std::string m = std::string(what) + ": " + cudaGetErrorString(e);
    delete ctx;
    return fail(nullptr, GPL_E_CUDA, m);
  };
  cudaError_t e;
  if ((e = cudaSetDevice(device)) != cudaSuccess) return bad(e, "cudaSetDevice");
  cudaDeviceProp p;
  if ((e = cudaGetDeviceProperties(&p, device)) != cudaSuccess) return bad(e, "cudaGetDeviceProperties");
  if (p.major < 10) {
    delete ctx;
    return fail(nullptr, GPL_E_CUDA, "device is not sm_100 class (this build targets sm_100a only)");
  }
  ctx->sms = p.multiProcessorCount;
  ctx->smem_optin = (int)p.sharedMemPerBlockOptin;
  ctx->l2_bytes = p.l2CacheSize;
  if (cuda_stream) {
    ctx->stream = (cudaStream_t)cuda_stream;
  } else {
    if ((e = cudaStreamCreateWithFlags(&ctx->stream, cudaStreamNonBlocking)) != cudaSuccess) return bad(e, "stream");
    ctx->own_stream = true;
  }
  if ((e = cudaMalloc(&ctx->d_scratch, kScratchBytes)) != cudaSuccess) return bad(e, "scratch");
  if ((e = cudaMemset(ctx->d_scratch, 0, kScratchBytes)) != cudaSuccess) return bad(e, "scratch");
  if ((e = cudaMallocHost(&ctx->h_stage, kScratchBytes)) != cudaSuccess) return bad(e, "pinned staging");
  ctx->h_stage_cap = kScratchBytes;
  if ((e = cudaHostGetDevicePointer((void**)&ctx->h_stage_dev, ctx->h_stage, 0)) != cudaSuccess)
    return bad(e, "mapped staging");
  if ((e = cudaMallocHost((void**)&ctx->h_err, 64)) != cudaSuccess) return bad(e, "pinned error word");
  if ((e = cudaMallocHost((void**)&ctx->h_minmax, kMinmaxSlots * 4 * sizeof(long long))) != cudaSuccess)
    return bad(e, "pinned min/max");
  if ((e = cudaEventCreate(&ctx->ev0)) != cudaSuccess) return bad(e, "event");
  if ((e = cudaEventCreate(&ctx->ev1)) != cudaSuccess) return bad(e, "event");
  *out = ctx;
  return GPL_OK;
}

GPL_API void gpl_destroy(gpl_ctx* ctx) {
  if (!ctx) return;
  if (!ctx->host_only) {
    cudaSetDevice(ctx->device);
    cudaStreamSynchronize(ctx->stream);
    if (ctx->mm_stream) cudaStreamSynchronize(ctx->mm_stream);  // min/max passes still reading columns
    for (auto& kv : ctx->tables)
      for (auto& c : kv.second.cols) free_column(ctx, c);
    for (auto& h : ctx->hts) {
      if (h.slots) cudaFree(h.slots);
      if (h.hdr) cudaFree(h.hdr);
      if (h.pay) cudaFree(h.pay);
      if (h.aux) cudaFree(h.aux);
      if (h.part_buf && h.part_buf != h.slots) cudaFree(h.part_buf);
    }
    if (ctx->d_scratch) cudaFree(ctx->d_scratch);
    for (auto& kv : ctx->graphs) cudaGraphExecDestroy(kv.second);
    for (auto& kv : ctx->kbe_graphs)
      if (kv.second.exec) cudaGraphExecDestroy(kv.second.exec);
    if (ctx->h_stage) cudaFreeHost(ctx->h_stage);
    if (ctx->h_err) cudaFreeHost(ctx->h_err);
    if (ctx->h_minmax) cudaFreeHost(ctx->h_minmax);
    if (ctx->d_minmax) cudaFree(ctx->d_minmax);
    if (ctx->d_bounds) cudaFree(ctx->d_bounds);
    if (ctx->d_kbe_bytes) cudaFree(ctx->d_kbe_bytes);
    if (ctx->kbe_buf) cudaFree(ctx->kbe_buf);
    if (ctx->d_hagg) cudaFree(ctx->d_hagg);
    if (ctx->d_hres) cudaFree(ctx->d_hres);
    if (ctx->d_hcand) cudaFree(ctx->d_hcand);
    if (ctx->d_sort) cudaFree(ctx->d_sort);
    if (ctx->side) cudaStreamDestroy(ctx->side);
    for (auto& e : ctx->fork_ev)
      if (e) cudaEventDestroy(e);
    if (ctx->ev0) cudaEventDestroy(ctx->ev0);
    if (ctx->ev1) cudaEventDestroy(ctx->ev1);
    if (ctx->mm_stream) cudaStreamSynchronize(ctx->mm_stream);
    if (ctx->mm_ev) cudaEventDestroy(ctx->mm_ev);
    for (auto& e : ctx->mm_col_ev)
      if (e) cudaEventDestroy(e);
    if (ctx->mm_stream) cudaStreamDestroy(ctx->mm_stream);
    if (ctx->own_stream) cudaStreamDestroy(ctx->stream);
  }
  delete ctx;
}

GPL_API gpl_status gpl_set_option(gpl_ctx* ctx, const char* key, int64_t value) {
  if (!ctx || !key) return GPL_E_ARG;
  std::string k = key;
  Options& o = ctx->opt;
  int64_t v = value;
  if (k == "stage_rows") {
    if (v >= 0 && (v % 128 || v < 128 || v > 8192)) return fail(ctx, GPL_E_ARG, "stage_rows: multiple of 128 in [128, 8192]");
    o.stage_rows = v;
  } else if (k == "ring_depth") {
    if (v >= 0 && (v < 2 || v > 8)) return fail(ctx, GPL_E_ARG, "ring_depth in [2, 8]");
    o.ring_depth = v;
  } else if (k == "consumer_warps") {
    if (v >= 0 && (v < 1 || v > 16)) return fail(ctx, GPL_E_ARG, "consumer_warps in [1, 16]");
    o.consumer_warps = v;
  } else if (k == "ctas_per_sm") {
    if (v >= 0 && (v < 1 || v > 4)) return fail(ctx, GPL_E_ARG, "ctas_per_sm in [1, 4]");
    o.ctas_per_sm = v;
  } else if (k == "packets") {
    if (v >= 0 && v != 1 && v != 2) return fail(ctx, GPL_E_ARG, "packets: 1 or 2");
    o.packets = v;
  } else if (k == "probe_split") {
    o.probe_split = v < -1 ? -2 : v;  // -1 = after every probe, >= 0 = count, < -1 auto
  } else if (k == "hash_load_pct") {
    if (v >= 0 && (v < 10 || v > 90)) return fail(ctx, GPL_E_ARG, "hash_load_pct in [10, 90]");
    o.hash_load_pct = v;
  } else if (k == "kbe_graph") {
    o.kbe_graph = v != 0 ? 1 : 0;
  } else if (k == "kbe_tile_rows") {
    if (v < 0) return fail(ctx, GPL_E_ARG, "kbe_tile_rows >= 0 (0 = whole input: KBE)");
    o.kbe_tile_rows = v;
  } else if (k == "lazy_columns") {
    o.lazy_columns = v < 0 ? -1 : v > 0 ? 1 : 0;
  } else if (k == "clustered") {
    o.clustered = v != 0 ? 1 : 0;
  } else if (k == "build_pipeline") {
    o.build_pipeline = v != 0 ? 1 : 0;
  } else if (k == "hash_slots_log2") {
    // slot indices are 32-bit in the ORDER BY/LIMIT selection (0xFFFFFFFF = none)
    if (v > 0 && (v < 12 || v > 31)) return fail(ctx, GPL_E_ARG, "hash_slots_log2 in [12, 31] (0 = auto)");
    o.hash_slots_log2 = v > 0 ? v : 0;
  } else if (k == "drain_warps") {
    if (v >= 0 && v > 4) return fail(ctx, GPL_E_ARG, "drain_warps in [0, 4] (-1 = model)");
    o.drain_warps = v < 0 ? -1 : v;
  } else if (k == "dense_build") {
    o.dense_build = v != 0 ? 1 : 0;
  } else if (k == "nibble_cells") {
    o.nibble_cells = v != 0 ? 1 : 0;
  } else if (k == "reg_fields") {
    o.reg_fields = v != 0 ? 1 : 0;
  } else if (k == "zone_restrict") {
    o.zone_restrict = v != 0 ? 1 : 0;
  } else if (k == "agg_mode") {
    if (v >= 0 && v != AGG_GLOBAL) return fail(ctx, GPL_E_ARG, "agg_mode: 2 (global int128 atomics) or -1 (auto)");
    o.agg_mode = v < 0 ? -1 : v;
  } else if (k == "graph_branches") {
    // only how whole-query graphs are recorded: drop them, keep plans and pinned shapes
    o.graph_branches = v != 0 ? 1 : 0;
    for (auto& kv : ctx->graphs) cudaGraphExecDestroy(kv.second);
    ctx->graphs.clear();
    return GPL_OK;
  } else if (k == "autotune_probe") {
    // only what gpl_autotune measures: plans and pinned shapes stay
    o.autotune_probe = v != 0 ? 1 : 0;
    return GPL_OK;
  } else if (k == "use_profile") {
    o.use_profile = v != 0 ? 1 : 0;
  } else if (k == "use_gamma") {
    o.use_gamma = v != 0 ? 1 : 0;
  } else if (k == "jit") {
    o.jit = v != 0 ? 1 : 0;
  } else if (k == "hbm_mbs") {
    o.hbm_gbs = v > 0 ? v / 1000.0 : -1;
  } else {
    return fail(ctx, GPL_E_ARG, "unknown option '" + k + "'");
  }
  ctx->opt_version++;
  ctx->tuned.clear();
  return GPL_OK;
}

GPL_API gpl_status gpl_load_columns(gpl_ctx* ctx, const char* table, int64_t nrows, int32_t ncols,
                                    const gpl_column* cols, uint32_t flags) {
  if (!ctx) return GPL_E_ARG;
  ctx->err.clear();
  if (!table || !*table) return fail(ctx, GPL_E_ARG, "table name is empty");
  if (nrows < 0 || nrows > ((int64_t)1 << 40)) return fail(ctx, GPL_E_ARG, "nrows out of range");
  if (ncols < 1 || ncols > 64 || !cols) return fail(ctx, GPL_E_ARG, "ncols must be in [1, 64] with a column array");
  if (flags != GPL_COPY && flags != GPL_BORROW) return fail(ctx, GPL_E_ARG, "flags must be GPL_COPY or GPL_BORROW");
  std::set<std::string> names;
  for (int i = 0; i < ncols; i++) {
    if (!cols[i].name || !*cols[i].name) return fail(ctx, GPL_E_ARG, "column name is empty");
    if (!names.insert(cols[i].name).second) return fail(ctx, GPL_E_ARG, std::string("duplicate column ") + cols[i].name);
    if (!type_width(cols[i].type)) return fail(ctx, GPL_E_ARG, std::string("bad type for column ") + cols[i].name);
    if (nrows > 0 && !cols[i].data) return fail(ctx, GPL_E_ARG, std::string("NULL data for column ") + cols[i].name);
    if (ctx->host_only && cols[i].on_device) return fail(ctx, GPL_E_NODEV, "device data given to a host-only context");
  }
  Table t;
  t.name = table;
  t.nrows = nrows;
  t.version = ctx->next_version++;
  if (ctx->host_only) {
    for (int i = 0; i < ncols; i++) {
      Column c;
      c.name = cols[i].name;
      c.type = cols[i].type;
      c.scale = cols[i].scale;
      c.width = type_width(c.type);
      c.host.assign((const char*)cols[i].data, (const char*)cols[i].data + nrows * c.width);
      c.vmin = LLONG_MAX;
      c.vmax = LLONG_MIN;
      c.sorted = true;
      c.strict = true;
      long long prev = LLONG_MIN;
      for (int64_t r = 0; r < nrows; r++) {
        long long v = c.width == 4 ? (long long)((const int32_t*)c.host.data())[r] : ((const int64_t*)c.host.data())[r];
        c.vmin = std::min<long long>(c.vmin, v);
        c.vmax = std::max<long long>(c.vmax, v);
        c.sorted = c.sorted && v >= prev;
        c.strict = c.strict && (r == 0 || v > prev);
        prev = v;
      }
      if (nrows == 0) c.vmin = c.vmax = 0;
      t.cols.push_back(std::move(c));
    }
  } else {
    gpl_status st = check_dev(ctx);
    if (st) return st;
    // a reload of a table whose previous load is still pending: resolve it first
    for (auto& pl : ctx->pending)
      if (pl.table == t.name) {
        if ((st = resolve_pending(ctx))) return st;
        break;
      }
    if (!ctx->d_minmax) {
      CK(cudaMalloc(&ctx->d_minmax, kMinmaxSlots * 4 * sizeof(long long)));
      ctx->minmax_cap = kMinmaxSlots;
    }
    if (!ctx->mm_ev) {
      CK(cudaEventCreateWithFlags(&ctx->mm_ev, cudaEventDisableTiming));
      CK(cudaStreamCreateWithFlags(&ctx->mm_stream, cudaStreamNonBlocking));
      for (auto& e : ctx->mm_col_ev) CK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    }
    if (ctx->mm_next + ncols > kMinmaxSlots && (st = resolve_pending(ctx))) return st;  // slots exhausted
    auto cleanup = [&]() {  // a failed reload hands reused buffers back to the old table
      auto oldt = ctx->tables.find(t.name);
      for (auto& c : t.cols) {
        bool given_back = false;
        if (oldt != ctx->tables.end())
          for (auto& oc : oldt->second.cols)
            if (oc.dev == c.dev && c.owned && !oc.owned) {
              oc.owned = true;
              given_back = true;
            }
        if (!given_back) free_column(ctx, c);
      }
    };
    for (int i = 0; i < ncols; i++) {
      Column c;
      c.name = cols[i].name;
      c.type = cols[i].type;
      c.scale = cols[i].scale;
      c.width = type_width(c.type);
      const int64_t need_cap = (nrows + 3) / 4 * 4;
      const int64_t cap = cols[i].capacity_rows > 0 ? cols[i].capacity_rows : nrows;
      bool borrow = flags == GPL_BORROW && cols[i].on_device && ((uintptr_t)cols[i].data % 16 == 0) && cap >= need_cap;
      if (flags == GPL_BORROW && !cols[i].on_device) {
        cleanup();
        return fail(ctx, GPL_E_ARG, std::string("GPL_BORROW needs device data: ") + c.name);
      }
      if (borrow) {
        c.dev = (char*)cols[i].data;
        c.owned = false;
        c.cap_rows = cap;
      } else {
        const int64_t rows = std::max<int64_t>(64, (nrows + 63) / 64 * 64);
        // reloading a table: reuse the old owned buffer of the same column when
        // it is large enough (stream order keeps earlier readers safe)
        Column* reuse = nullptr;
        auto oldt = ctx->tables.find(t.name);
        if (oldt != ctx->tables.end())
          for (auto& oc : oldt->second.cols)
            if (oc.name == c.name && oc.owned && oc.dev && oc.width == c.width && oc.cap_rows >= rows) reuse = &oc;
        if (reuse) {
          c.dev = reuse->dev;
          c.cap_rows = reuse->cap_rows;
          reuse->owned = false;  // ownership moves to the new column (dev kept for the same-shape check)
        } else {
          cudaError_t e = cudaMalloc(&c.dev, (size_t)rows * c.width);
          if (e != cudaSuccess) {
            cleanup();
            return fail(ctx, GPL_E_NOMEM, std::string("cudaMalloc for column ") + c.name + ": " + cudaGetErrorString(e));
          }
          c.cap_rows = rows;
        }
        c.owned = true;
        const int64_t cap_rows = c.cap_rows;
        t.cols.push_back(c);  // owned from here on (cleanup frees it)
        if (nrows > 0)
          CK(cudaMemcpyAsync(c.dev, cols[i].data, (size_t)nrows * c.width, cudaMemcpyDefault, ctx->stream));
        CK(cudaMemsetAsync(c.dev + (size_t)nrows * c.width, 0, (size_t)(std::min(cap_rows, rows + 64) - nrows) * c.width,
                           ctx->stream));
        t.cols.pop_back();
      }
      t.cols.push_back(c);
      // per-column min/max/sortedness on a side stream, as soon as the column
      // has landed: the pass overlaps the next columns' copies (the copy engine
      // and the SMs work at once), and nothing synchronises here — the pinned
      // slots are read by resolve_pending at the first call that plans
      const int slot = ctx->mm_next + i;
      CK(cudaEventRecord(ctx->mm_col_ev[i], ctx->stream));
      CK(cudaStreamWaitEvent(ctx->mm_stream, ctx->mm_col_ev[i], 0));
      const char* cp1 = c.dev;
      const int cw1 = c.width;
      CK(launch_minmax_cols(&cp1, &cw1, 1, nrows, ctx->d_minmax + 4 * slot, ctx->mm_stream));
    }
    const int slot0 = ctx->mm_next;
    CK(cudaMemcpyAsync(ctx->h_minmax + 4 * slot0, ctx->d_minmax + 4 * slot0, sizeof(long long) * 4 * ncols,
                       cudaMemcpyDeviceToHost, ctx->mm_stream));
    CK(cudaEventRecord(ctx->mm_ev, ctx->mm_stream));
    ctx->mm_next += ncols;
    PendingLoad pl;
    pl.table = t.name;
    pl.slot0 = slot0;
    pl.ncols = ncols;
    ctx->pending.push_back(std::move(pl));
  }
  auto old = ctx->tables.find(t.name);
  if (old != ctx->tables.end()) {
    // A reload into the same buffers with the same rows and value ranges keeps
    // the table's version (decided by resolve_pending once the min/max are
    // back): prepared plans and query graphs depend only on those (hash tables
    // built from it are still marked stale until rebuilt).
    if (!ctx->host_only) {
      PendingLoad& pl = ctx->pending.back();
      pl.has_old = true;
      pl.old_meta.name = old->second.name;
      pl.old_meta.nrows = old->second.nrows;
      pl.old_meta.version = old->second.version;
      for (const Column& oc : old->second.cols) {
        Column m = oc;
        m.host.clear();
        m.owned = false;
        pl.old_meta.cols.push_back(std::move(m));
      }
    }
    bool any_owned = false;
    for (auto& c : old->second.cols) any_owned |= c.owned && c.dev;
    if (!ctx->host_only && any_owned) cudaStreamSynchronize(ctx->stream);
    for (auto& c : old->second.cols) free_column(ctx, c);
    for (auto& h : ctx->hts)
      if (h.src_table == t.name) h.valid = false;
  }
  ctx->tables[t.name] = std::move(t);
  return GPL_OK;
}

GPL_API gpl_status gpl_check_plan(gpl_ctx* ctx, const char* segment) {
  if (!ctx || !segment) return GPL_E_ARG;
  if (gpl_status rs = resolve_pending(ctx)) return rs;  // loads still in flight (A0)
  ctx->err.clear();
  Segment s;
  std::string err;
  if (!parse_segment(segment, &s, &err)) return fail(ctx, GPL_E_PLAN, err);
  gpl_status st;
  if (s.is_build) {
    BuildDesc d;
    HashTable shape;
    bool trivial;
    st = lower_build(ctx, s, &d, &shape, &trivial, &err);
  } else {
    PipeDesc d;
    LowerInfo li;
    st = lower_probe(ctx, s, choose_split(ctx, s), &d, &li, &err);
  }
  return st ? fail(ctx, st, err) : GPL_OK;
}

// A prepared build is reusable while its scanned table, its destination and
// source hash tables and the options are unchanged.
// `rebuilt`: hash tables that the same query rebuilds before this segment
// runs (a whole-query graph replays every build), so their staleness after a
// same-shape table reload does not matter.
static bool build_cache_valid(gpl_ctx* ctx, const PreparedBuild& P, const std::set<int>* rebuilt = nullptr) {
  auto ti = ctx->tables.find(P.table);
  bool ok = ti != ctx->tables.end() && ti->second.version == P.table_version && P.opt_version == ctx->opt_version &&
            P.ht_index >= 0 && P.ht_index < (int)ctx->hts.size();
  if (ok) {
    const HTRef r = ctx->hts[P.ht_index].ref();
    ok = std::memcmp(&r, &P.dest_ref, sizeof(HTRef)) == 0;
  }
  for (size_t i = 0; ok && i < P.src_ids.size(); i++) {
    const HashTable& Hs = ctx->hts[P.src_ids[i]];
    const HTRef r = Hs.ref();
    ok = (Hs.valid || (rebuilt && rebuilt->count(Hs.id))) && std::memcmp(&r, &P.desc.src[i], sizeof(HTRef)) == 0;
  }
  return ok;
}

static bool run_cache_valid(gpl_ctx* ctx, const PreparedRun& P, const std::set<int>* rebuilt = nullptr) {
  auto lam = ctx->lambda.find(P.text);
  const size_t lambda_n = lam == ctx->lambda.end() ? 0 : lam->second.size();
  auto ti = ctx->tables.find(P.li.table);
  bool ok = ti != ctx->tables.end() && ti->second.version == P.table_version && P.opt_version == ctx->opt_version &&
            P.lambda_n == lambda_n && P.profiled == profile_current(ctx, P.text, P.li.table);
  if (ok && P.li.hash_group) {
    auto ge = ctx->hagg_groups.find(P.text);
    ok = P.desc.hagg_keys == ctx->d_hagg && P.hres.rows == ctx->d_hres && P.hres.cand == ctx->d_hcand &&
         (ge == ctx->hagg_groups.end() || 2 * ge->second.first <= P.hagg_cap || ctx->opt.hash_slots_log2 > 0);
  }
  for (int i = 0; ok && i < P.desc.nht; i++) {
    const HashTable& H = ctx->hts[P.li.ht_ids[i]];
    const HTRef r = H.ref();
    ok = (H.valid || (rebuilt && rebuilt->count(H.id))) && std::memcmp(&r, &P.desc.ht[i], sizeof(HTRef)) == 0;
  }
  return ok;
}

// Events around the fused kernel; inside a graph capture they must be
// external so the replayed graph still reports the kernel time.
static cudaError_t record_event(gpl_ctx* ctx, cudaEvent_t ev) {
  cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
  cudaStreamIsCapturing(ctx->stream, &cs);
  if (cs == cudaStreamCaptureStatusActive) return cudaEventRecordWithFlags(ev, ctx->stream, cudaEventRecordExternal);
  return cudaEventRecord(ev, ctx->stream);
}

// A DIRECT build segment lowered to the fused pipeline with an insert sink
// (shape + schedule; the caller fills the run-time pointers).
// A shape pinned by gpl_autotune (keyed by the segment text) wins over the
// model; shortlist (optional) receives the model's per-shape candidates.
static gpl_status lower_build_pipe(gpl_ctx* ctx, const Segment& s, const HashTable& H, PipeDesc* pd, Config* cfg,
                                   std::vector<Config>* shortlist = nullptr, int force_split = -2) {
  LowerInfo li;
  std::string err;
  gpl_status st;
  // Probe split: the option / plan hint, else a split pinned by gpl_autotune,
  // else the heuristic (choose_build_split): every probe in the stage phase (the
  // insert runs straight from the staged tile, no survivor queue) unless the
  // filters keep <= 5% of the rows (then the probes and the insert run in the
  // drain on the queued survivors). The build's pass fractions are estimated
  // from column statistics until known.
  if (!ctx->lambda.count(s.text)) ctx->lambda[s.text] = build_lambda_estimate(ctx, s);
  auto tu = shortlist ? ctx->tuned.end() : ctx->tuned.find(s.text);
  int split = ctx->opt.probe_split >= -1 || s.split_hint >= -1 ? choose_split(ctx, s) : choose_build_split(ctx, s);
  if (force_split >= -1) split = force_split < 0 ? (int)s.probes.size() : force_split;
  else if (tu != ctx->tuned.end() && tu->second.split >= -1 && ctx->opt.probe_split < -1 && s.split_hint < -1)
    split = tu->second.split < 0 ? (int)s.probes.size() : tu->second.split;
  if ((st = lower_probe(ctx, s, split, pd, &li, &err, &H))) return fail(ctx, st, err);
  for (int i = 0; i < pd->nht; i++) {
    const HashTable& h = ctx->hts[li.ht_ids[i]];
    li.ht_bytes[i] = (int64_t)(h.kind == HT_DIRECT ? h.bytes() : h.bytes() / 2);
  }
  if (tu != ctx->tuned.end()) {
    const TunedShape& t = tu->second;
    *cfg = predict(ctx, *pd, li, std::max<int64_t>(pd->nrows, 1), t.tile_rows, t.stage_rows, t.depth, t.warps,
                   t.ctas_per_sm, t.npack, t.ndrain);
  } else if (!choose_config(ctx, *pd, li, pd->nrows, 0, cfg, &err, shortlist)) {
    return fail(ctx, GPL_E_ARG, err);
  }
  if (std::getenv("GPL_DEBUG_MODEL") && !shortlist)
    std::fprintf(stderr, "build %s: split %d/%d tile %lld stage %d depth %d warps %d k %d pk %d pred %.4f ms%s\n",
                 s.name.c_str(), pd->nsprobe, pd->nprobe, (long long)cfg->tile_rows, cfg->stage_rows, cfg->depth,
                 cfg->warps, cfg->ctas_per_sm, cfg->npack, cfg->pred_ms, tu != ctx->tuned.end() ? " (pinned)" : "");
  apply_config(pd, li, *cfg);
  return GPL_OK;
}

// partition phase: count pass, exclusive scan of the counts, scatter pass (stream order is the
// blocking barrier before the probe segment that scans the partitioned table)
static gpl_status launch_partition(gpl_ctx* ctx, const PreparedBuild& P, cudaStream_t st) {
  CK(launch_pipeline_fn(P.pfn, P.pdesc, P.pgrid, st));
  CK(launch_part_scan(P.part_hist, P.part_offs, P.part_n, P.part_total, P.scan_tmp, P.scan_bytes, st));
  CK(launch_pipeline_fn(P.pfn2, P.pdesc2, P.pgrid, st));
  return GPL_OK;
}

static gpl_status launch_prepared_build(gpl_ctx* ctx, const PreparedBuild& P) {
  if (P.part) return launch_partition(ctx, P, ctx->stream);
  if (P.pipe) {
    CK(cudaMemsetAsync((char*)P.pdesc.ins_slots + P.clear_off, 0, P.clear_bytes, ctx->stream));
    CK(launch_pipeline_fn(P.pfn, P.pdesc, P.pgrid, ctx->stream));
  } else {
    CK(launch_build(P.desc, P.trivial, P.known, ctx->sms, ctx->stream));
  }
  return GPL_OK;
}

// A partition segment ("the partition phase also can be implemented in a
// non-blocking manner"): the scanned rows that pass its operators are range-partitioned by the key
// over the DIRECT domain of `by` into a derived table NAME (key + source row id) grouped by
// partition. Two pipelined passes over the source (count per (partition, CTA) in shared memory, then
// scatter at the CTA's own offsets) around one scan of the counts: no global atomics, no host round
// trip. A later 'run NAME' probes the big table partition by partition (each partition's slice of
// the table stays cache-resident) and gathers any other source column through the row id.
static gpl_status build_partition(gpl_ctx* ctx, const Segment& s, const char* text, int32_t* ht_id) {
  gpl_status st;
  std::string err;
  auto ti = ctx->tables.find(s.table);
  if (ti == ctx->tables.end()) return fail(ctx, GPL_E_STATE, "unknown table '" + s.table + "'");
  if (ti->second.derived) return fail(ctx, GPL_E_PLAN, "partition a base table");
  const int64_t cap = std::max<int64_t>(ti->second.nrows, 1);
  if (cap >= (1ll << 31)) return fail(ctx, GPL_E_PLAN, "partition source larger than 2^31 rows");
  PipeDesc pd;
  LowerInfo li;
  if ((st = lower_probe(ctx, s, (int)s.probes.size(), &pd, &li, &err))) return fail(ctx, st, err);
  Config cfg;
  if (!choose_config(ctx, pd, li, pd.nrows, 0, &cfg, &err)) return fail(ctx, GPL_E_ARG, err);
  apply_config(&pd, li, cfg);
  const int key_ci = pd.ins_kcol;
  // the output's placeholder entry (owns the buffers; probes by its name are rejected)
  int idx;
  auto it = ctx->ht_by_name.find(s.name);
  if (it == ctx->ht_by_name.end()) {
    idx = (int)ctx->hts.size();
    ctx->hts.push_back(HashTable());
    ctx->hts[idx].id = idx;
    ctx->ht_by_name[s.name] = idx;
  } else {
    idx = it->second;
  }
  HashTable& H = ctx->hts[idx];
  if (H.slots && H.kind != HT_PART) return fail(ctx, GPL_E_PLAN, "'" + s.name + "' is a hash table");
  if (ctx->host_only) {
    H.kind = HT_PART;
    H.name = s.name;
    H.valid = true;
    if (ht_id) *ht_id = idx;
  }
  const size_t n = (size_t)s.nparts * (size_t)cfg.grid;
  auto r256 = [](size_t b) { return (b + 255) / 256 * 256; };
  const size_t tmp = part_scan_tmp_bytes(n);
  const size_t need = 2 * r256(n * 4) + 256 + r256(tmp) + 2 * r256((size_t)cap * 4);
  if (!ctx->host_only && (!H.part_buf || H.part_alloc < need)) {
    CK(cudaStreamSynchronize(ctx->stream));
    if (H.part_buf) cudaFree(H.part_buf);
    H.part_buf = nullptr;
    H.part_alloc = 0;
    cudaError_t e = cudaMalloc(&H.part_buf, need);
    if (e != cudaSuccess) return fail(ctx, GPL_E_NOMEM, std::string("partition buffers: ") + cudaGetErrorString(e));
    H.part_alloc = need;
  }
  char* b = (char*)H.part_buf;
  PreparedBuild P;
  P.part = true;
  P.part_n = n;
  P.part_hist = (unsigned*)b;
  P.part_offs = (unsigned*)(b + r256(n * 4));
  P.part_total = (unsigned*)(b + 2 * r256(n * 4));
  P.scan_tmp = b + 2 * r256(n * 4) + 256;
  P.scan_bytes = tmp;
  int* keys = (int*)(b + 2 * r256(n * 4) + 256 + r256(tmp));
  int* rows = (int*)((char*)keys + r256((size_t)cap * 4));
  pd.part_hist = P.part_hist;
  pd.part_key_out = keys;
  pd.part_row_out = rows;
  pd.tile_counter = counter_ptr(ctx);  // (static tiles: never claimed)
  pd.op_pass = build_ops_ptr(ctx);
  pd.err = err_ptr(ctx);
  pd.partials = partials_ptr(ctx);
  P.pdesc = pd;
  P.pdesc2 = pd;
  P.pdesc2.sink = SINK_PSCATTER;
  P.pdesc2.part_hist = P.part_offs;  // the scatter starts each (partition, CTA) at its offset
  P.pgrid = cfg.grid;
  // the derived table: its key column + the source row id, `cap` rows of capacity
  const Column* kc = ti->second.find(s.key[0]);
  Table T;
  T.name = s.name;
  T.nrows = cap;
  T.derived = true;
  T.src_table = s.table;
  T.nrows_dev = P.part_total;
  Column ck;
  ck.name = s.key[0];
  ck.type = GPL_I32;
  ck.width = 4;
  ck.dev = (char*)keys;
  ck.cap_rows = cap;
  ck.vmin = kc ? kc->vmin : 0;
  ck.vmax = kc ? kc->vmax : 0;
  Column cr;
  cr.name = T.rowid_col;
  cr.type = GPL_I32;
  cr.width = 4;
  cr.dev = (char*)rows;
  cr.cap_rows = cap;
  cr.vmin = 0;
  cr.vmax = cap - 1;
  T.cols = {ck, cr};
  auto old = ctx->tables.find(s.name);
  bool same = old != ctx->tables.end() && old->second.derived && old->second.nrows == T.nrows &&
              old->second.cols.size() == 2 && old->second.cols[0].dev == ck.dev && old->second.cols[1].dev == cr.dev &&
              old->second.cols[0].name == ck.name && old->second.nrows_dev == T.nrows_dev && old->second.src_table == T.src_table;
  T.version = same ? old->second.version : ctx->next_version++;
  ctx->tables[s.name] = T;
  if (ctx->host_only) return GPL_OK;
  (void)key_ci;
  std::string jerr;
  P.pfn = resolve_pipeline_fn(P.pdesc, ctx->opt.jit != 0, &jerr);
  P.pfn2 = resolve_pipeline_fn(P.pdesc2, ctx->opt.jit != 0, &jerr);
  if (!P.pfn || !P.pfn2) return fail(ctx, GPL_E_CUDA, "cannot configure the partition kernels: " + jerr);
  if ((st = launch_partition(ctx, P, ctx->stream))) return st;
  H.kind = HT_PART;
  H.name = s.name;
  H.slots = H.part_buf;
  H.src_table = s.table;
  H.src_version = ti->second.version;
  H.valid = true;
  if (ht_id) *ht_id = idx;
  P.ht_index = idx;
  P.dest_ref = H.ref();
  P.name = s.name;
  P.table = s.table;
  P.table_version = ti->second.version;
  P.opt_version = ctx->opt_version;
  for (int i = 0; i < pd.nht; i++)
    for (auto& h : ctx->hts)
      if (h.slots == pd.ht[i].slots && h.slots) {
        P.src_ids.push_back(h.id);
        break;
      }
  // cached only when every probed table was found (as for builds)
  if ((int)P.src_ids.size() == pd.nht) ctx->build_cache[text] = P;
  return GPL_OK;
}

GPL_API gpl_status gpl_build_hash(gpl_ctx* ctx, const char* build_segment, int32_t* ht_id) {
  if (!ctx || !build_segment) return GPL_E_ARG;
  if (gpl_status rs = resolve_pending(ctx)) return rs;  // loads still in flight (A0)
  ctx->err.clear();
  // fast path: the same segment over unchanged tables / hash tables / options
  if (!ctx->host_only) {
    auto ci = ctx->build_cache.find(build_segment);
    if (ci != ctx->build_cache.end()) {
      const PreparedBuild& P = ci->second;
      if (build_cache_valid(ctx, P)) {
        gpl_status st = check_dev(ctx);
        if (st) return st;
        if ((st = launch_prepared_build(ctx, P))) return st;
        ctx->hts[P.ht_index].valid = true;
        if (ht_id) *ht_id = P.ht_index;
        return GPL_OK;
      }
      ctx->build_cache.erase(ci);
    }
  }
  Segment s;
  std::string err;
  if (!parse_segment(build_segment, &s, &err)) return fail(ctx, GPL_E_PLAN, err);
  if (!s.is_build) return fail(ctx, GPL_E_PLAN, "expected a build segment ('build NAME')");
  if (s.is_partition) return build_partition(ctx, s, build_segment, ht_id);
  gpl_status st;
  BuildDesc d;
  HashTable shape;
  bool trivial = false;
  if ((st = lower_build(ctx, s, &d, &shape, &trivial, &err))) return fail(ctx, st, err);
  if (ctx->host_only) {  // dry run: register the table's shape so later segments validate
    auto it = ctx->ht_by_name.find(s.name);
    int idx = it == ctx->ht_by_name.end() ? (int)ctx->hts.size() : it->second;
    if (it == ctx->ht_by_name.end()) {
      ctx->hts.push_back(HashTable());
      ctx->ht_by_name[s.name] = idx;
    }
    HashTable& H = ctx->hts[idx];
    H = shape;
    H.id = idx;
    H.name = s.name;
    H.valid = true;
    if (ht_id) *ht_id = idx;
    return GPL_OK;
  }
  if ((st = check_dev(ctx))) return st;
  // (re)allocate the destination table
  int idx;
  auto it = ctx->ht_by_name.find(s.name);
  if (it == ctx->ht_by_name.end()) {
    idx = (int)ctx->hts.size();
    ctx->hts.push_back(HashTable());
    ctx->hts[idx].id = idx;
    ctx->ht_by_name[s.name] = idx;
  } else {
    idx = it->second;
  }
  HashTable& H = ctx->hts[idx];
  // rounded to 256 B: kernels stage small tables with 16-B vector loads
  // (+16: the pipelined build's tile counter after DIRECT cells)
  const size_t need = (std::max<size_t>(shape.bytes(), 16) + 16 + 255) / 256 * 256;
  if (!H.slots || H.alloc_bytes < need) {
    CK(cudaStreamSynchronize(ctx->stream));
    if (H.slots) cudaFree(H.slots);
    H.slots = nullptr;
    H.alloc_bytes = 0;
    cudaError_t e = cudaMalloc(&H.slots, need);
    if (e != cudaSuccess) {
      H.valid = false;
      return fail(ctx, GPL_E_NOMEM, std::string("hash table allocation: ") + cudaGetErrorString(e));
    }
    H.alloc_bytes = need;
  }
  H.cap_slots = shape.cap_slots;
  H.width = shape.width;
  H.dkmin = shape.dkmin;
  H.dnslots = shape.dnslots;
  H.pay_base = shape.pay_base;
  if (shape.kind == HT_MULTI) {
    // fan-out table (NEXT-4): int32 payload per qualifying row (at most the
    // table's rows) + scratch for the per-key counts/cursors and the scan
    const size_t pneed = (std::max<size_t>((size_t)ctx->tables[s.table].nrows, 4) * 4 + 255) / 256 * 256;
    const size_t cbytes = ((size_t)(shape.dnslots + 1) * 4 + 255) / 256 * 256;
    const size_t tbytes = multi_scan_tmp_bytes(shape.dnslots);
    const size_t aneed = cbytes + tbytes + 256;
    auto grow = [&](void** ptr, size_t* have, size_t want) -> gpl_status {
      if (*have >= want) return GPL_OK;
      CK(cudaStreamSynchronize(ctx->stream));
      if (*ptr) cudaFree(*ptr);
      *ptr = nullptr;
      *have = 0;
      cudaError_t e = cudaMalloc(ptr, want);
      if (e != cudaSuccess) return fail(ctx, GPL_E_NOMEM, std::string("multi table allocation: ") + cudaGetErrorString(e));
      *have = want;
      return GPL_OK;
    };
    if ((st = grow(&H.pay, &H.pay_alloc, pneed)) || (st = grow(&H.aux, &H.aux_alloc, aneed))) {
      H.valid = false;
      return st;
    }
    d.pay = H.pay;
    d.cursor = (unsigned int*)H.aux;
    d.scan_tmp = (char*)H.aux + cbytes;
    d.scan_tmp_bytes = tbytes;
  }
  if (!H.hdr) {
    CK(cudaMalloc(&H.hdr, sizeof(HTHeader)));
    CK(launch_header_init(H.hdr, ctx->stream));
  }
  H.name = s.name;
  H.kind = shape.kind;
  H.hash = shape.hash;
  H.key_arity = shape.key_arity;
  H.has_payload = shape.has_payload;
  H.pay_min = shape.pay_min;
  H.pay_max = shape.pay_max;
  H.src_table = shape.src_table;
  H.src_version = shape.src_version;
  d.slots = H.slots;
  d.hdr = H.hdr;
  d.cap_slots = H.cap_slots;
  d.err = err_ptr(ctx);
  HTHeader known{};
  if (trivial) {
    const Table& T = ctx->tables[s.table];
    long long kmin = 0, kmax = 0;
    if (H.key_arity == 1) {
      const Column* kc = T.find(s.key[0]);
      kmin = (long long)(uint32_t)kc->vmin;
      kmax = (long long)(uint32_t)kc->vmax;
      if (kc->vmin < 0) { kmin = 0; kmax = 0xFFFFFFFFll; }  // negative keys: whole unsigned range
    }
    known = trivial_header(T.nrows, kmin, kmax, H.cap_slots, d.load_pct);
  }
  PreparedBuild P;
  if (H.kind == HT_DIRECT && ctx->opt.build_pipeline) {
    // the build segment as a pipeline: scan -> filters -> probes -> insert sink
    PipeDesc pd;
    Config cfg;
    if ((st = lower_build_pipe(ctx, s, H, &pd, &cfg))) return st;
    pd.ins_slots = H.slots;
    pd.tile_counter = (unsigned long long*)((char*)H.slots + direct_counter_off(H.bytes()));
    pd.op_pass = build_ops_ptr(ctx);
    pd.err = err_ptr(ctx);
    pd.partials = partials_ptr(ctx);  // no aggregates: never written
    std::string jerr;
    P.pfn = resolve_pipeline_fn(pd, ctx->opt.jit != 0, &jerr);
    if (!P.pfn) return fail(ctx, GPL_E_CUDA, "cannot configure the pipelined build kernel");
    P.pipe = true;
    P.pdesc = pd;
    P.pgrid = cfg.grid;
    P.clear_bytes = direct_counter_off(H.bytes()) + 16;
    P.clear_off = 0;
    if (pd.ins_dense) {
      // the build writes every cell: clear only the bytes past the domain's
      // last cell (a clustered probe stages 16-B rounded ranges, so they must
      // read as empty) and the tile counter; 8-B granular (the query graph's
      // clear kernel), the few cells below it are rewritten by the build
      const size_t last = H.width == W_NIBBLE ? (size_t)(H.dnslots >> 1) : (size_t)H.dnslots * (size_t)H.width;
      P.clear_off = last & ~(size_t)7;
      P.clear_bytes = direct_counter_off(H.bytes()) + 16 - P.clear_off;
    }
  }
  P.desc = d;
  P.trivial = trivial;
  P.known = known;
  if ((st = launch_prepared_build(ctx, P))) return st;
  H.valid = true;
  if (ht_id) *ht_id = H.id;
  // invalidate prepared builds/runs that referenced this table's old shape
  P.desc = d;
  P.shape = shape;
  P.trivial = trivial;
  P.known = known;
  P.ht_index = H.id;
  P.dest_ref = H.ref();
  P.name = s.name;
  P.table = s.table;
  P.table_version = ctx->tables[s.table].version;
  P.opt_version = ctx->opt_version;
  for (int i = 0; i < d.nht; i++)
    for (auto& h : ctx->hts)
      if (h.slots == d.src[i].slots && h.slots) {
        P.src_ids.push_back(h.id);
        break;
      }
  if ((int)P.src_ids.size() == d.nht) ctx->build_cache[build_segment] = P;
  return GPL_OK;
}

static gpl_status prepare_run(gpl_ctx* ctx, const char* text, int64_t tile_rows, PipeDesc* d, LowerInfo* li,
                              Config* cfg, Segment* seg, int force_split = -2) {
  std::string err;
  if (!parse_segment(text, seg, &err)) return fail(ctx, GPL_E_PLAN, err);
  if (seg->is_build) return fail(ctx, GPL_E_PLAN, "expected a probe segment ('run TABLE')");
  if (force_split >= 0) seg->split_hint = force_split;
  auto tu0 = tile_rows == 0 && force_split < 0 ? ctx->tuned.find(seg->text) : ctx->tuned.end();
  const int split = force_split >= 0 ? force_split
                    : (tu0 != ctx->tuned.end() && tu0->second.split >= 0) ? tu0->second.split
                                                                          : choose_split(ctx, *seg);
  gpl_status st = lower_probe(ctx, *seg, split, d, li, &err);
  if (st) return fail(ctx, st, err);
  auto lit = ctx->lambda.find(seg->text);
  if (lit != ctx->lambda.end()) li->lambda = lit->second;
  for (int i = 0; i < d->nht; i++) {
    for (auto& h : ctx->hts)
      if (h.slots == d->ht[i].slots)
        li->ht_bytes[i] = (int64_t)(h.kind == HT_DIRECT ? h.bytes() : h.bytes() / 2);
  }
  apply_profile(ctx, *d, li, seg->text);
  if (tile_rows < 0) return fail(ctx, GPL_E_ARG, "tile_rows must be >= 0");
  auto tu = tile_rows == 0 ? ctx->tuned.find(seg->text) : ctx->tuned.end();
  if (tu != ctx->tuned.end()) {  // shape pinned by gpl_autotune
    const TunedShape& t = tu->second;
    *cfg = predict(ctx, *d, *li, std::max<int64_t>(d->nrows, 1), t.tile_rows, t.stage_rows, t.depth, t.warps,
                   t.ctas_per_sm, t.npack, t.ndrain);
  } else if (!choose_config(ctx, *d, *li, d->nrows, tile_rows, cfg, &err)) {
    return fail(ctx, GPL_E_ARG, err);
  }
  apply_config(d, *li, *cfg);
  return GPL_OK;
}

// Prepared (parsed, lowered, configured, kernel-resolved) probe segment,
// cached by text + tile_rows and revalidated against the scanned table's
// version, the referenced hash tables, the options and the λ profile.
static gpl_status get_prepared_run(gpl_ctx* ctx, const char* text, int64_t tile_rows, PreparedRun** out) {
  const std::string key = std::string(text) + "\x1f" + std::to_string(tile_rows);
  auto lam = ctx->lambda.find(text);
  const size_t lambda_n = lam == ctx->lambda.end() ? 0 : lam->second.size();
  auto it = ctx->run_cache.find(key);
  if (it != ctx->run_cache.end()) {
    PreparedRun& P = *it->second;
    if (run_cache_valid(ctx, P)) {
      *out = &P;
      return GPL_OK;
    }
    ctx->run_cache.erase(it);
  }
  PipeDesc d;
  LowerInfo li;
  Config cfg;
  Segment seg;
  gpl_status st;
  if ((st = prepare_run(ctx, text, tile_rows, &d, &li, &cfg, &seg))) return st;
  PreparedRun P;
  li.table = seg.table;
  if (li.hash_group) {
    // aggregation table: 2^k slots >= 2 x the distinct groups of the plan's
    // last run (load <= 1/2), else min(rows, 2^21) groups assumed; keys then
    // accumulators, zeroed per run. Selection scratch and the row buffer too.
    // (groups scale with the fact rows when the table was reloaded at another size)
    auto ge = ctx->hagg_groups.find(seg.text);
    const uint64_t est =
        ge != ctx->hagg_groups.end()
            ? (uint64_t)((double)ge->second.first * std::max(1.0, (double)d.nrows / (double)std::max<int64_t>(ge->second.second, 1)))
            : (uint64_t)std::min<int64_t>(std::max<int64_t>(d.nrows, 1), 1 << 21);
    int lg = 12;
    while ((1ull << lg) < 2 * est && lg < 31) lg++;  // 32-bit slot indices in the selection
    if (ctx->opt.hash_slots_log2 > 0) lg = (int)ctx->opt.hash_slots_log2;
    const uint64_t cap = 1ull << lg;
    const size_t bytes = (size_t)cap * 8 * (1 + li.nagg);
    const size_t rbytes = (size_t)cap * 8 * (1 + li.nagg);
    const int nblocks = hagg_select_blocks(cap, ctx->sms);
    const size_t cbytes = (size_t)nblocks * std::max(1, li.limit) * 5 * 8;
    auto grow = [&](void** p, size_t* have, size_t need) -> cudaError_t {
      if (*have >= need) return cudaSuccess;
      cudaError_t e = cudaStreamSynchronize(ctx->stream);
      if (e != cudaSuccess) return e;
      if (*p) cudaFree(*p);
      *p = nullptr;
      *have = 0;
      e = cudaMalloc(p, need);
      if (e == cudaSuccess) *have = need;
      return e;
    };
    if (grow(&ctx->d_hagg, &ctx->hagg_alloc, bytes) != cudaSuccess ||
        grow((void**)&ctx->d_hres, &ctx->hres_alloc, li.limit ? (size_t)li.limit * 8 * (1 + li.nagg) : rbytes) != cudaSuccess ||
        grow((void**)&ctx->d_hcand, &ctx->hcand_alloc, cbytes) != cudaSuccess) {
      cudaGetLastError();
      return fail(ctx, GPL_E_NOMEM, "hash group-by: cannot allocate a " + std::to_string(cap) + "-slot table");
    }
    d.hagg_keys = (unsigned long long*)ctx->d_hagg;
    d.hagg_accs = (long long*)((char*)ctx->d_hagg + (size_t)cap * 8);
    d.hagg_count = partials_ptr(ctx);  // result word 0: distinct groups
    d.hagg_log2 = lg;
    P.hagg_cap = cap;
    P.hagg_clear = bytes;
    HaggResultDesc& R = P.hres;
    R.keys = d.hagg_keys;
    R.accs = d.hagg_accs;
    R.nslots = cap;
    R.nagg = li.nagg;
    R.nkeys = li.ngroup_dims;
    R.limit = li.limit;
    R.norder = li.norder;
    for (int i = 0; i < 3; i++) {
      R.ord_is_agg[i] = li.ord_is_agg[i];
      R.ord_idx[i] = li.ord_idx[i];
      R.ord_desc[i] = li.ord_desc[i];
    }
    R.cand = ctx->d_hcand;
    R.nblocks = nblocks;
    R.rows = ctx->d_hres;
    R.small_out = partials_ptr(ctx);
    R.n_out = partials_ptr(ctx) + 1;
  }
  d.partials = partials_ptr(ctx);
  d.tile_counter = counter_ptr(ctx);
  d.op_pass = op_pass_ptr(ctx);
  d.err = err_ptr(ctx);
  P.desc = d;
  P.li = li;
  P.grid = cfg.grid;
  P.pred_ms = cfg.pred_ms;
  P.text = seg.text;
  P.table_version = ctx->tables[seg.table].version;
  P.opt_version = ctx->opt_version;
  P.lambda_n = lambda_n;
  P.profiled = profile_current(ctx, P.text, li.table);
  std::string jerr;
  P.fn = resolve_pipeline_fn(d, ctx->opt.jit != 0, &jerr);
  P.jit = ctx->opt.jit != 0 && jerr.empty();
  if (std::getenv("GPL_DEBUG_DESC")) {  // diagnostics: the launch layout of each prepared run
    std::fprintf(stderr, "prepared run: nrows %lld tile %lld S %d D %d W %d npack %d grid %d smem %d off_ring %d slot %d ncols %d split %d:",
                 d.nrows, d.tile_rows, d.stage_rows, d.depth, d.nwarps, d.npack, P.grid, d.smem_bytes, d.off_ring,
                 d.slot_bytes, d.ncols, d.nsprobe);
    for (int c = 0; c < d.ncols; c++) std::fprintf(stderr, " [%d:w%d off%d lazy%d %p]", c, d.colw[c], d.coloff[c], d.lazy[c], (const void*)d.col[c]);
    std::fprintf(stderr, " jit=%d %s\n", (int)P.jit, jerr.c_str());
  }
  if (!P.fn) return fail(ctx, GPL_E_CUDA, "cannot configure the pipeline kernel");
  auto sp = std::make_shared<PreparedRun>(P);
  ctx->run_cache[key] = sp;
  *out = sp.get();
  return GPL_OK;
}

GPL_API gpl_status gpl_run_plan(gpl_ctx* ctx, const char* probe_segment, int64_t tile_rows) {
  if (!ctx || !probe_segment) return GPL_E_ARG;
  if (gpl_status rs = resolve_pending(ctx)) return rs;  // loads still in flight (A0)
  ctx->err.clear();
  gpl_status st = check_dev(ctx);
  if (st) return st;
  if (tile_rows < 0) return fail(ctx, GPL_E_ARG, "tile_rows must be >= 0");
  PreparedRun* P = nullptr;
  if ((st = get_prepared_run(ctx, probe_segment, tile_rows, &P))) return st;
  const PipeDesc& d = P->desc;
  const LowerInfo& li = P->li;
  const size_t pbytes = run_pbytes(li);
  // one memset: tile counter, op_pass and the partials are contiguous
  CK(cudaMemsetAsync(counter_ptr(ctx), 0, run_clear_bytes(pbytes), ctx->stream));
  if (li.hash_group) CK(cudaMemsetAsync(d.hagg_keys, 0, P->hagg_clear, ctx->stream));
  CK(record_event(ctx, ctx->ev0));
  CK(launch_pipeline_fn(P->fn, d, P->grid, ctx->stream));
  CK(record_event(ctx, ctx->ev1));
  if (li.hash_group) CK(launch_hagg_result(P->hres, d.hagg_count, ctx->sms, ctx->stream));
  CK(launch_copyout(ctx->d_scratch, ctx->h_stage_dev, result_words(pbytes), ctx->stream));
  LastRun& L = ctx->last;
  L.valid = true;
  L.kbe = false;
  L.copied_out = true;
  L.overflowed = false;
  L.run = ctx->run_cache[std::string(probe_segment) + "\x1f" + std::to_string(tile_rows)];
  L.timed = true;
  gpl_stats& S = L.stats;
  S = gpl_stats{};
  S.rows_scanned = d.nrows;
  S.tile_rows_used = d.tile_rows;
  S.stage_rows = d.stage_rows;
  S.ring_depth = d.depth;
  S.consumer_warps = d.nwarps;
  S.grid = P->grid;
  S.n_ops = li.nops;
  S.probe_split = d.nsprobe;
  S.predicted_ms = P->pred_ms;
  S.bytes_scanned = (double)d.nrows * li.bytes_per_row;
  S.bytes_full_scan = (double)d.nrows * li.bytes_per_row_all;
  S.lazy_columns = (int32_t)li.lazy_w.size();
  S.packets = d.npack;
  S.agg_mode = d.agg_mode;
  S.jit = P->jit ? 1 : 0;
  S.hash_slots = (int64_t)P->hagg_cap;
  S.drain_warps = d.ndrain;
  return GPL_OK;
}

// Split a whole plan into its segments at 'build NAME' / 'run TABLE' lines.
static std::vector<std::string> split_segments(const std::string& plan) {
  std::vector<std::string> segs;
  std::string cur;
  bool cur_has_head = false;
  size_t i = 0;
  while (i <= plan.size()) {
    size_t j = plan.find('\n', i);
    if (j == std::string::npos) j = plan.size();
    const std::string line = plan.substr(i, j - i);
    size_t k = line.find_first_not_of(" \t\r");
    const std::string head = k == std::string::npos ? "" : line.substr(k, line.find_first_of(" \t\r#", k) - k);
    const bool seg_head = head == "build" || head == "partition" || head == "run";
    if (seg_head && cur_has_head) {
      segs.push_back(cur);
      cur.clear();
    }
    if (seg_head) cur_has_head = true;
    cur += line + "\n";
    i = j + 1;
  }
  if (cur_has_head) segs.push_back(cur);
  return segs;
}

GPL_API gpl_status gpl_run_query(gpl_ctx* ctx, const char* plan, int64_t tile_rows) {
  if (!ctx || !plan) return GPL_E_ARG;
  if (gpl_status rs = resolve_pending(ctx)) return rs;  // loads still in flight (A0)
  ctx->err.clear();
  gpl_status st = check_dev(ctx);
  if (st) return st;
  auto ps = ctx->plan_segs.find(plan);
  if (ps == ctx->plan_segs.end()) ps = ctx->plan_segs.emplace(plan, split_segments(plan)).first;
  const std::vector<std::string>& segs = ps->second;
  if (segs.empty()) return fail(ctx, GPL_E_PLAN, "plan has no segment");
  const std::string key = std::string(plan) + "\x1f" + std::to_string(tile_rows);
  const std::string run_key = segs.back() + "\x1f" + std::to_string(tile_rows);
  // are all segments prepared and still valid?
  std::set<int> rebuilt;  // tables this query's build segments (re)build, in order
  auto all_valid = [&]() {
    rebuilt.clear();
    for (size_t i = 0; i + 1 < segs.size(); i++) {
      auto b = ctx->build_cache.find(segs[i]);
      if (b == ctx->build_cache.end() || !build_cache_valid(ctx, b->second, &rebuilt)) return false;
      rebuilt.insert(b->second.ht_index);
    }
    auto r = ctx->run_cache.find(run_key);
    return r != ctx->run_cache.end() && run_cache_valid(ctx, *r->second, &rebuilt) && ctx->lambda.count(r->second->text);
  };
  auto eager = [&]() -> gpl_status {
    for (size_t i = 0; i + 1 < segs.size(); i++) {
      gpl_status s2 = gpl_build_hash(ctx, segs[i].c_str(), nullptr);
      if (s2) return s2;
    }
    return gpl_run_plan(ctx, segs.back().c_str(), tile_rows);
  };
  auto g = ctx->graphs.find(key);
  if (g != ctx->graphs.end()) {
    static const bool trace = std::getenv("GPL_TRACE_HOST") != nullptr;
    const auto t0 = std::chrono::steady_clock::now();
    if (all_valid()) {
      const auto t1 = std::chrono::steady_clock::now();
      CK(cudaGraphLaunch(g->second, ctx->stream));
      for (int h : rebuilt) ctx->hts[h].valid = true;  // the replay rebuilt them
      if (trace) {
        const auto t2 = std::chrono::steady_clock::now();
        std::fprintf(stderr, "gpl_run_query host: validate %.1f us, cudaGraphLaunch %.1f us\n",
                     std::chrono::duration<double, std::micro>(t1 - t0).count(),
                     std::chrono::duration<double, std::micro>(t2 - t1).count());
      }
      // the run's bookkeeping is the cached plan's
      const std::shared_ptr<PreparedRun>& PP = ctx->run_cache[run_key];
      const PreparedRun& P = *PP;
      LastRun& L = ctx->last;
      L.valid = true;
      L.kbe = false;
      L.copied_out = true;
      L.overflowed = false;
      L.run = PP;
      L.timed = true;
      gpl_stats& S = L.stats;
      S = gpl_stats{};
      S.rows_scanned = P.desc.nrows;
      S.tile_rows_used = P.desc.tile_rows;
      S.stage_rows = P.desc.stage_rows;
      S.ring_depth = P.desc.depth;
      S.consumer_warps = P.desc.nwarps;
      S.grid = P.grid;
      S.n_ops = P.li.nops;
      S.probe_split = P.desc.nsprobe;
      S.predicted_ms = P.pred_ms;
      S.bytes_scanned = (double)P.desc.nrows * P.li.bytes_per_row;
      S.bytes_full_scan = (double)P.desc.nrows * P.li.bytes_per_row_all;
      S.lazy_columns = (int32_t)P.li.lazy_w.size();
      S.packets = P.desc.npack;
      S.agg_mode = P.desc.agg_mode;
      S.jit = P.jit ? 1 : 0;
      {
        auto gk = ctx->graph_kernels.find(key);
        S.launches = gk != ctx->graph_kernels.end() ? gk->second : 0;
      }
      S.hash_slots = (int64_t)P.hagg_cap;
      S.drain_warps = P.desc.ndrain;
      return GPL_OK;
    }
    cudaGraphExecDestroy(g->second);
    ctx->graphs.erase(g);
  }
  // run eagerly (refreshes the prepared caches); once everything is prepared
  // and profiled, record the same sequence as a graph for the next call
  // the recorded sequence: ONE clear kernel for every DIRECT table of a
  // pipelined build (cells + tile counter) and the run's counters/partials,
  // then the build pipelines (other builds: their own kernels) and the fused run
  auto fused_sequence = [&]() -> gpl_status {
    ClearList L{};
    auto add = [&](void* p, size_t b) {
      if (L.n < 16) {
        L.ptr[L.n] = p;
        L.bytes[L.n] = b;
      }
      L.n++;
    };
    std::vector<const PreparedBuild*> builds;
    for (size_t i = 0; i + 1 < segs.size(); i++) {
      const PreparedBuild& B = ctx->build_cache.at(segs[i]);
      builds.push_back(&B);
      if (B.pipe && !B.part) add((char*)B.pdesc.ins_slots + B.clear_off, B.clear_bytes);
    }
    const PreparedRun& R = *ctx->run_cache.at(run_key);
    add(counter_ptr(ctx), run_clear_bytes(run_pbytes(R.li)));
    if (R.li.hash_group) add(R.desc.hagg_keys, R.hagg_clear);
    if (L.n > 16) return eager();
    CK(launch_clear(L, ctx->sms, ctx->stream));
    // Build segments form a DAG (a build depends on the tables it probes,
    // each segment ends at its blocking build). Two capture lanes:
    // a build runs on the lane of the builds it depends on (joining the other
    // lane by an event when it depends on both), an independent build on the
    // lane that has fewer; the run joins both. Small dimension builds then
    // overlap instead of queueing behind each other.
    auto launch_b = [&](const PreparedBuild* B, cudaStream_t st) -> gpl_status {
      if (B->part) return launch_partition(ctx, *B, st);
      if (B->pipe) CK(launch_pipeline_fn(B->pfn, B->pdesc, B->pgrid, st));
      else CK(launch_build(B->desc, B->trivial, B->known, ctx->sms, st));
      return GPL_OK;
    };
    bool two = ctx->opt.graph_branches && builds.size() >= 2;
    if (two && !ctx->side) {
      two = cudaStreamCreateWithFlags(&ctx->side, cudaStreamNonBlocking) == cudaSuccess;
      for (auto& e : ctx->fork_ev)
        if (two && !e) two = cudaEventCreateWithFlags(&e, cudaEventDisableTiming) == cudaSuccess;
    }
    if (!two) {
      for (const PreparedBuild* B : builds)
        if (gpl_status s2 = launch_b(B, ctx->stream)) return s2;
    } else {
      int nev = 0;
      auto join = [&](cudaStream_t from, cudaStream_t to) -> gpl_status {
        if (nev >= 8) return fail(ctx, GPL_E_CUDA, "too many graph lane joins");
        CK(cudaEventRecord(ctx->fork_ev[nev], from));
        CK(cudaStreamWaitEvent(to, ctx->fork_ev[nev], 0));
        nev++;
        return GPL_OK;
      };
      cudaStream_t lane_st[2] = {ctx->stream, ctx->side};
      if (gpl_status s2 = join(ctx->stream, ctx->side)) return s2;  // the side lane starts after the clear
      std::map<int, int> lane_of;  // hash-table id -> lane that builds it
      int count[2] = {0, 0};
      for (const PreparedBuild* B : builds) {
        bool dep[2] = {false, false};
        for (int id : B->src_ids) {
          auto it = lane_of.find(id);
          if (it != lane_of.end()) dep[it->second] = true;
        }
        int ln = dep[0] ? 0 : dep[1] ? 1 : (count[1] < count[0] ? 1 : 0);
        if (dep[0] && dep[1])
          if (gpl_status s2 = join(lane_st[1], lane_st[0])) return s2;
        if (gpl_status s2 = launch_b(B, lane_st[ln])) return s2;
        lane_of[B->ht_index] = ln;
        count[ln]++;
      }
      if (gpl_status s2 = join(ctx->side, ctx->stream)) return s2;  // the run waits for both lanes
    }
    CK(record_event(ctx, ctx->ev0));
    CK(launch_pipeline_fn(R.fn, R.desc, R.grid, ctx->stream));
    CK(record_event(ctx, ctx->ev1));
    if (R.li.hash_group) CK(launch_hagg_result(R.hres, R.desc.hagg_count, ctx->sms, ctx->stream));
    CK(launch_copyout(ctx->d_scratch, ctx->h_stage_dev, result_words(run_pbytes(R.li)), ctx->stream));
    return GPL_OK;
  };
  if ((st = eager())) return st;
  if (all_valid()) {
    const LastRun saved = ctx->last;
    cudaGraph_t graph = nullptr;
    bool ok = cudaStreamBeginCapture(ctx->stream, cudaStreamCaptureModeThreadLocal) == cudaSuccess;
    gpl_status cst = ok ? fused_sequence() : GPL_E_CUDA;
    cudaError_t ce = cudaStreamEndCapture(ctx->stream, &graph);
    ctx->last = saved;
    cudaGraphExec_t exec = nullptr;
    if (ok && cst == GPL_OK && ce == cudaSuccess && graph &&
        cudaGraphInstantiate(&exec, graph, 0) == cudaSuccess) {
      ctx->graphs[key] = exec;
      // kernels one replay launches (stats.launches): the graph's kernel nodes
      size_t nn = 0;
      int nk = 0;
      if (cudaGraphGetNodes(graph, nullptr, &nn) == cudaSuccess && nn) {
        std::vector<cudaGraphNode_t> nodes(nn);
        if (cudaGraphGetNodes(graph, nodes.data(), &nn) == cudaSuccess)
          for (size_t i = 0; i < nn; i++) {
            cudaGraphNodeType t;
            if (cudaGraphNodeGetType(nodes[i], &t) == cudaSuccess && t == cudaGraphNodeTypeKernel) nk++;
          }
      }
      ctx->graph_kernels[key] = nk;
    }
    if (graph) cudaGraphDestroy(graph);
    cudaGetLastError();  // a failed capture only means no graph; the eager run above stands
    ctx->err.clear();
  }
  return GPL_OK;
}

// The model's per-shape candidates plus, for the `top` best predicted, the
// other consumer-warp counts that fit (the model's W is the least certain
// knob: the work-group sweep of P:366 / Figs 14-15 is measured, not only
// modelled; every extra shape costs one plan-specialised compile), tile
// sizes of 1, 2 and 4 stages (same kernel) and drain-warp splits.
static void with_warp_variants(const gpl_ctx* ctx, const PipeDesc& d, const LowerInfo& li, int64_t N,
                               std::vector<Config>* cs, size_t top = 3) {
  if (ctx->opt.consumer_warps > 0) return;
  std::vector<Config> out;
  for (size_t i = 0; i < cs->size(); i++) {
    const Config& c = (*cs)[i];
    out.push_back(c);
    if (i >= top) continue;
    for (int W : {4, 8, 12, 16}) {
      if (W == c.warps) continue;
      Config v = predict(ctx, d, li, std::max<int64_t>(N, 1), c.tile_rows, c.stage_rows, c.depth, W, c.ctas_per_sm, c.npack,
                         c.ndrain);
      if (v.feasible) out.push_back(v);
    }
    // scheduling granularity (Eq 3's waves / last-wave tail): the same shape at Δ = 1, 2, 4 stages
    for (int m : {1, 2, 4}) {
      const int64_t t = (int64_t)c.stage_rows * m;
      if (t == c.tile_rows) continue;
      Config v = predict(ctx, d, li, std::max<int64_t>(N, 1), t, c.stage_rows, c.depth, c.warps, c.ctas_per_sm, c.npack,
                         c.ndrain);
      if (v.feasible) out.push_back(v);
    }
    // operator-specialised drain warps (NEXT-1): the same shape with 0, 1, 2 of its warps draining
    if (ctx->opt.drain_warps < 0)
      for (int nd : {0, 1, 2}) {
        if (nd == c.ndrain) continue;
        Config v = predict(ctx, d, li, std::max<int64_t>(N, 1), c.tile_rows, c.stage_rows, c.depth, c.warps,
                           c.ctas_per_sm, c.npack, nd);
        if (v.feasible) out.push_back(v);
      }
  }
  cs->swap(out);
}

// gpl_autotune for one build segment that runs as a pipeline (DIRECT table):
// time the model's per-shape candidates on rebuilds of the same table
// (L2 flushed, median of 3) and pin the fastest under the segment's text.
// Earlier tables of the plan are already built; the contents never change.
static gpl_status tune_build(gpl_ctx* ctx, const std::string& text, void* flush, size_t fbytes,
                             int32_t max_candidates, double* model_ms, double* best_ms_out, int* tuned) {
  Segment s;
  std::string err;
  if (!parse_segment(text, &s, &err) || !s.is_build) return GPL_OK;
  auto hi = ctx->ht_by_name.find(s.name);
  if (hi == ctx->ht_by_name.end() || !ctx->opt.build_pipeline) return GPL_OK;
  const HashTable H = ctx->hts[hi->second];
  if (H.kind != HT_DIRECT) return GPL_OK;
  ctx->tuned.erase(s.text);
  // candidates per probe split: every probe in the stage phase, and (a build
  // with filters before its probes) the probes + insert in the queue phase
  const int np = (int)s.probes.size();
  std::vector<int> splits{-1};
  if (np > 0 && !s.filters.empty() && ctx->opt.probe_split < -1 && s.split_hint < -1) splits.push_back(0);
  std::vector<std::pair<Config, int>> cands;  // (shape, split)
  for (int sp : splits) {
    PipeDesc pd;
    Config c0;
    std::vector<Config> cs;
    gpl_status st = lower_build_pipe(ctx, s, H, &pd, &c0, &cs, sp);
    if (st) return st;
    if (max_candidates > 0 && (int)cs.size() > max_candidates) cs.resize(max_candidates);
    {
      LowerInfo lb;  // the build pipeline's facts for the warp variants (as lower_build_pipe computed them)
      PipeDesc pb;
      std::string e2;
      if (lower_probe(ctx, s, sp < 0 ? np : sp, &pb, &lb, &e2, &H) == GPL_OK) {
        for (int i = 0; i < pb.nht; i++) {
          const HashTable& h = ctx->hts[lb.ht_ids[i]];
          lb.ht_bytes[i] = (int64_t)(h.kind == HT_DIRECT ? h.bytes() : h.bytes() / 2);
        }
        with_warp_variants(ctx, pb, lb, pb.nrows, &cs);
      }
    }
    bool has0 = false;
    for (const Config& c : cs)
      has0 |= c.tile_rows == c0.tile_rows && c.stage_rows == c0.stage_rows && c.depth == c0.depth &&
              c.warps == c0.warps && c.ctas_per_sm == c0.ctas_per_sm && c.npack == c0.npack && c.ndrain == c0.ndrain;
    if (!has0) cs.insert(cs.begin(), c0);
    for (const Config& c : cs) cands.push_back({c, sp});
  }
  // the model's own pick (its split, its shape): the model-predicted build time reported
  PipeDesc pm;
  Config cm;
  if (gpl_status st = lower_build_pipe(ctx, s, H, &pm, &cm)) return st;
  const int sm = pm.nsprobe == pm.nprobe && pm.nresid == 0 ? -1 : pm.nsprobe;
  gpl_status st = GPL_OK;
  cudaEvent_t a = nullptr, b = nullptr;
  CK(cudaEventCreate(&a));
  CK(cudaEventCreate(&b));
  double best_ms = 1e300, m0 = -1;
  TunedShape best;
  for (const auto& [c, sp] : cands) {
    TunedShape t{c.tile_rows, c.stage_rows, c.depth, c.warps, c.ctas_per_sm, sp, c.npack, c.ndrain};
    ctx->tuned[s.text] = t;
    ctx->build_cache.erase(text);
    std::vector<float> ms;
    st = GPL_OK;
    for (int rep = 0; rep < 4 && !st; rep++) {
      if (cudaMemsetAsync(flush, rep, fbytes, ctx->stream) != cudaSuccess) break;
      cudaEventRecord(a, ctx->stream);
      st = gpl_build_hash(ctx, text.c_str(), nullptr);
      cudaEventRecord(b, ctx->stream);
      if (cudaStreamSynchronize(ctx->stream) != cudaSuccess) break;
      float m = 0;
      cudaEventElapsedTime(&m, a, b);
      if (rep > 0) ms.push_back(m);
    }
    if (st || ms.size() < 3) {  // a shape that cannot run (resources) is skipped
      st = GPL_OK;
      ctx->err.clear();
      cudaGetLastError();
      continue;
    }
    std::sort(ms.begin(), ms.end());
    if (std::getenv("GPL_DEBUG_TUNE"))
      std::fprintf(stderr, "[tune build %s] split %d tile %lld stage %d depth %d warps %d k %d pk %d: %.4f ms (pred %.4f)%s\n",
                   s.name.c_str(), sp, (long long)c.tile_rows, c.stage_rows, c.depth, c.warps, c.ctas_per_sm, c.npack,
                   ms[1], c.pred_ms,
                   sp == sm && c.tile_rows == cm.tile_rows && c.stage_rows == cm.stage_rows && c.depth == cm.depth &&
                           c.warps == cm.warps && c.ctas_per_sm == cm.ctas_per_sm && c.npack == cm.npack
                       ? " <- model"
                       : "");
    if (m0 < 0 && sp == sm && c.tile_rows == cm.tile_rows && c.stage_rows == cm.stage_rows && c.depth == cm.depth &&
        c.warps == cm.warps && c.ctas_per_sm == cm.ctas_per_sm && c.npack == cm.npack && c.ndrain == cm.ndrain)
      m0 = ms[1];
    if (ms[1] < best_ms) {
      best_ms = ms[1];
      best = t;
    }
  }
  cudaEventDestroy(a);
  cudaEventDestroy(b);
  if (best_ms < 1e300) {
    ctx->tuned[s.text] = best;
    (*tuned)++;
    *best_ms_out += best_ms;
    *model_ms += m0 < 0 ? best_ms : m0;
  } else {
    ctx->tuned.erase(s.text);
  }
  ctx->build_cache.erase(text);
  // leave the table built at the pinned shape
  return gpl_build_hash(ctx, text.c_str(), nullptr);
}

GPL_API gpl_status gpl_autotune(gpl_ctx* ctx, const char* plan, int32_t max_candidates, gpl_model_report* out) {
  if (!ctx || !plan) return GPL_E_ARG;
  if (gpl_status rs = resolve_pending(ctx)) return rs;  // loads still in flight (A0)
  ctx->err.clear();
  gpl_status st = check_dev(ctx);
  if (st) return st;
  const std::vector<std::string> segs = split_segments(plan);
  if (segs.empty()) return fail(ctx, GPL_E_PLAN, "plan has no segment");
  for (size_t i = 0; i + 1 < segs.size(); i++)
    if ((st = gpl_build_hash(ctx, segs[i].c_str(), nullptr))) return st;
  // L2 flush buffer (2x L2) so every timing starts cold, as the bench does
  void* flush = nullptr;
  const size_t fbytes = (size_t)2 * ctx->l2_bytes;
  CK(cudaMalloc(&flush, fbytes));
  struct FreeOnExit {
    void* p;
    ~FreeOnExit() { cudaFree(p); }
  } flush_guard{flush};
  int builds_tuned = 0;
  double build_ms_model = 0, build_ms = 0;
  for (size_t i = 0; i + 1 < segs.size(); i++)
    if ((st = tune_build(ctx, segs[i], flush, fbytes, max_candidates, &build_ms_model, &build_ms, &builds_tuned)))
      return st;
  if (!ctx->opt.autotune_probe) {
    // the build segments only: the probe segment keeps the A9 model's own
    // pick; query graphs recorded with the old build shapes are dropped
    for (auto& kv : ctx->graphs) cudaGraphExecDestroy(kv.second);
    ctx->graphs.clear();
    if (out) {
      *out = gpl_model_report{};
      out->builds_tuned = builds_tuned;
      out->build_ms_model = build_ms_model;
      out->build_ms = build_ms;
    }
    return GPL_OK;
  }
  const std::string& probe = segs.back();
  // one eager run profiles λ (the split and the model depend on it)
  if ((st = gpl_run_plan(ctx, probe.c_str(), 0))) return st;
  gpl_result tmp{};
  tmp.cap_groups = 0;
  gpl_fetch_result(ctx, &tmp);  // records λ; capacity errors are irrelevant here
  ctx->err.clear();
  // the model's shortlist, for the heuristic's probe split and every other
  // split (how many probes run before the survivor queue)
  Segment seg;
  std::string err;
  if (!parse_segment(probe, &seg, &err)) return fail(ctx, GPL_E_PLAN, err);
  PipeDesc d;
  LowerInfo li;
  const int split0 = choose_split(ctx, seg);
  std::vector<int> splits{split0};
  if (seg.split_hint < -1 && ctx->opt.probe_split < -1)
    for (int sp = 0; sp <= std::min<int>((int)seg.probes.size(), MAXSP); sp++)
      if (sp != split0) splits.push_back(sp);
  std::vector<std::pair<int, Config>> cands;
  std::vector<int> cand_split_eff;  // the split the lowering kept (late materialisation may move a probe to the queue)
  ctx->tuned.erase(seg.text);
  for (int sp : splits) {
    PipeDesc ds;
    LowerInfo ls;
    if ((st = lower_probe(ctx, seg, sp, &ds, &ls, &err))) {
      if (sp == split0) return fail(ctx, st, err);
      st = GPL_OK;
      continue;
    }
    auto lit = ctx->lambda.find(seg.text);
    if (lit != ctx->lambda.end()) ls.lambda = lit->second;
    for (int i = 0; i < ds.nht; i++) {
      const HashTable& h = ctx->hts[ls.ht_ids[i]];
      ls.ht_bytes[i] = (int64_t)(h.kind == HT_DIRECT ? h.bytes() : h.bytes() / 2);
    }
    apply_profile(ctx, ds, &ls, seg.text);
    Config best_model;
    std::vector<Config> cs;
    if (!choose_config(ctx, ds, ls, ds.nrows, 0, &best_model, &err, &cs)) {
      if (sp == split0) return fail(ctx, GPL_E_ARG, err);
      continue;
    }
    if (max_candidates > 0 && (int)cs.size() > max_candidates) cs.resize(max_candidates);
    with_warp_variants(ctx, ds, ls, ds.nrows, &cs);
    if (ls.cons_factor != 1 || ls.bw_factor != 1) {
      // the profile-fitted model and the plain one disagree on each shape's best
      // depth / warps / Δ: measure both shortlists (a fitted model must never
      // hide a configuration the plain model would have offered)
      LowerInfo lr = ls;
      lr.cons_factor = lr.bw_factor = 1;
      Config b2;
      std::vector<Config> cr;
      if (choose_config(ctx, ds, lr, ds.nrows, 0, &b2, &err, &cr)) {
        if (max_candidates > 0 && (int)cr.size() > max_candidates) cr.resize(max_candidates);
        with_warp_variants(ctx, ds, lr, ds.nrows, &cr);
        for (const Config& c : cr) {
          bool dup = false;
          for (const Config& x : cs)
            dup |= x.tile_rows == c.tile_rows && x.stage_rows == c.stage_rows && x.depth == c.depth &&
                   x.warps == c.warps && x.ctas_per_sm == c.ctas_per_sm && x.npack == c.npack && x.ndrain == c.ndrain;
          if (dup) continue;
          // ranked (and reported) by the fitted model like the rest
          Config cf = predict(ctx, ds, ls, std::max<int64_t>(ds.nrows, 1), c.tile_rows, c.stage_rows, c.depth, c.warps,
                              c.ctas_per_sm, c.npack, c.ndrain);
          cs.push_back(cf);
        }
      }
      err.clear();
    }
    for (const Config& c : cs) {
      cands.push_back({sp, c});
      cand_split_eff.push_back(ds.nsprobe);
    }
    if (sp == split0) {
      d = ds;
      li = ls;
    }
  }
  double best_ms = 1e300;
  TunedShape best;
  int best_eff_split = -1;
  int tried = 0;
  for (size_t ci = 0; ci < cands.size(); ci++) {
    const auto& sc = cands[ci];
    const Config& c = sc.second;
    TunedShape t{c.tile_rows, c.stage_rows, c.depth, c.warps, c.ctas_per_sm, sc.first, c.npack, c.ndrain};
    ctx->tuned[seg.text] = t;
    ctx->run_cache.erase(probe + "\x1f" + std::to_string(0));
    std::vector<float> ms;
    for (int rep = 0; rep < 4; rep++) {
      if (cudaMemsetAsync(flush, rep, fbytes, ctx->stream) != cudaSuccess) break;
      if ((st = gpl_run_plan(ctx, probe.c_str(), 0))) break;
      if (cudaStreamSynchronize(ctx->stream) != cudaSuccess) break;
      float m = 0;
      cudaEventElapsedTime(&m, ctx->ev0, ctx->ev1);
      if (rep > 0) ms.push_back(m);
    }
    if (st) {  // a candidate that cannot run (resources) is skipped
      st = GPL_OK;
      ctx->err.clear();
      continue;
    }
    if (ms.size() < 3) continue;
    std::sort(ms.begin(), ms.end());
    tried++;
    if (std::getenv("GPL_DEBUG_TUNE"))
      std::fprintf(stderr, "autotune: split %d(eff %d) k %d S %d D %d W %d dr %d np %d tile %lld: %.4f ms (model %.4f)"
                   " prod %.4f cons %.4f launch %.4f r_issue %.3f r_lat %.3f\n",
                   sc.first, cand_split_eff[ci], c.ctas_per_sm, c.stage_rows, c.depth, c.warps, c.ndrain, c.npack,
                   (long long)c.tile_rows, ms[1], c.pred_ms, c.t_prod_ms, c.t_cons_ms, c.t_launch_ms, c.r_issue,
                   c.r_lat);
    if (ms[1] < best_ms) {
      best_ms = ms[1];
      best = t;
      best_eff_split = cand_split_eff[ci];
    }
  }
  take_device_errors(ctx);
  if (tried == 0) {
    ctx->tuned.erase(seg.text);
    return fail(ctx, GPL_E_CUDA, "no candidate configuration could run");
  }
  ctx->tuned[seg.text] = best;
  ctx->run_cache.erase(probe + "\x1f" + std::to_string(0));
  for (auto& kv : ctx->graphs) cudaGraphExecDestroy(kv.second);
  ctx->graphs.clear();
  if (out) {
    const Config c = predict(ctx, d, li, std::max<int64_t>(d.nrows, 1), best.tile_rows, best.stage_rows, best.depth,
                             best.warps, best.ctas_per_sm, best.npack, best.ndrain);
    *out = gpl_model_report{};
    out->tile_rows = c.tile_rows;
    out->stage_rows = c.stage_rows;
    out->ring_depth = c.depth;
    out->consumer_warps = c.warps;
    out->grid = c.grid;
    out->predicted_ms = c.pred_ms;
    out->t_stream_ms = c.t_stream_ms;
    out->t_probe_ms = c.t_probe_ms;
    out->t_tail_ms = c.t_tail_ms;
    out->t_launch_ms = c.t_launch_ms;
    out->bw_gbs = c.bw_gbs;
    out->smem_bytes = c.smem;
    out->feasible = c.feasible;
    out->ctas_per_sm = c.ctas_per_sm;
    out->candidates = tried;
    out->measured_ms = best_ms;
    out->probe_split = best_eff_split;
    out->builds_tuned = builds_tuned;
    out->build_ms_model = build_ms_model;
    out->build_ms = build_ms;
  }
  return GPL_OK;
}

GPL_API gpl_status gpl_compile_plan(gpl_ctx* ctx, const char* probe_segment, int64_t tile_rows) {
  if (!ctx || !probe_segment) return GPL_E_ARG;
  if (gpl_status rs = resolve_pending(ctx)) return rs;  // loads still in flight (A0)
  ctx->err.clear();
  PipeDesc d;
  LowerInfo li;
  Config cfg;
  Segment seg;
  gpl_status st;
  std::string err;
  if (!parse_segment(probe_segment, &seg, &err)) return fail(ctx, GPL_E_PLAN, err);
  if (seg.is_build) {  // the pipelined build of a DIRECT table (others use the precompiled build kernels)
    BuildDesc bd;
    HashTable shape;
    bool trivial = false;
    if ((st = lower_build(ctx, seg, &bd, &shape, &trivial, &err))) return fail(ctx, st, err);
    if (shape.kind != HT_DIRECT || !ctx->opt.build_pipeline) return GPL_OK;
    if ((st = lower_build_pipe(ctx, seg, shape, &d, &cfg))) return st;
  } else if ((st = prepare_run(ctx, probe_segment, tile_rows, &d, &li, &cfg, &seg))) {
    return st;
  }
  if (!ctx->host_only && (st = check_dev(ctx))) return st;
  if (!jit_prepare(d, !ctx->host_only, &err)) return fail(ctx, GPL_E_STATE, err);
  return GPL_OK;
}

GPL_API gpl_status gpl_run_plan_kbe(gpl_ctx* ctx, const char* probe_segment) {
  if (!ctx || !probe_segment) return GPL_E_ARG;
  if (gpl_status rs = resolve_pending(ctx)) return rs;  // loads still in flight (A0)
  ctx->err.clear();
  gpl_status st = check_dev(ctx);
  if (st) return st;
  PipeDesc d;
  LowerInfo li;
  Config cfg;
  Segment seg;
  // every probe reads its keys from materialised columns: lower with no
  // stage-phase probe, and every column materialised by the map kernels (no
  // late materialisation: KBE reads each column it uses in full)
  const int64_t lazy_opt = ctx->opt.lazy_columns;
  ctx->opt.lazy_columns = 0;
  st = prepare_run(ctx, probe_segment, 0, &d, &li, &cfg, &seg, 0);
  ctx->opt.lazy_columns = lazy_opt;
  if (st) return st;
  if (li.hash_group) return fail(ctx, GPL_E_PLAN, "the KBE baseline has no hash group-by ('group hash')");
  if (d.fan_probe >= 0) return fail(ctx, GPL_E_PLAN, "the KBE baseline has no fan-out join (a 'multi' table)");
  const size_t pbytes = (size_t)li.ngroups_total * li.nagg * 16;
  d.partials = partials_ptr(ctx);
  d.tile_counter = counter_ptr(ctx);
  d.op_pass = op_pass_ptr(ctx);
  d.err = err_ptr(ctx);
  CK(cudaMemsetAsync(counter_ptr(ctx), 0, run_clear_bytes(pbytes), ctx->stream));
  double inter = 0;
  // GPL (w/o CE): the same kernel-at-a-time sequence, one tile
  // of kbe_tile_rows at a time (tiling without concurrency or channels)
  const int64_t tile = ctx->opt.kbe_tile_rows > 0 ? std::min<int64_t>(ctx->opt.kbe_tile_rows, std::max<long long>(d.nrows, 1))
                                                   : std::max<long long>(d.nrows, 1);
  PipeDesc dt = d;
  dt.nrows = tile;
  const size_t need = kbe_pool_bytes(dt, ctx->opt.kbe_tile_rows > 0);
  if (ctx->kbe_cap < need) {
    CK(cudaStreamSynchronize(ctx->stream));
    if (ctx->kbe_buf) cudaFree(ctx->kbe_buf);
    ctx->kbe_buf = nullptr;
    ctx->kbe_cap = 0;
    cudaError_t e = cudaMalloc(&ctx->kbe_buf, need);
    if (e != cudaSuccess) return fail(ctx, GPL_E_NOMEM, std::string("KBE buffers: ") + cudaGetErrorString(e));
    ctx->kbe_cap = need;
  }
  // GPL (w/o CE): tiles run back to back with device-side cardinalities (no
  // host round trip per tile or operator); KBE: the host sizes each operator
  const bool tiled = ctx->opt.kbe_tile_rows > 0;
  if (tiled && !ctx->d_kbe_bytes) CK(cudaMalloc(&ctx->d_kbe_bytes, sizeof(unsigned long long)));
  if (tiled) CK(cudaMemsetAsync(ctx->d_kbe_bytes, 0, sizeof(unsigned long long), ctx->stream));
  auto tile_loop = [&](double* inter_out) -> cudaError_t {
    for (long long r0 = 0; r0 < d.nrows || (r0 == 0 && d.nrows == 0); r0 += tile) {
      dt = d;
      dt.nrows = std::min<long long>(tile, d.nrows - r0);
      for (int c = 0; c < d.ncols; c++) dt.col[c] = d.col[c] + r0 * d.colw[c];
      double tb = 0;
      cudaError_t e = run_kbe(dt, ctx->sms, ctx->stream, ctx->kbe_buf, ctx->kbe_cap, &tb, tiled ? ctx->d_kbe_bytes : nullptr);
      if (e != cudaSuccess) return e;
      *inter_out += tb;
      if (d.nrows == 0) break;
    }
    return cudaSuccess;
  };
  // GPL (w/o CE) on B200: the tiles' kernel sequence (map, scan, count, scatter
  // per operator, device-side cardinalities) is launch-bound at small tiles, so
  // the whole loop is captured once as a CUDA graph and replayed (the kernels
  // still run one after another, tile by tile, intermediates materialised)
  cudaStreamCaptureStatus capturing = cudaStreamCaptureStatusNone;
  CK(cudaStreamIsCapturing(ctx->stream, &capturing));
  const bool use_graph = tiled && ctx->opt.kbe_graph != 0 && d.nrows > tile && capturing == cudaStreamCaptureStatusNone;
  gpl_ctx::KbeGraph* G = nullptr;
  if (use_graph) {
    G = &ctx->kbe_graphs[seg.text + "#" + std::to_string(tile)];
    const std::vector<char> key((const char*)&d, (const char*)&d + sizeof(d));
    if (!G->exec || G->desc != key || G->buf != ctx->kbe_buf || G->cap != ctx->kbe_cap || G->opt_version != ctx->opt_version) {
      if (G->exec) cudaGraphExecDestroy(G->exec);
      G->exec = nullptr;
      double gi = 0;
      cudaGraph_t graph = nullptr;
      // a stream that cannot be captured (the legacy default stream) or a graph
      // that does not instantiate falls back to launching the loop
      if (cudaStreamBeginCapture(ctx->stream, cudaStreamCaptureModeThreadLocal) == cudaSuccess) {
        const cudaError_t le = tile_loop(&gi);
        const cudaError_t ce = cudaStreamEndCapture(ctx->stream, &graph);
        CK(le);
        if (ce == cudaSuccess && graph && cudaGraphInstantiate(&G->exec, graph, 0) != cudaSuccess) G->exec = nullptr;
        if (graph) cudaGraphDestroy(graph);
      }
      cudaGetLastError();
      if (G->exec) {
        G->desc = key;
        G->buf = ctx->kbe_buf;
        G->cap = ctx->kbe_cap;
        G->opt_version = ctx->opt_version;
        G->inter = gi;
      } else {
        G = nullptr;
      }
    }
  }
  CK(cudaEventRecord(ctx->ev0, ctx->stream));
  if (G) {
    CK(cudaGraphLaunch(G->exec, ctx->stream));
    inter += G->inter;
  } else {
    CK(tile_loop(&inter));
  }
  CK(cudaEventRecord(ctx->ev1, ctx->stream));
  if (tiled) {  // the materialised bytes, read once after the run
    unsigned long long db = 0;
    CK(cudaMemcpyAsync(&db, ctx->d_kbe_bytes, sizeof(db), cudaMemcpyDeviceToHost, ctx->stream));
    CK(cudaStreamSynchronize(ctx->stream));
    inter += (double)db;
  }
  LastRun& L = ctx->last;
  L.valid = true;
  L.kbe = true;
  L.copied_out = false;
  L.overflowed = false;
  {
    auto kr = std::make_shared<PreparedRun>();
    kr->desc = d;
    kr->li = li;
    kr->text = seg.text;
    L.run = kr;
  }
  L.timed = true;
  gpl_stats& S = L.stats;
  S = gpl_stats{};
  S.rows_scanned = d.nrows;
  S.n_ops = li.nops;
  S.probe_split = -1;
  S.bytes_scanned = (double)d.nrows * li.bytes_per_row_all;  // KBE reads every column it uses
  S.bytes_full_scan = S.bytes_scanned;
  S.agg_mode = AGG_GLOBAL;
  S.kbe = 1;
  S.intermediate_bytes = inter;
  S.tile_rows_used = ctx->opt.kbe_tile_rows > 0 ? tile : 0;
  return GPL_OK;
}

GPL_API gpl_status gpl_sync(gpl_ctx* ctx) {
  if (!ctx) return GPL_E_ARG;
  if (gpl_status rs = resolve_pending(ctx)) return rs;  // loads still in flight (A0)
  gpl_status st = check_dev(ctx);
  if (st) return st;
  CK(cudaStreamSynchronize(ctx->stream));
  return take_device_errors(ctx);
}

// The host-visible side of a finished run (its counters are in h_stage after
// a stream synchronise): kernel time, pass counts, the kernel's own bytes, and
// the plan's λ profile / the model's profiling input while they are missing.
static void observe_run(gpl_ctx* ctx) {
  const LowerInfo& li = ctx->last.run->li;
  const unsigned long long* hs = (const unsigned long long*)ctx->h_stage;
  const unsigned long long* ops = hs + 2;
  gpl_stats& S = ctx->last.stats;
  if (ctx->last.timed) {
    float ms = 0;
    if (cudaEventElapsedTime(&ms, ctx->ev0, ctx->ev1) == cudaSuccess) S.kernel_ms = ms;
  }
  for (int i = 0; i < MAXOPS && i < 16; i++) S.op_pass[i] = (int64_t)ops[i];
  if (!ctx->last.kbe) {
    // the kernel's own HBM bytes per launch (sector-granular):
    // staged columns x rows + the clustered probe's table cells + for every
    // lazy column one 32-B sector per row that reached its first use (a
    // scattered gather moves a whole sector), at most the column's full scan
    const double N = (double)S.rows_scanned;
    double b = N * li.bytes_per_row + (N > 0 ? li.cl_bytes : 0.0);
    for (size_t i = 0; i < li.lazy_w.size(); i++) {
      const int op = li.lazy_reach[i];
      const double reach = op >= 0 && op < MAXOPS ? (double)ops[op] : N;
      b += std::min(reach * 32.0, N * li.lazy_w[i]);
    }
    S.bytes_scanned = b;
  }
  // λ cache for the model / split choice (cumulative pass fraction after each op)
  // (recorded once per plan text: the first run profiles the plan)
  if (!ctx->last.kbe && S.rows_scanned > 0 && !ctx->lambda.count(ctx->last.run->text)) {
    std::vector<double> lam;
    for (int i = 0; i < li.nops; i++) lam.push_back((double)ops[i] / (double)S.rows_scanned);
    ctx->lambda[ctx->last.run->text] = lam;
  } else if (!ctx->last.kbe && ctx->last.timed && S.kernel_ms > 0 && S.rows_scanned > 0 && ctx->last.run->lambda_n > 0 &&
             !profile_current(ctx, ctx->last.run->text, ctx->last.run->li.table)) {
    // the first two timed runs planned with λ (same shape; the faster one —
    // the first may pay cold TLB/L2 misses after a load): the model's
    // profiling input
    const PreparedRun& R = *ctx->last.run;
    auto ti = ctx->tables.find(R.li.table);
    const uint64_t ver = ti != ctx->tables.end() ? ti->second.version : 0;
    auto old = ctx->profile.find(R.text);
    if (old != ctx->profile.end() && old->second.runs == 1 && old->second.table_version == ver &&
        old->second.tile_rows == R.desc.tile_rows && old->second.stage_rows == R.desc.stage_rows &&
        old->second.depth == R.desc.depth && old->second.warps == R.desc.nwarps && old->second.npack == R.desc.npack &&
        old->second.ndrain == R.desc.ndrain) {
      old->second.kernel_ms = std::min(old->second.kernel_ms, S.kernel_ms);
      old->second.runs = 2;
    } else {
      RunProfile p;
      p.nrows = R.desc.nrows;
      p.tile_rows = R.desc.tile_rows;
      p.stage_rows = R.desc.stage_rows;
      p.depth = R.desc.depth;
      p.warps = R.desc.nwarps;
      p.npack = R.desc.npack;
      p.ndrain = R.desc.ndrain;
      p.ctas_per_sm = std::max(1, R.grid / std::max(1, ctx->sms));
      p.kernel_ms = S.kernel_ms;
      p.table_version = ver;
      p.runs = 1;
      ctx->profile[R.text] = p;
    }
  }
}

// Whether the plan of the last run still profiles (λ, then the model's two
// profiled runs): its counters must then reach the host even when the caller
// only takes the partials on the device (multi-rank merge).
static bool run_profiling(gpl_ctx* ctx) {
  if (ctx->last.kbe || !ctx->last.run) return false;
  if (!ctx->lambda.count(ctx->last.run->text)) return true;
  return ctx->last.timed && ctx->last.run->lambda_n > 0 &&
         !profile_current(ctx, ctx->last.run->text, ctx->last.run->li.table);
}

// Bring the run's error bits, counters and partials to h_stage (one D2H unless
// the fused run's copy-out kernel already wrote them) and synchronise.
static gpl_status stage_run_to_host(gpl_ctx* ctx) {
  const size_t pbytes = run_pbytes(ctx->last.run->li);
  if (!ctx->last.copied_out)
    CK(cudaMemcpyAsync(ctx->h_stage, ctx->d_scratch, kScratchHead * 8 + pbytes, cudaMemcpyDeviceToHost, ctx->stream));
  CK(cudaStreamSynchronize(ctx->stream));
  return GPL_OK;
}

GPL_API gpl_status gpl_fetch_result(gpl_ctx* ctx, gpl_result* out) {
  if (!ctx || !out) return GPL_E_ARG;
  if (gpl_status rs = resolve_pending(ctx)) return rs;  // loads still in flight (A0)
  ctx->err.clear();
  gpl_status st = check_dev(ctx);
  if (st) return st;
  if (!ctx->last.valid) return fail(ctx, GPL_E_STATE, "no run to fetch");
  const LowerInfo& li = ctx->last.run->li;
  // one D2H: error bits, counter, op_pass and partials are contiguous
  if ((st = stage_run_to_host(ctx))) return st;
  const unsigned long long* hs = (const unsigned long long*)ctx->h_stage;
  const unsigned int bits = (unsigned int)hs[0];
  const unsigned long long* part = hs + kScratchHead;
  gpl_stats& S = ctx->last.stats;
  observe_run(ctx);
  if (li.hash_group) {
    // distinct groups size the next run's table (load <= 1/2); an overflow
    // (ERR_CAPACITY) quadruples it
    const uint64_t seen = part[0];
    const uint64_t cap = ctx->last.run->hagg_cap;
    auto& est = ctx->hagg_groups[ctx->last.run->text];
    est.first = (bits & ERR_CAPACITY) ? std::max<uint64_t>(2 * cap, seen) : seen;
    if (bits & ERR_CAPACITY) ctx->last.overflowed = true;
    est.second = (int64_t)S.rows_scanned;
    S.groups_total = (int64_t)seen;
  }
  out->stats = S;
  if (bits) {
    if ((st = take_device_errors(ctx))) {
      if (li.hash_group && st == GPL_E_CAPACITY)
        return fail(ctx, st, "hash group-by table overflowed (" + std::to_string(ctx->last.run->hagg_cap) +
                                 " slots); the next run of the plan uses a larger table");
      return st;
    }
  }
  if (li.hash_group) return decode_hash(ctx, part, out);
  return decode(ctx, part, out);
}

GPL_API gpl_status gpl_fetch_partials(gpl_ctx* ctx, void* dst, int32_t dst_on_device, size_t cap_bytes, size_t* nbytes) {
  if (!ctx || !nbytes) return GPL_E_ARG;
  gpl_status st = check_dev(ctx);
  if (st) return st;
  if (!ctx->last.valid) return fail(ctx, GPL_E_STATE, "no run");
  if (ctx->last.run->li.hash_group)
    return fail(ctx, GPL_E_STATE, "a hash group-by has no dense partial vector (fetch its rows with gpl_fetch_result)");
  const size_t b = (size_t)ctx->last.run->li.ngroups_total * ctx->last.run->li.nagg * 16;
  *nbytes = b;
  if (cap_bytes < b || !dst) return fail(ctx, GPL_E_CAPACITY, "partials buffer too small");
  // while the plan profiles (its first runs), the counters reach the host
  // here too, so a multi-rank caller (which never fetches the rank's own
  // result) gets the same λ-planned, profile-fitted plan as a single rank
  if (run_profiling(ctx)) {
    if ((st = stage_run_to_host(ctx))) return st;
    observe_run(ctx);
  }
  CK(cudaMemcpyAsync(dst, partials_ptr(ctx), b, dst_on_device ? cudaMemcpyDeviceToDevice : cudaMemcpyDeviceToHost,
                     ctx->stream));
  if (!dst_on_device) CK(cudaStreamSynchronize(ctx->stream));
  return GPL_OK;
}

GPL_API gpl_status gpl_decode_partials(gpl_ctx* ctx, const void* host_partials, size_t nbytes, gpl_result* out) {
  if (!ctx || !host_partials || !out) return GPL_E_ARG;
  if (gpl_status rs = resolve_pending(ctx)) return rs;  // loads still in flight (A0)
  if (!ctx->last.valid) return fail(ctx, GPL_E_STATE, "no run (the plan of the last run defines the layout)");
  if (ctx->last.run->li.hash_group) return fail(ctx, GPL_E_STATE, "a hash group-by has no dense partial vector");
  const size_t b = (size_t)ctx->last.run->li.ngroups_total * ctx->last.run->li.nagg * 16;
  if (nbytes != b) return fail(ctx, GPL_E_ARG, "partials size does not match the last run's plan");
  gpl_stats& S = ctx->last.stats;
  if (ctx->last.timed && !ctx->host_only && cudaEventQuery(ctx->ev1) == cudaSuccess) {
    float ms = 0;
    if (cudaEventElapsedTime(&ms, ctx->ev0, ctx->ev1) == cudaSuccess) S.kernel_ms = ms;
  }
  out->stats = S;
  return decode(ctx, (const unsigned long long*)host_partials, out);
}

GPL_API gpl_status gpl_merge_partials(const void* gathered, int32_t nranks, size_t nbytes_each, void* out) {
  if (!gathered || !out || nranks < 1 || nbytes_each % 16) return GPL_E_ARG;
  const size_t n = nbytes_each / 16;
  const unsigned long long* in = (const unsigned long long*)gathered;
  unsigned long long* o = (unsigned long long*)out;
  for (size_t i = 0; i < n; i++) {
    unsigned __int128 acc = 0;
    for (int r = 0; r < nranks; r++) {  // fixed order: rank 0, 1, ...
      const unsigned long long* p = in + (size_t)r * n * 2 + 2 * i;
      acc += ((unsigned __int128)p[1] << 64) | p[0];
    }
    o[2 * i] = (unsigned long long)acc;
    o[2 * i + 1] = (unsigned long long)(acc >> 64);
  }
  return GPL_OK;
}

// Hash group-by rows of the last run (NEXT-4 multi-GPU): [packed key, acc 0 .. nagg-1] int64 words per row —
// the LIMIT rows in ORDER BY order, else every group (device compaction order).
GPL_API gpl_status gpl_fetch_groups(gpl_ctx* ctx, int64_t* rows, int64_t cap_rows, int64_t* n_rows,
                                    int32_t* row_words) {
  if (!ctx || !n_rows || cap_rows < 0 || (cap_rows > 0 && !rows)) return GPL_E_ARG;
  ctx->err.clear();
  gpl_status st = check_dev(ctx);
  if (st) return st;
  if (!ctx->last.valid || !ctx->last.run || !ctx->last.run->li.hash_group)
    return fail(ctx, GPL_E_STATE, "gpl_fetch_groups: the last run is not a hash group-by");
  CK(cudaStreamSynchronize(ctx->stream));
  if (run_profiling(ctx)) {  // a multi-rank caller profiles the plan through this call (see gpl_fetch_partials)
    if ((st = stage_run_to_host(ctx))) return st;
    observe_run(ctx);
  }
  // an overflowed aggregation table holds an incomplete group set: never
  // returned as rows (whether or not gpl_fetch_result already took the bits)
  const gpl_status dev_st = take_device_errors(ctx);
  if (dev_st == GPL_E_CAPACITY || ctx->last.overflowed)
    return fail(ctx, GPL_E_STATE, "gpl_fetch_groups: the last run's hash group-by table overflowed; run the plan "
                                  "again (the next run is sized from this one)");
  if (dev_st) return dev_st;
  const LowerInfo& li = ctx->last.run->li;
  const int W = 1 + li.nagg;
  const unsigned long long* part = (const unsigned long long*)ctx->h_stage + kScratchHead;
  const int64_t n = (int64_t)part[1];
  *n_rows = n;
  if (row_words) *row_words = W;
  if (n > cap_rows) return fail(ctx, GPL_E_CAPACITY, "gpl_fetch_groups: rows capacity too small");
  if (n == 0) return GPL_OK;
  if (li.limit > 0) {
    std::memcpy(rows, part + 2, (size_t)n * W * 8);
  } else {
    CK(cudaMemcpyAsync(rows, ctx->last.run->hres.rows, (size_t)n * W * 8, cudaMemcpyDeviceToHost, ctx->stream));
    CK(cudaStreamSynchronize(ctx->stream));
  }
  return GPL_OK;
}

// Merge hash group-by rows of several ranks (concatenated gpl_fetch_groups
// outputs) exactly — int128 sums per key, in input order — then apply the
// probe segment's ORDER BY / LIMIT (else key order) into `out`, as
// gpl_fetch_result would. For a LIMIT plan every rank must ship ALL its
// groups (run the plan without 'order'/'limit') unless the shard key is part
// of the group key (disjoint groups: the union of the ranks' top-k rows holds
// the global top-k).
GPL_API gpl_status gpl_merge_groups(gpl_ctx* ctx, const char* probe_segment, const int64_t* rows, int64_t n_rows,
                                    gpl_result* out) {
  if (!ctx || !probe_segment || !out || n_rows < 0 || (n_rows > 0 && !rows)) return GPL_E_ARG;
  ctx->err.clear();
  Segment s;
  std::string err;
  if (!parse_segment(probe_segment, &s, &err)) return fail(ctx, GPL_E_PLAN, err);
  if (!s.hash_group) return fail(ctx, GPL_E_PLAN, "gpl_merge_groups: the segment has no 'group hash'");
  const int NK = (int)s.groups.size(), A = (int)s.aggs.size(), W = 1 + A;
  auto field = [&](unsigned long long key, int k) {
    return NK == 2 ? (int32_t)(uint32_t)(k == 0 ? key >> 32 : key) : (int32_t)(uint32_t)key;
  };
  std::map<unsigned long long, std::vector<__int128>> acc;
  for (int64_t r = 0; r < n_rows; r++) {
    const unsigned long long key = (unsigned long long)rows[r * W];
    auto it = acc.find(key);
    if (it == acc.end()) it = acc.emplace(key, std::vector<__int128>(A, 0)).first;
    for (int a = 0; a < A; a++) it->second[a] += (__int128)rows[r * W + 1 + a];
  }
  std::vector<std::pair<unsigned long long, const std::vector<__int128>*>> v;
  v.reserve(acc.size());
  for (auto& kv : acc) v.push_back({kv.first, &kv.second});
  auto key_less = [&](unsigned long long a, unsigned long long b) {
    for (int k = 0; k < NK; k++)
      if (field(a, k) != field(b, k)) return field(a, k) < field(b, k);
    return false;
  };
  std::sort(v.begin(), v.end(), [&](const auto& x, const auto& y) {
    for (const OrderIR& o : s.order) {
      __int128 a = o.is_agg ? (*x.second)[o.idx] : (__int128)field(x.first, o.idx);
      __int128 b = o.is_agg ? (*y.second)[o.idx] : (__int128)field(y.first, o.idx);
      if (a != b) return o.desc ? a > b : a < b;
    }
    return key_less(x.first, y.first);
  });
  const int64_t n = s.limit > 0 ? std::min<int64_t>((int64_t)v.size(), s.limit) : (int64_t)v.size();
  out->n_keys = NK;
  out->n_aggs = A;
  out->n_ratios = (int32_t)s.ratios.size();
  out->n_groups = (int32_t)std::min<int64_t>(n, INT32_MAX);
  out->stats = gpl_stats{};
  out->stats.groups_total = (int64_t)v.size();
  out->stats.agg_mode = AGG_HASH;
  if (n > out->cap_groups) return fail(ctx, GPL_E_CAPACITY, "result capacity too small");
  if (n && (!out->keys || !out->aggs)) return fail(ctx, GPL_E_ARG, "NULL result arrays");
  for (int64_t r = 0; r < n; r++) {
    for (int k = 0; k < NK; k++) out->keys[r * NK + k] = field(v[r].first, k);
    for (int a = 0; a < A; a++) {
      const unsigned __int128 u = (unsigned __int128)(*v[r].second)[a];
      out->aggs[(r * A + a) * 2] = (int64_t)(uint64_t)u;
      out->aggs[(r * A + a) * 2 + 1] = (int64_t)(uint64_t)(u >> 64);
    }
  }
  fill_ratios(s.ratios, out, (int)n);
  return GPL_OK;
}

GPL_API gpl_status gpl_choose_tile_rows(gpl_ctx* ctx, const char* probe_segment, int64_t n_rows, gpl_model_report* out) {
  if (!ctx || !probe_segment || !out) return GPL_E_ARG;
  if (gpl_status rs = resolve_pending(ctx)) return rs;  // loads still in flight (A0)
  ctx->err.clear();
  Segment s;
  std::string err;
  if (!parse_segment(probe_segment, &s, &err)) return fail(ctx, GPL_E_PLAN, err);
  PipeDesc d;
  LowerInfo li;
  gpl_status st = lower_probe(ctx, s, choose_split(ctx, s), &d, &li, &err);
  if (st) return fail(ctx, st, err);
  auto lit = ctx->lambda.find(s.text);
  if (lit != ctx->lambda.end()) li.lambda = lit->second;
  for (int i = 0; i < d.nht; i++)
    for (auto& h : ctx->hts)
      if (h.slots == d.ht[i].slots) li.ht_bytes[i] = (int64_t)(h.kind == HT_DIRECT ? h.bytes() : h.bytes() / 2);
  apply_profile(ctx, d, &li, s.text);
  Config c;
  const int64_t N = n_rows > 0 ? n_rows : d.nrows;
  if (!choose_config(ctx, d, li, N, 0, &c, &err)) return fail(ctx, GPL_E_ARG, err);
  out->tile_rows = c.tile_rows;
  out->stage_rows = c.stage_rows;
  out->ring_depth = c.depth;
  out->consumer_warps = c.warps;
  out->grid = c.grid;
  out->predicted_ms = c.pred_ms;
  out->t_stream_ms = c.t_stream_ms;
  out->t_probe_ms = c.t_probe_ms;
  out->t_tail_ms = c.t_tail_ms;
  out->t_launch_ms = c.t_launch_ms;
  out->bw_gbs = c.bw_gbs;
  out->smem_bytes = c.smem;
  out->feasible = c.feasible;
  out->ctas_per_sm = c.ctas_per_sm;
  out->probe_split = d.nsprobe;
  return GPL_OK;
}
