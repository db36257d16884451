// calibrate.cpp — Γ, the channel calibration of the A9 model (SURVEY §8(f)
// NEXT-1; §2.1, §4.1 Eq 1, App. A).
//
// The paper calibrates its data channels with "a simple chain of two kernels,
// producer and consumer. The producer kernel generates N integers and passes
// them to the consumer kernel", for varying data size d, number of
// channels n and packet size p, and feeds the measured throughput Γ(n, p, d)
// to the cost model (Eq 1; Table 2 "calibration").
//
// B200 analog: the channel is the fused kernel's shared-memory ring (TMA
// producer warp -> mbarrier full/empty -> consumer warps). Γ is measured by
// streaming a synthetic table of d rows (2 int32 + 1 int64 columns, 16 B/row,
// all zero) through the pipeline kernel with a consumer that touches every
// staged byte (two all-pass filters, a column sum), for every ring shape
// (n = ring depth, s = stage rows — the packet analog — and k CTAs per SM):
//   Γ(n, s, k, d) = d·16 B / (t(d) − t0(n, s, k)),
// with t(d) the median kernel time over an L2 flush (CUDA events on the ctx
// stream) and t0 the same shape over an empty input (launch + prologue +
// teardown). The model (costmodel.cpp predict) then uses Γ of its candidate
// shape at d = N·b in place of the copy bandwidth, and t0 as its launch term.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstring>
#include <iterator>
#include <string>
#include <vector>

#include "ctx.h"
#include "gpl.h"

#define GPL_API extern "C" __attribute__((visibility("default")))

using namespace gpl;

namespace {

const char* kGammaTable = "__gamma";
const char* kGammaPlan =
    "run __gamma\n"
    "filter g0 >= 0\n"
    "filter g1 >= 0\n"
    "value x0\n"
    "agg count\n"
    "agg sum\n";
constexpr int kRowBytes = 16;

gpl_status cfail(gpl_ctx* ctx, gpl_status st, const std::string& m) {
  ctx->err = m;
  return st;
}

}  // namespace

namespace gpl {

// Γ of a shape at `bytes` streamed (GB/s) and its empty-input time (ms): the
// calibrated shape with the same stage rows and CTAs per SM and the nearest
// ring depth, log-linear in d between calibrated sizes (clamped at the ends).
// Returns false when the context has no calibration.
bool gamma_lookup(const gpl_ctx* ctx, int depth, int stage_rows, int k, double bytes, double* gbs, double* t0_ms) {
  if (ctx->gamma.empty() || !ctx->opt.use_gamma) return false;
  const GammaCurve* best = nullptr;
  int best_d = 1 << 30;
  for (const auto& kv : ctx->gamma) {
    const GammaCurve& c = kv.second;
    if (c.stage_rows != stage_rows || c.ctas_per_sm != k || c.pts.empty()) continue;
    const int dd = std::abs(c.depth - depth);
    if (dd < best_d) {
      best_d = dd;
      best = &c;
    }
  }
  if (!best) return false;
  const auto& P = best->pts;  // sorted by bytes
  double g;
  if (bytes <= P.front().first) {
    g = P.front().second;
  } else if (bytes >= P.back().first) {
    g = P.back().second;
  } else {
    size_t i = 1;
    while (P[i].first < bytes) i++;
    const double x0 = std::log(P[i - 1].first), x1 = std::log(P[i].first);
    const double w = (std::log(bytes) - x0) / (x1 - x0);
    g = P[i - 1].second * (1 - w) + P[i].second * w;
  }
  *gbs = g;
  *t0_ms = best->t0_ms;
  return true;
}

}  // namespace gpl

GPL_API gpl_status gpl_set_option(gpl_ctx* ctx, const char* key, int64_t value);
GPL_API gpl_status gpl_load_columns(gpl_ctx* ctx, const char* table, int64_t nrows, int32_t ncols,
                                    const gpl_column* cols, uint32_t flags);
GPL_API gpl_status gpl_run_plan(gpl_ctx* ctx, const char* probe_segment, int64_t tile_rows);

GPL_API gpl_status gpl_set_calibration(gpl_ctx* ctx, const gpl_gamma_point* pts, int32_t n) {
  if (!ctx || (n > 0 && !pts) || n < 0) return GPL_E_ARG;
  ctx->err.clear();
  ctx->gamma.clear();
  for (int i = 0; i < n; i++) {
    const gpl_gamma_point& p = pts[i];
    if (p.gbs <= 0 || p.bytes <= 0 || p.stage_rows <= 0 || p.ring_depth <= 0 || p.ctas_per_sm <= 0)
      return cfail(ctx, GPL_E_ARG, "gpl_set_calibration: point " + std::to_string(i) + " is not positive");
    GammaCurve& c = ctx->gamma[{p.ring_depth, p.stage_rows, p.ctas_per_sm}];
    c.depth = p.ring_depth;
    c.stage_rows = p.stage_rows;
    c.ctas_per_sm = p.ctas_per_sm;
    c.t0_ms = p.t0_ms;
    c.pts.push_back({p.bytes, p.gbs});
  }
  for (auto& kv : ctx->gamma) std::sort(kv.second.pts.begin(), kv.second.pts.end());
  ctx->opt_version++;  // prepared plans were configured with the old model
  ctx->tuned.clear();
  return GPL_OK;
}

GPL_API gpl_status gpl_calibrate(gpl_ctx* ctx, const int64_t* rows, int32_t n_rows, gpl_gamma_point* out,
                                 int32_t cap, int32_t* n_out) {
  if (!ctx || n_rows < 0 || (n_rows > 0 && !rows) || cap < 0 || (cap > 0 && !out)) return GPL_E_ARG;
  ctx->err.clear();
  if (ctx->host_only) return cfail(ctx, GPL_E_NODEV, "gpl_calibrate needs a device context");
  std::vector<int64_t> sizes;
  if (n_rows > 0) sizes.assign(rows, rows + n_rows);
  else sizes = {1 << 19, 1 << 20, 1 << 21, 1 << 22, 1 << 23, 1 << 24, 1 << 26};  // 16 MB .. 2 GB (512K..8M)
  for (int64_t r : sizes)
    if (r <= 0 || r > (int64_t)1 << 28) return cfail(ctx, GPL_E_ARG, "gpl_calibrate: rows in [1, 2^28]");
  std::sort(sizes.begin(), sizes.end());
  const int64_t maxr = sizes.back();
  const int64_t capr = (maxr + 8191) / 8192 * 8192 + 8192;
  // one zeroed buffer: 2 int32 + 1 int64 columns of capr rows; an L2 flush buffer
  char* buf = nullptr;
  void* flush = nullptr;
  const size_t fbytes = (size_t)2 * ctx->l2_bytes;
  auto release = [&]() {
    if (buf) cudaFree(buf);
    if (flush) cudaFree(flush);
  };
  if (cudaMalloc(&buf, (size_t)capr * kRowBytes) != cudaSuccess || cudaMalloc(&flush, fbytes) != cudaSuccess) {
    release();
    cudaGetLastError();
    return cfail(ctx, GPL_E_NOMEM, "gpl_calibrate: device allocation");
  }
  if (cudaMemsetAsync(buf, 0, (size_t)capr * kRowBytes, ctx->stream) != cudaSuccess) {
    release();
    return cfail(ctx, GPL_E_CUDA, "gpl_calibrate: memset");
  }
  const char* names[3] = {"g0", "g1", "x0"};
  gpl_column cols[3];
  size_t off = 0;
  for (int i = 0; i < 3; i++) {
    cols[i] = gpl_column{names[i], i < 2 ? GPL_I32 : GPL_I64, 0, buf + off, 1, 0, capr};
    off += (size_t)capr * (i < 2 ? 4 : 8);
  }
  const Options saved = ctx->opt;
  std::vector<gpl_gamma_point> pts;
  gpl_status st = GPL_OK;
  auto set = [&](const char* k, int64_t v) { return gpl_set_option(ctx, k, v); };
  // the shapes: ring depth n, stage rows s (the packet analog), CTAs per SM k;
  // 8 consumer warps, a plan-specialised kernel per shape as in a query
  const int depths[] = {2, 3, 4};
  const int stages[] = {1024, 2048, 4096};
  const int ks[] = {1, 2};
  set("lazy_columns", 0);
  set("consumer_warps", 8);
  set("packets", 1);
  for (int k : ks)
    for (int s : stages)
      for (int n : depths) {
        if (set("ctas_per_sm", k) || set("stage_rows", s) || set("ring_depth", n)) continue;
        auto time_rows = [&](int64_t r, double* ms_out) -> gpl_status {
          gpl_status e = gpl_load_columns(ctx, kGammaTable, r, 3, cols, GPL_BORROW);
          if (e) return e;
          std::vector<float> ms;
          for (int rep = 0; rep < 4; rep++) {
            if (cudaMemsetAsync(flush, rep, fbytes, ctx->stream) != cudaSuccess) return GPL_E_CUDA;
            // Δ = 2 stages per claim: the scheduler is calibrated, not the wave tail
            if ((e = gpl_run_plan(ctx, kGammaPlan, 2 * (int64_t)s))) return e;
            if (cudaStreamSynchronize(ctx->stream) != cudaSuccess) return GPL_E_CUDA;
            float m = 0;
            cudaEventElapsedTime(&m, ctx->ev0, ctx->ev1);
            if (rep > 0) ms.push_back(m);
          }
          std::sort(ms.begin(), ms.end());
          *ms_out = ms[1];
          return GPL_OK;
        };
        double t0 = 0;
        if (time_rows(1, &t0)) {  // shape does not fit (shared memory): skipped
          ctx->err.clear();
          cudaGetLastError();
          continue;
        }
        for (int64_t r : sizes) {
          double t = 0;
          if ((st = time_rows(r, &t))) break;
          gpl_gamma_point p{};
          p.ring_depth = n;
          p.stage_rows = s;
          p.ctas_per_sm = k;
          p.consumer_warps = 8;
          p.rows = r;
          p.bytes = (double)r * kRowBytes;
          p.ms = t;
          p.t0_ms = t0;
          p.gbs = p.bytes / (std::max(t - t0, 1e-4) * 1e-3) / 1e9;
          pts.push_back(p);
        }
        if (st) break;
      }
  // restore the caller's options, drop the synthetic table and its plan state
  ctx->opt = saved;
  ctx->opt_version++;
  ctx->tuned.clear();
  ctx->tables.erase(kGammaTable);
  ctx->lambda.erase(kGammaPlan);
  for (auto it = ctx->run_cache.begin(); it != ctx->run_cache.end();)
    it = it->first.compare(0, std::strlen(kGammaPlan), kGammaPlan) == 0 ? ctx->run_cache.erase(it) : std::next(it);
  ctx->last = LastRun{};
  cudaStreamSynchronize(ctx->stream);
  release();
  if (st) return st;
  if (pts.empty()) return cfail(ctx, GPL_E_CUDA, "gpl_calibrate: no ring shape could run");
  gpl_status s2 = gpl_set_calibration(ctx, pts.data(), (int32_t)pts.size());
  if (s2) return s2;
  if (n_out) *n_out = (int32_t)pts.size();
  if (cap < (int32_t)pts.size()) return out ? cfail(ctx, GPL_E_CAPACITY, "gpl_calibrate: out too small") : GPL_OK;
  std::copy(pts.begin(), pts.end(), out);
  return GPL_OK;
}
