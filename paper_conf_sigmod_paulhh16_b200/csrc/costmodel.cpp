// costmodel.cpp — A9: the paper's analytical model (§4.1, Table 2,
// Eqs 1-9) re-derived for one fused persistent kernel on B200.
//
// Paper term (AMD APU / K40)             -> here (B200, one kernel per segment)
//   Γ(n,p,d), Eq 1 (channel calibration) -> B_eff: calibrated HBM stream rate
//                                           (gpl ctx hbm_gbs, the measured copy BW)
//   Eq 2 resource constraints             -> smem_bytes() <= 227 KB/CTA, warps <= 16
//   Eq 3 req = wg / (a_wg * a_CU)         -> waves = ceil(ceil(N/Δ) / G), G = k * #SM
//   Eq 4 compute cost (inst * w * req)    -> t_cons: per warp iteration, probe latencies +
//                                           warp-instructions (profile-scaled) + stage
//                                           hand-off, over the warps with work; soft-capped
//                                           by 4 schedulers * f * #SM * 70% issue; per wave
//   Eq 5 memory cost, cache hit ratio cr  -> t_prod: (N*b + Σ_j λ_j N 32B (1-cr_j)) / B_eff,
//                                           cr_j = min(1, L2_eff / HT_bytes_j)
//   Eq 6 channel cost Δλ/Γ                -> ≈0: channels are on-chip smem queues;
//                                           kept as the per-stage ring handoff cost and
//                                           the ring-refill latency the n-1 other slots
//                                           must cover
//   Eq 7 T_K = c_K + m_K                  -> per-role times t_prod (TMA warp), t_cons
//   Eq 8 delay |T_i r_i - T_j r_j|        -> |t_prod - t_cons| between the two roles
//   Eq 9 T_S = (1/C) Σ T_K + delay, C = 2 -> T = ½(t_prod + t_cons) + ½|t_prod - t_cons|
//                                           (= max of the two roles: C = 2 roles overlap,
//                                           the delay is shared by both), plus the
//                                           last-wave tail and launch/fill latency
//   Search over (Δ, n, p, wg_K), <5 ms    -> grid search over (Δ, stage rows, ring depth,
//                                           consumer warps); microseconds
// λ (Table 2, "query optimizer") comes from the previous run's per-operator
// pass counters — the paper profiles the first tile for the same purpose.
// Parity of this model is UNPINNED against the paper (its numbers were in the
// missing figures); experiments.py knobs / model report Eq 10's relative error
// over the config-2 sweep and the model's pick against gpl_autotune at SF 100.
#include "costmodel.h"

#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <map>
#include <tuple>

namespace gpl {

int pipeline_fixed_smem();
int pipeline_max_consumer_warps();
bool gamma_lookup(const gpl_ctx* ctx, int depth, int stage_rows, int k, double bytes, double* gbs, double* t0_ms);

namespace {
constexpr int kFixed = 4096;
int align128(int x) { return (x + 127) & ~127; }
}  // namespace

// Cell buffer of a clustered probe per ring slot: a stage's key range spans
// cl_kpr keys per row (twice the column's average, set by the lowering; a
// wider range falls back to probing the table in memory).
int cl_cap_bytes(const PipeDesc& d, int S) {
  if (d.cl_probe < 0) return 0;
  const int w = d.ht[d.probe[d.cl_probe].ht].width;
  const int kpr = d.cl_kpr > 0 ? d.cl_kpr : 4;
  return align128((w == 0 ? (kpr * S + 7) / 8 : w == W_NIBBLE ? (kpr * S + 1) / 2 : kpr * S * w) + 32);
}

int smem_bytes(const PipeDesc& d, const LowerInfo& li, int stage_rows, int depth, int warps, int ndrain) {
  // per-warp queues of the stage warps + the 2*ndrain hand-off slots
  int q = (warps + ndrain) * d.qbytes;
  int agg = d.agg_mode == AGG_SMEM ? li.ngroups_total * li.nagg * 8 * std::max(1, d.agg_lanes) : 0;
  int slot = 0;
  for (int c = 0; c < d.ncols; c++)
    if (!d.lazy[c]) slot += align128(stage_rows * d.colw[c]);
  slot += cl_cap_bytes(d, stage_rows);
  return align128(kFixed + q) + align128(agg) + align128(d.smem_tables_bytes) + depth * slot;
}

void apply_config(PipeDesc* d, const LowerInfo& li, const Config& c) {
  d->tile_rows = c.tile_rows;
  d->stage_rows = c.stage_rows;
  d->depth = c.depth;
  d->nwarps = c.warps;
  d->npack = c.npack;
  d->min_blocks = c.ctas_per_sm;
  d->ndrain = c.ndrain;
  d->off_queue = kFixed;
  d->off_agg = align128(kFixed + (c.warps + c.ndrain) * d->qbytes);
  int agg = d->agg_mode == AGG_SMEM ? li.ngroups_total * li.nagg * 8 * std::max(1, d->agg_lanes) : 0;
  const int off_tables = d->off_agg + align128(agg);
  for (int i = 0; i < d->nht; i++)
    if (d->ht_smem_off[i] >= 0) d->ht_smem_off[i] += off_tables;  // relative -> absolute
  d->off_ring = off_tables + align128(d->smem_tables_bytes);
  int off = 0;
  for (int i = 0; i < d->ncols; i++) {
    if (d->lazy[i]) {  // gathered per surviving row, not staged
      d->coloff[i] = -1;
      continue;
    }
    d->coloff[i] = off;
    off += align128(c.stage_rows * d->colw[i]);
  }
  d->cl_off = off;
  d->cl_cap = cl_cap_bytes(*d, c.stage_rows);
  off += d->cl_cap;
  d->slot_bytes = off;
  d->smem_bytes = d->off_ring + c.depth * off;
}

Config predict(const gpl_ctx* ctx, const PipeDesc& d, const LowerInfo& li, int64_t N, int64_t tile,
               int S, int depth, int W, int k, int npack, int ndrain) {
  Config c;
  c.npack = npack;
  c.ndrain = ndrain;
  c.tile_rows = tile;
  c.stage_rows = S;
  c.depth = depth;
  c.warps = W;
  c.ctas_per_sm = k;
  c.grid = ctx->sms * k;
  c.smem = smem_bytes(d, li, S, depth, W, ndrain);
  // Eq 2 analog: shared memory (228 KB per SM, 1 KB reserved per CTA),
  // threads and registers (<= 80 per thread assumed) of k resident CTAs
  // registers: the generic kernel needs ~80 (112 with two packets); a
  // plan-specialised kernel is compiled with the shape's exact launch bounds,
  // so it fits down to 64 (80) registers per thread
  const int regs_need = ctx->opt.jit ? (npack == 2 ? 80 : 64) : (npack == 2 ? 112 : 80);
  c.feasible = c.smem <= ctx->smem_optin && k * (c.smem + 1024) <= 228 * 1024 && W >= 1 &&
               W <= pipeline_max_consumer_warps() && depth >= 2 && k * (W + 1) * 32 <= 2048 &&
               k * (W + 1) * 32 * regs_need <= 65536 && (npack == 1 || npack == 2) && ndrain >= 0 &&
               ndrain <= 4 && W - ndrain >= 1 && (ndrain == 0 || (d.npush > 0 && !(d.sink != SINK_AGG && d.ins_kcol >= 0 && !d.ins_q) && !d.ins_dense));
  const double B = (ctx->opt.hbm_gbs > 0 ? ctx->opt.hbm_gbs : ctx->hbm_gbs) * 1e9;
  c.bw_gbs = B / 1e9;
  // bytes per row: staged columns, plus one 32-B sector per surviving row of
  // each lazy (gathered) column
  double b = std::max(1, li.bytes_per_row);
  for (size_t i = 0; i < li.lazy_reach.size(); i++) {
    const int op = li.lambda.empty() ? -1 : li.lazy_reach[i];
    b += 32.0 * (op >= 0 && op < (int)li.lambda.size() ? li.lambda[op] : 0.05);
  }
  if (d.cl_probe >= 0 && N > 0) b += li.cl_bytes / (double)N;  // the clustered probe's cells, streamed once
  const double f_sm = 1.9e9;
  // Eq 1 analog: the calibrated ring throughput Γ(n, s, k, d) of this shape at
  // d = N·b (gpl_calibrate) replaces the copy bandwidth as the streaming rate,
  // and the shape's measured empty-input time replaces the launch estimate
  double G_ring = B, t0_cal = -1;
  {
    double g = 0, t0 = 0;
    if (gamma_lookup(ctx, depth, S, k, (double)std::max<int64_t>(N, 1) * b, &g, &t0)) {
      G_ring = g * 1e9;
      t0_cal = t0;
    }
  }
  G_ring *= std::max(li.bw_factor, 1.0);
  c.bw_gbs = G_ring / 1e9;
  const double B_sm = 1.6 * G_ring / ctx->sms;  // one SM's TMA/L2 fill cap
  N = std::max<int64_t>(N, 1);

  // λ: fraction of rows reaching each operator (previous run, else defaults)
  double frac = 1.0;
  std::vector<double> reach;  // rows reaching op i / N
  for (int i = 0; i < li.nops; i++) {
    reach.push_back(frac);
    frac = (int)li.lambda.size() > i ? li.lambda[i] : frac * 0.3;
  }
  reach.push_back(frac);
  // Eq 5 analog: probe sectors that miss L2
  const double L2_eff = 0.5 * ctx->l2_bytes;
  double probe_bytes = 0;
  for (int p = 0; p < li.nprobe; p++) {
    // a clustered probe reads cells the producer streams (counted in b below), a
    // shared-memory table never misses: only the other probes pay L2 misses
    if (p == d.cl_probe || d.ht_smem_off[li.probe_ht[p]] >= 0) continue;
    double ht = li.ht_bytes.empty() ? 1 << 20 : (double)li.ht_bytes[li.probe_ht[p]];
    double cr = std::min(1.0, L2_eff / std::max(ht, 1.0));
    probe_bytes += reach[li.nfilt + p] * N * 32.0 * (1.0 - cr);
  }
  // Eq 4 analog: warp-instructions per 128-row warp packet (4 rows per lane)
  const double qfrac = reach.size() > (size_t)(li.nfilt + d.nsprobe) ? reach[li.nfilt + d.nsprobe] : 1.0;
  const double stage_cost = 40 + 12.0 * d.nfilt + 60.0 * d.nsprobe + 14.0 * d.npush * std::min(1.0, 8 * qfrac);
  const double queue_cost = 60 + 90.0 * (d.nprobe - d.nsprobe) + 25.0 * d.nresid + 40.0 * d.nterm + 12.0 * d.nagg;
  const double instr_iter = stage_cost + qfrac * queue_cost;  // per warp per 128 rows
  // Latency of the probes on a warp iteration's critical path, by where the
  // table lives: staged in smem, small enough for L1, L2-resident, or HBM.
  auto lat = [&](int t) {
    if (d.ht_smem_off[t] >= 0) return 40.0;
    const double bytes = li.ht_bytes.empty() ? 1e6 : (double)li.ht_bytes[t];
    // calibrated on B200 (Q5 SF 1, ncu: a stage-phase L2 probe keeps a warp
    // ~1500 cycles per packet; two dies, so half the L2 is far)
    return bytes <= 64e3 ? 80.0 : bytes <= L2_eff ? 1200.0 : 2000.0;
  };
  double lat_stage = 0, lat_queue = 0;
  for (int p = 0; p < li.nprobe; p++)  // a clustered probe reads its staged cells from shared memory
    (p < d.nsprobe ? lat_stage : lat_queue) += p == d.cl_probe ? 40.0 : lat(li.probe_ht[p]);
  // lazy columns: one HBM gather round trip per drain (per 128 queued rows)
  if (!li.lazy_reach.empty()) lat_queue += 2000.0;
  // a hash group-by sink: the group's slot load, the group count and the CAS
  // that claims a new group are dependent round trips into a global table
  if (d.agg_mode == AGG_HASH) lat_queue += 3 * 2000.0;
  // cycles per warp iteration of `npack` packets: the stage-phase probe
  // latency is paid once per iteration (all npack*4 loads of a lane in flight).
  // cons_rate(ka): fact rows per cycle per SM the consumer warps sustain with
  // ka CTAs of this shape active on the SM (fewer than k in a last, partial wave)
  const double cf = std::max(li.cons_factor, 1e-3);
  // ring refill: a released slot is refilled after the producer's load latency
  // (~1.2 us; twice that with a clustered probe whose cells come from HBM: its
  // cell range needs the stage's keys first); the other D-1 slots must cover
  // it, or every stage exposes the rest (fitted on the autotune candidates:
  // depth 2 loses 15-30% on SF 100 Q5/Q8 and nothing on Q9; SF 1 Q5, cells in
  // L2, exposes ~1.2 us per 512-row stage at depth 2)
  const double L_ring = 1.2e-6 + (d.cl_probe >= 0 && li.cl_bytes > L2_eff ? 1.2e-6 : 0.0);
  auto cons_rate = [&](double ka, Config* rep) -> double {
    double r_issue, r_lat, rl;
    if (ndrain == 0) {
      // A warp's iteration: the probe latencies and its work (scaled by the
      // profile fit), plus the stage hand-off (full-barrier wait + empty arrive,
      // ~800 cycles, not scaled) shared by the packets the warp takes from one
      // stage. A second packet per iteration overlaps less than the latency sum
      // suggests (register-limited ILP; 1.3x fitted on the SF 100 autotune
      // candidates of Q5-Q14, profiles/r2/experiments/).
      const double ppw = std::max(1.0, (double)S / (128.0 * npack * W));
      const double crit = 150.0 + lat_stage + npack * (qfrac * lat_queue + instr_iter);
      const double w_eff = (double)std::min(W, S / (128 * npack)) * ka;  // warps with work per stage
      const double num = w_eff * 128.0 * npack / (npack == 2 ? 1.3 : 1.0);
      // issue cap: 4 schedulers at 70% issue efficiency (ncu: the best Q5 / Q9
      // shapes sustain 57-61% of the SM's issue slots while not purely
      // issue-bound; the soft combination below keeps a shape at the cap under it)
      r_issue = 4.0 * 0.7 * 128.0 / instr_iter;
      r_lat = num / (crit + 800.0 / ppw);
      rl = num / (crit * cf + 800.0 / ppw);
    } else {
      // operator-specialised warps (NEXT-1): stage warps never block on the
      // queue phase; drain warps absorb qfrac of the rows at one 128-row packet
      // per (queue latency + queue work + hand-off). The consumers sustain the
      // slower of the two groups; Eq 8's delay between them is what the ring and
      // the hand-off slots must absorb (min() below: the faster group idles).
      const int Wsg = W - ndrain;
      const double ppw = std::max(1.0, (double)S / (128.0 * npack * Wsg));
      const double crit_s = 150.0 + lat_stage + npack * stage_cost;
      const double w_eff = (double)std::min(Wsg, S / (128 * npack)) * ka;
      const double num = w_eff * 128.0 * npack / (npack == 2 ? 1.3 : 1.0);
      const double crit_d = lat_queue + queue_cost + 60.0;
      auto drain = [&](double f) {
        return qfrac > 0 ? (double)ndrain * ka * 128.0 / (crit_d * f + 800.0) / qfrac : 1e30;
      };
      r_issue = 4.0 * 0.7 * 128.0 / instr_iter;
      r_lat = std::min(num / (crit_s + 800.0 / ppw), drain(1.0));
      rl = std::min(num / (crit_s * cf + 800.0 / ppw), drain(cf));
    }
    if (rep) {
      rep->r_issue = r_issue;
      rep->r_lat = r_lat;
    }
    // the profile fit scales the latency terms only (the instruction count is
    // the kernel's own); the two bounds combine softly (p = 2), so more latency
    // hiding still helps near the issue cap
    double rows = 1.0 / std::sqrt(1.0 / (r_issue * r_issue) + 1.0 / (rl * rl));
    const double t_st = (double)S * ka / (rows * f_sm);  // one stage's consumption
    const double expo = std::max(0.0, L_ring - (depth - 1) * t_st);
    return rows * t_st / (t_st + expo);
  };

  // Eq 3 analog: waves of Δ-row tiles over G persistent CTAs, with the last wave's tail
  const int64_t tiles = (N + tile - 1) / tile;
  const int64_t G = c.grid;
  const int64_t waves = (tiles + G - 1) / G;
  const int64_t last = tiles - (waves - 1) * G;
  // CTAs with work per SM in the full waves and in the last one
  auto ka_of = [&](int64_t active) {
    return std::min<double>(k, std::max<double>(1.0, (double)((active + ctx->sms - 1) / ctx->sms)));
  };
  const int64_t act_full = std::min<int64_t>(G, tiles);
  const double kf = ka_of(act_full), kl = ka_of(last);
  const double rows_cyc = cons_rate(kf, &c), rows_last = cons_rate(kl, nullptr);
  const double R_cons = rows_cyc * f_sm * b;  // bytes/s one SM's consumers absorb
  // per-CTA rates (bytes/s): the SM's fill cap and consumers shared by its active
  // CTAs, the device stream shared by every active CTA
  const double rate_full = std::min(std::min(B_sm, R_cons) / kf, G_ring / (double)act_full);
  const double rate_last = std::min(std::min(B_sm, rows_last * f_sm * b) / kl, G_ring / (double)last);
  const double last_rows = (double)(N - (tiles - 1) * tile);
  const double t_cons = (waves - 1) * (double)tile / (rows_cyc * f_sm / kf) +
                        (last == 1 ? last_rows : (double)tile) / (rows_last * f_sm / kl);
  const double t_tile = tile * b / rate_full;
  const double t_last = (last == 1 ? last_rows : (double)tile) * b / rate_last;
  const double t_stage = S * b / rate_full;
  const double t_claim = std::max(0.0, 1.5e-6 - (depth - 1) * t_stage);  // producer's claim latency not hidden by the ring
  double t_prod = (waves - 1) * (t_tile + t_claim) + t_last + probe_bytes / B;
  // Eq 6 analog (ring handoff, ~mbarrier round trip per stage per CTA)
  const double stages_per_cta = (double)N / S / std::min<int64_t>(G, tiles);
  const double t_chan = stages_per_cta * 0.3e-6 / depth;
  // Convoy (no drain warps): a warp draining 128 queued rows consumes none of
  // its packets meanwhile; the ring's other depth - 1 stages cover up to
  // (depth - 1) stage times of that, the rest stalls the CTA behind the slot
  // the warp has not released (measured, SF 100 Q3: D = 2 drain warps 1.60 ms
  // vs the best D = 0 shape 1.97 ms). Drains spread over the CTAs.
  double t_convoy = 0;
  if (ndrain == 0 && d.npush > 0 && qfrac > 0) {
    const double t_drain = (lat_queue + queue_cost) * cf / f_sm;
    const double drains_per_cta = (double)N * qfrac / 128.0 / (double)std::min<int64_t>(G, tiles);
    t_convoy = drains_per_cta * std::max(0.0, t_drain - (depth - 1) * t_stage);
  }
  // Eq 8/9 analog
  const double tp = t_prod + t_chan, tc = t_cons + t_convoy;
  const double T = 0.5 * (tp + tc) + 0.5 * std::fabs(tp - tc);
  c.t_launch_ms = t0_cal >= 0 ? t0_cal : 4e-3 + 1e3 * (depth * t_stage);  // launch + prologue + ring fill
  c.t_stream_ms = 1e3 * (N * b / B);
  c.t_probe_ms = 1e3 * probe_bytes / B;
  c.t_tail_ms = 1e3 * (T - N * b / B - probe_bytes / B);
  c.pred_ms = c.t_launch_ms + 1e3 * T;
  c.t_cons_ms = 1e3 * tc;
  c.t_prod_ms = 1e3 * tp;
  return c;
}

bool choose_config(const gpl_ctx* ctx, const PipeDesc& d, const LowerInfo& li, int64_t N, int64_t tile_req,
                   Config* out, std::string* err, std::vector<Config>* shortlist) {
  std::map<std::tuple<int, int, int>, Config> per_shape;  // best predicted per (CTAs/SM, stage rows, packets)
  const Options& o = ctx->opt;
  std::vector<int> Ss = o.stage_rows > 0 ? std::vector<int>{(int)o.stage_rows} : std::vector<int>{512, 1024, 2048, 4096, 8192};
  std::vector<int> Ds = o.ring_depth > 0 ? std::vector<int>{(int)o.ring_depth} : std::vector<int>{2, 3, 4, 6};
  std::vector<int> Ws = o.consumer_warps > 0 ? std::vector<int>{(int)o.consumer_warps} : std::vector<int>{4, 8, 12, 16};
  std::vector<int> Ks = o.ctas_per_sm > 0 ? std::vector<int>{(int)o.ctas_per_sm} : std::vector<int>{1, 2};
  std::vector<int> Ps = o.packets > 0 ? std::vector<int>{(int)o.packets} : std::vector<int>{1, 2};
  // drain warps only for a segment with a queue phase (not a stage-phase insert)
  // (a dense build's cells are written by the warp that zero-filled their packet: no drain warps)
  const bool can_drain = d.npush > 0 && !(d.sink != SINK_AGG && d.ins_kcol >= 0 && !d.ins_q) && !d.ins_dense;
  std::vector<int> Dr = !can_drain ? std::vector<int>{0}
                        : o.drain_warps >= 0 ? std::vector<int>{(int)o.drain_warps} : std::vector<int>{0, 1, 2};
  Config best;
  bool found = false;
  for (int S : Ss) {
    if (S % 128 || S < 128 || S > 8192) { *err = "stage_rows must be a multiple of 128 in [128, 8192]"; return false; }
    std::vector<int64_t> tiles;
    if (tile_req > 0) {
      tiles.push_back((tile_req + S - 1) / S * S);
    } else {
      for (int64_t t = S; ; t *= 2) {
        tiles.push_back(t);
        if (t >= N) break;
      }
    }
    for (int k : Ks)
    for (int np : Ps)
    for (int D : Ds)
      for (int W : Ws)
        for (int nd : Dr)
        for (int64_t t : tiles) {
          if (d.flush_each_tile && (long double)(t + QCAP) * std::max<long double>(li.maxabs, 1) >= 4.6e18L) continue;
          Config c = predict(ctx, d, li, N, t, S, D, W, k, np, nd);
          if (!c.feasible) continue;
          {
            auto key = std::make_tuple(k, S, np);
            auto it = per_shape.find(key);
            if (it == per_shape.end() || c.pred_ms < it->second.pred_ms) per_shape[key] = c;
          }
          if (!found || c.pred_ms < best.pred_ms * (1 - 1e-9) ||
              (std::fabs(c.pred_ms - best.pred_ms) <= best.pred_ms * 1e-9 && c.tile_rows > best.tile_rows)) {
            best = c;
            found = true;
          }
        }
  }
  if (!found) {
    *err = "no feasible pipeline configuration (shared memory / options)";
    return false;
  }
  *out = best;
  if (shortlist) {
    shortlist->clear();
    for (auto& kv : per_shape) shortlist->push_back(kv.second);
    std::sort(shortlist->begin(), shortlist->end(), [](const Config& a, const Config& b) { return a.pred_ms < b.pred_ms; });
  }
  return true;
}

void apply_profile(const gpl_ctx* ctx, const PipeDesc& d, LowerInfo* li, const std::string& plan_text) {
  li->cons_factor = 1;
  li->bw_factor = 1;
  auto it = ctx->profile.find(plan_text);
  if (it == ctx->profile.end() || !ctx->opt.use_profile) return;
  const RunProfile& p = it->second;
  auto ti = ctx->tables.find(li->table.empty() ? std::string() : li->table);
  if (ti != ctx->tables.end() && ti->second.version != p.table_version) return;  // profiled on other data
  if (p.runs < 2) return;
  auto pred = [&](double f) {
    li->cons_factor = f;
    return predict(ctx, d, *li, std::max<int64_t>(p.nrows, 1), p.tile_rows, p.stage_rows, p.depth, p.warps,
                   p.ctas_per_sm, p.npack, p.ndrain).pred_ms;
  };
  // the prediction is non-decreasing in the factor: geometric bisection. The
  // factor is not taken below 0.3: a profiled run at the producer's bound only
  // says the consumers kept up, and scaling their latency terms towards zero
  // makes shapes with a few warps look as fast as many (measured, SF 100 Q9:
  // a fitted 0.086 picked 4 consumer warps, 0.74 ms, over 12, 0.66 ms)
  const double lo = 0.3, hi = 50;
  auto bisect = [](double a, double b, auto&& below) {  // below(x): the prediction at x is under the target
    for (int i = 0; i < 40; i++) {
      const double mid = std::sqrt(a * b);
      (below(mid) ? a : b) = mid;
    }
    return std::sqrt(a * b);
  };
  const char* path = "consumer";
  if (pred(hi) <= p.kernel_ms) {
    li->cons_factor = hi;
  } else if (pred(lo) < p.kernel_ms) {
    // the usual case: the consumers' latency-bound rate sets the time
    li->cons_factor = bisect(lo, hi, [&](double f) { return pred(f) < p.kernel_ms; });
  } else {
    // at or under the model's stream bound (an L2-resident input, or a stream
    // model too slow for this plan): fit the streaming rate to the run, then
    // make the consumers just fast enough — their own time equals the measured
    // time — instead of arbitrarily fast (which would make shapes whose
    // consumers are the bound, e.g. few CTAs on a large tile, look free)
    path = "stream";
    li->cons_factor = lo;
    auto predb = [&](double f) {
      li->bw_factor = f;
      return pred(lo);
    };
    li->bw_factor = predb(32) >= p.kernel_ms ? 32 : bisect(1, 32, [&](double f) { return predb(f) > p.kernel_ms; });
    auto cons_only = [&](double f) {
      li->cons_factor = f;
      const Config c = predict(ctx, d, *li, std::max<int64_t>(p.nrows, 1), p.tile_rows, p.stage_rows, p.depth, p.warps,
                               p.ctas_per_sm, p.npack, p.ndrain);
      return c.t_cons_ms + c.t_launch_ms;
    };
    li->cons_factor = cons_only(lo) >= p.kernel_ms ? lo
                      : cons_only(hi) <= p.kernel_ms ? hi
                      : bisect(lo, hi, [&](double f) { return cons_only(f) < p.kernel_ms; });
  }
  if (std::getenv("GPL_DEBUG_MODEL")) {
    const Config c = predict(ctx, d, *li, std::max<int64_t>(p.nrows, 1), p.tile_rows, p.stage_rows, p.depth, p.warps,
                             p.ctas_per_sm, p.npack, p.ndrain);
    std::fprintf(stderr,
                 "apply_profile: measured %.4f ms at S %d D %d W %d k %d np %d tile %lld N %lld -> %s cons %.3f bw %.3f "
                 "pred %.4f (prod %.4f cons %.4f stream %.4f probe %.4f launch %.4f)\n",
                 p.kernel_ms, p.stage_rows, p.depth, p.warps, p.ctas_per_sm, p.npack, (long long)p.tile_rows,
                 (long long)p.nrows, path, li->cons_factor, li->bw_factor, c.pred_ms, c.t_prod_ms, c.t_cons_ms,
                 c.t_stream_ms, c.t_probe_ms, c.t_launch_ms);
  }
}

int choose_split(const gpl_ctx* ctx, const Segment& s) {
  if (s.split_hint >= -1) return s.split_hint < 0 ? (int)s.probes.size() : s.split_hint;
  if (ctx->opt.probe_split >= -1) return ctx->opt.probe_split < 0 ? (int)s.probes.size() : (int)ctx->opt.probe_split;
  const int np = (int)s.probes.size(), nf = (int)s.filters.size();
  auto it = ctx->lambda.find(s.text);
  // Stage-phase probes read their keys straight from the staged tile with all
  // RPL loads of a lane in flight; queue-phase probes first pay the survivor
  // queue's smem writes and reads. Measured on B200 (SF 20, Q5/Q7/Q8 with the
  // clustered HT_O probe first): running every probe (up to MAXSP) in the stage
  // phase is fastest even at 3-30% survival, so the queue is entered before a
  // probe only when the filters alone already drop >= 95% of the rows (Q14).
  // gpl_autotune measures every split and pins the best.
  if (it != ctx->lambda.end() && (int)it->second.size() >= nf + np) {
    const std::vector<double>& lam = it->second;
    const double after_filters = nf ? lam[nf - 1] : 1.0;
    if (after_filters <= 0.05) return 0;
    return std::min(np, MAXSP);
  }
  return nf ? 0 : std::min(np, MAXSP);
}

std::vector<double> build_lambda_estimate(const gpl_ctx* ctx, const Segment& s) {
  std::vector<double> lam;
  double frac = 1.0;
  auto ti = ctx->tables.find(s.table);
  for (const FilterIR& F : s.filters) {
    double sel = 0.3;
    const Column* c = ti != ctx->tables.end() ? ti->second.find(F.col) : nullptr;
    if (c && c->vmax >= c->vmin) {
      const long double dom = (long double)c->vmax - (long double)c->vmin + 1;
      if (F.kind == F_RANGE) {
        const long double lo = std::max<long double>(F.lo, c->vmin), hi = std::min<long double>(F.hi, c->vmax);
        sel = hi >= lo ? (double)((hi - lo + 1) / dom) : 0.0;
      } else if (F.kind == F_MASK) {
        int in = 0;
        for (int b = 0; b < 64; b++)
          if (((F.mask >> b) & 1ull) && b >= c->vmin && b <= c->vmax) in++;
        sel = std::min(1.0, (double)(in / dom));
      } else {
        sel = 1.0 - (double)(1 / dom);
      }
    }
    frac *= sel;
    lam.push_back(frac);
  }
  for (size_t p = 0; p < s.probes.size(); p++) {
    if (s.probes[p].kind != P_MARK) frac *= 0.3;
    lam.push_back(frac);
  }
  for (size_t r = 0; r < s.wheres.size(); r++) {
    frac *= 0.3;
    lam.push_back(frac);
  }
  return lam;
}

int choose_build_split(const gpl_ctx* ctx, const Segment& s) {
  const int np = (int)s.probes.size(), nf = (int)s.filters.size();
  if (np == 0 || nf == 0) return std::min(np, MAXSP);
  auto it = ctx->lambda.find(s.text);
  const std::vector<double> lam = it != ctx->lambda.end() ? it->second : build_lambda_estimate(ctx, s);
  return (int)lam.size() >= nf && lam[nf - 1] <= 0.05 ? 0 : std::min(np, MAXSP);
}

}  // namespace gpl
