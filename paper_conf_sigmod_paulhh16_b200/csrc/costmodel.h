// costmodel.h — A9: tile-size / pipeline-shape selection, the B200
// re-derivation of the paper's analytical model (§4, Eqs 1-9,
// P:205-315) — see costmodel.cpp for the term-by-term mapping.
#pragma once
#include <string>
#include <vector>

#include "ctx.h"

namespace gpl {

struct Config {
  int64_t tile_rows = 0;
  int stage_rows = 0, depth = 0, warps = 0, ctas_per_sm = 1, grid = 0, smem = 0;
  int npack = 1;  // 128-row packets a consumer warp takes per iteration (1 or 2)
  int ndrain = 0; // of the consumer warps, those that only drain hand-off packets (NEXT-1)
  double pred_ms = 0, t_stream_ms = 0, t_probe_ms = 0, t_tail_ms = 0, t_launch_ms = 0, bw_gbs = 0;
  double t_cons_ms = 0;  // the consumer warps' time alone (Eq 4 analog, all waves)
  double t_prod_ms = 0;  // the producer's time alone (Eq 5/6 analog: stream, probe misses, ring)
  double r_issue = 0, r_lat = 0;  // consumer rows/cycle/SM at the issue cap and the latency bound (unscaled)
  bool feasible = false;
};

// Shared-memory bytes of a configuration (Eq 2 feasibility input).
int smem_bytes(const PipeDesc& d, const LowerInfo& li, int stage_rows, int depth, int warps, int ndrain = 0);

// Predicted time (ms) of one configuration (Eqs 3-9 analog).
Config predict(const gpl_ctx* ctx, const PipeDesc& d, const LowerInfo& li, int64_t nrows, int64_t tile_rows,
               int stage_rows, int depth, int warps, int ctas_per_sm, int npack = 1, int ndrain = 0);

// Search the feasible space (Δ, stage rows, depth, consumer warps), honouring
// options and a requested tile_rows (> 0 fixes Δ). Returns false if nothing fits.
// shortlist (optional): the best predicted configuration for every
// (CTAs per SM, stage rows) shape, best first — the candidates gpl_autotune measures.
bool choose_config(const gpl_ctx* ctx, const PipeDesc& d, const LowerInfo& li, int64_t nrows, int64_t tile_req,
                   Config* out, std::string* err, std::vector<Config>* shortlist = nullptr);

// Fill the schedule and shared-memory layout fields of d from c.
void apply_config(PipeDesc* d, const LowerInfo& li, const Config& c);

// Table 2 "profiling input": fit li->cons_factor, the scale of
// the consumer warps' per-iteration cost, so that the model reproduces the
// plan's profiled run (shape, rows, measured kernel time); 1 without one.
void apply_profile(const gpl_ctx* ctx, const PipeDesc& d, LowerInfo* li, const std::string& plan_text);

// Probes run before the survivor queue, from the previous run's pass
// fractions (the paper profiles the first tile) or a heuristic.
int choose_split(const gpl_ctx* ctx, const Segment& s);

// A build segment's pass fractions before its first run: each filter's
// selectivity from its column's [min, max] under the uniformity assumption
// (the textbook optimizer estimate; the paper takes a plan's statistics as
// given), a probe's hit fraction 0.3. Cumulative, one per operator.
std::vector<double> build_lambda_estimate(const gpl_ctx* ctx, const Segment& s);

// A build's probe split: the probes move to the queue phase (the insert then
// runs in the drain) when the filters keep at most 5% of the rows, else every
// probe runs in the stage phase (measured on B200, SF 100: with the model's
// shapes the queue split loses at 15-30% survival, Q5 0.51 vs 0.55 ms, Q8 0.59
// vs 0.69; gpl_autotune measures both splits).
int choose_build_split(const gpl_ctx* ctx, const Segment& s);

}  // namespace gpl
