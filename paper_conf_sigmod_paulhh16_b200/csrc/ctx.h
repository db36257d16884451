// ctx.h — the opaque gpl_ctx: column store (A0), hash tables (A1), run state.
#pragma once
#include <cuda_runtime.h>

#include <cstdint>
#include <map>
#include <memory>
#include <string>
#include <tuple>
#include <vector>

#include "common.h"
#include "gpl.h"
#include "plan.h"

namespace gpl {

struct Column {
  std::string name;
  int type = 0, scale = 0, width = 4;
  char* dev = nullptr;   // device base (owned or borrowed)
  bool owned = false;
  int64_t cap_rows = 0;
  int64_t vmin = 0, vmax = 0;
  bool sorted = false;     // non-decreasing (e.g. lineitem.l_orderkey): enables clustered probe staging
  bool strict = false;     // strictly increasing (a primary key in key order, e.g. orders.o_orderkey): dense builds
  std::vector<char> host;  // host-only context storage
};

struct Table {
  std::string name;
  int64_t nrows = 0;
  uint64_t version = 0;
  std::vector<Column> cols;
  // a partitioned table (the output of a partition segment, NEXT-4): nrows is its
  // capacity, the live row count is written on the device; columns of src_table are
  // reachable through the row-id column
  bool derived = false;
  std::string src_table, rowid_col = "rowid";
  const unsigned* nrows_dev = nullptr;
  const Column* find(const std::string& n) const {
    for (auto& c : cols)
      if (c.name == n) return &c;
    return nullptr;
  }
};

struct HashTable {
  std::string name;
  int32_t id = -1;
  int kind = HT_SET32, hash = H_MULT, key_arity = 1;
  bool has_payload = false;
  int64_t pay_min = 1, pay_max = 1;  // payload value range (validator)
  void* slots = nullptr;
  size_t alloc_bytes = 0;
  HTHeader* hdr = nullptr;
  int64_t cap_slots = 0;
  // DIRECT tables (kind == HT_DIRECT)
  int width = 0;
  long long dkmin = 0, pay_base = 0;
  unsigned long long dnslots = 0;
  // partition segment output buffers (kind == HT_PART): counts, offsets, row count, key + row id columns
  void* part_buf = nullptr;
  size_t part_alloc = 0;
  // MULTI (fan-out): payload array and scan/scatter scratch
  void* pay = nullptr;
  size_t pay_alloc = 0;
  void* aux = nullptr;
  size_t aux_alloc = 0;
  size_t bytes() const {
    if (kind == HT_MULTI) return (dnslots + 1) * 4;
    if (kind == HT_DIRECT)
      return width == 0 ? (dnslots + 31) / 32 * 4 : width == W_NIBBLE ? (dnslots + 7) / 8 * 4 : (dnslots * width + 3) / 4 * 4;
    return (size_t)cap_slots * (kind == HT_SET32 ? 4 : kind == HT_MAP32 ? 8 : 16);
  }
  HTRef ref() const { return HTRef{slots, hdr, kind, hash, dkmin, dnslots, pay_base, width, 0, pay}; }
  std::string src_table;
  uint64_t src_version = 0;
  bool valid = false;
};

// Host-side facts produced by lowering a probe segment.
struct LowerInfo {
  int ngroups_total = 1, nagg = 1, nops = 0, ngroup_dims = 0;
  int glo[MAXG] = {0, 0, 0}, gsize[MAXG] = {1, 1, 1}, gstride[MAXG] = {1, 1, 1};
  int bytes_per_row = 0;        // TMA-staged (eager) column bytes per row
  int bytes_per_row_all = 0;    // every column the segment reads
  std::vector<int> lazy_w;      // width of each lazy column
  std::vector<int> lazy_reach;  // op whose pass count = rows reaching the column (-1: all rows)
  double cl_bytes = 0;          // clustered probe: cell bytes of the table the producer stages with the columns
  long double maxabs = 0;  // bound on |value| per row
  std::vector<std::string> op_names;
  std::vector<int64_t> ht_bytes;  // slot bytes of each probed table
  std::vector<int> probe_ht;      // probe index -> d.ht index
  std::vector<int> ht_ids;        // d.ht index -> ctx hash-table id
  std::string table;              // scanned (fact) table
  int nprobe = 0, nfilt = 0;
  bool has_groups = false;
  std::vector<double> lambda;     // cumulative pass fraction after each op (previous run)
  double cons_factor = 1;         // consumer cost scale fitted to the plan's profiled run (costmodel apply_profile)
  // hash group-by (NEXT-4): the result step's ORDER BY / LIMIT
  bool hash_group = false;
  int limit = 0, norder = 0;
  int ord_is_agg[3] = {0, 0, 0}, ord_idx[3] = {0, 0, 0}, ord_desc[3] = {0, 0, 0};
  std::vector<DecodeIR> decodes;  // A10: group key decodes through loaded tables
  std::vector<RatioIR> ratios;    // A10: derived ratio columns
  double bw_factor = 1;           // streaming-rate scale, fitted only when the run beat the model's stream bound (L2-resident input)
};

// The first timed run of a plan after its λ profile (the paper profiles the
// first tile): its shape, rows and measured kernel time.
struct RunProfile {
  uint64_t table_version = 0;  // the fact table's version when profiled (a reload re-profiles)
  int runs = 0;                // timed runs folded in (the profile is used from 2 on)
  int64_t nrows = 0, tile_rows = 0;
  int stage_rows = 0, depth = 0, warps = 0, ctas_per_sm = 1, npack = 1, ndrain = 0;
  double kernel_ms = 0;
};

struct PreparedRun;

// The last run: a shared reference to its prepared plan (no per-run copies)
struct LastRun {
  bool valid = false;
  std::shared_ptr<const PreparedRun> run;
  gpl_stats stats{};
  bool timed = false;
  bool kbe = false;
  bool copied_out = false;  // the run's results were copied to h_stage by the copy-out kernel
  bool overflowed = false;  // hash group-by: the run's aggregation table overflowed (rows incomplete)
};

struct PreparedRun {
  PipeDesc desc{};
  LowerInfo li;
  int grid = 0;
  double pred_ms = 0;
  const void* fn = nullptr;  // kernel to launch (JIT or generic)
  bool jit = false;
  uint64_t table_version = 0, opt_version = 0;
  size_t lambda_n = 0;
  bool profiled = false;  // planned with the plan's RunProfile
  // hash group-by (NEXT-4): the aggregation table's size and the result step
  uint64_t hagg_cap = 0;
  size_t hagg_clear = 0;  // bytes zeroed per run (keys + accumulators)
  HaggResultDesc hres{};
  std::string text;
};

struct PreparedBuild {
  BuildDesc desc{};
  HashTable shape;
  bool trivial = false;
  HTHeader known{};
  int ht_index = -1;
  HTRef dest_ref{};
  std::string name, table;
  uint64_t table_version = 0, opt_version = 0;
  std::vector<int> src_ids;
  // DIRECT builds run through the fused pipeline with an insert sink
  bool pipe = false;
  PipeDesc pdesc{};
  const void* pfn = nullptr;
  int pgrid = 0;
  size_t clear_bytes = 0;  // table cells + the trailing tile counter
  size_t clear_off = 0;    // dense builds: only the tile counter (the build writes every cell)
  // partition segment (NEXT-4 partitioned hash join): count pass, scan, scatter pass
  bool part = false;
  PipeDesc pdesc2{};        // the scatter pass (pdesc: the count pass)
  const void* pfn2 = nullptr;
  unsigned* part_hist = nullptr;  // [nparts][grid] counts
  unsigned* part_offs = nullptr;  // ... their exclusive scan
  unsigned* part_total = nullptr;
  void* scan_tmp = nullptr;
  size_t scan_bytes = 0;
  size_t part_n = 0;
};

// A0 load whose per-column min/max/sortedness are still in flight (a load
// enqueues its copies + one min/max pass and returns without synchronising;
// the first call that plans or validates reads them back: one synchronise per
// batch of loads instead of one per table)
struct PendingLoad {
  std::string table;
  int slot0 = 0, ncols = 0;   // column slots in ctx->d_minmax / h_minmax
  bool has_old = false;       // the table replaced an earlier version of itself
  Table old_meta;             // that version's shape (no data): keeps its version when the shape is unchanged
};

// gpl_autotune's pinned pipeline shape for one probe segment
struct TunedShape {
  int64_t tile_rows = 0;
  int stage_rows = 0, depth = 0, warps = 0, ctas_per_sm = 1;
  int split = -2;  // probes run in the stage phase (-2: the heuristic's)
  int npack = 1;
  int ndrain = 0;
};

struct Options {
  int64_t stage_rows = -1, ring_depth = -1, consumer_warps = -1, ctas_per_sm = -1, probe_split = -2,
          hash_load_pct = -1, packets = -1;
  int64_t jit = 1;
  int64_t lazy_columns = -1;   // late materialisation: -1 auto (from λ), 0 off, 1 every eligible column
  int64_t build_pipeline = 1;
  int64_t clustered = 1;       // stage the cell range of a probe keyed by a sorted column (0: probe L2/HBM)
  int64_t autotune_probe = 1;  // gpl_autotune: 1 = builds and the probe segment; 0 = the build segments only
  int64_t kbe_graph = 1;       // GPL (w/o CE): the tile loop replayed as one captured CUDA graph (0: launched)
  int64_t kbe_tile_rows = 0;   // gpl_run_plan_kbe: > 0 = GPL (w/o CE), the KBE sequence tile by tile  // DIRECT builds through the fused pipeline (0: build kernels)
  double hbm_gbs = -1;
  int64_t use_gamma = 1;       // the model uses the channel calibration Γ when one is loaded
  int64_t use_profile = 1;     // the model fits its consumer cost to the plan's profiled run
  int64_t hash_slots_log2 = 0; // hash group-by table size (tests): 0 = from the last run's distinct groups
  int64_t graph_branches = 1;  // whole-query graph: independent build segments on two capture lanes
  int64_t drain_warps = -1;    // operator-specialised drain warps (NEXT-1): -1 = the model's choice
  int64_t dense_build = 1;     // sorted-key DIRECT builds write their cell ranges densely (no clear, no atomics)
  // DIRECT payloads of <= 15 values in 4-bit cells (1) or byte cells (0, default). Measured on B200,
  // SF 100, autotuned shapes: Q7 step 2.15 -> 2.00 ms (kernel 1.32 -> 1.20), Q9 1.085 -> 1.073, but
  // Q5 1.32 -> 1.39 and Q8 1.71 -> 1.73: the nibble extraction in the clustered probe and the dense
  // build's byte assembly cost more issue slots than the halved cell bytes save there.
  int64_t nibble_cells = 0;
  int64_t reg_fields = 1;      // JIT kernels keep drain-produced queue fields in registers
  int64_t zone_restrict = 1;   // scan only the row range of range filters on sorted columns
  int64_t agg_mode = -1;       // dense group accumulators: -1 exactness-driven choice, 2 = force global int128 atomics
};

// Γ of one ring shape (gpl_calibrate, Eq 1): (bytes, GB/s)
// points sorted by bytes, and the shape's empty-input kernel time.
struct GammaCurve {
  int depth = 0, stage_rows = 0, ctas_per_sm = 0;
  double t0_ms = 0;
  std::vector<std::pair<double, double>> pts;
};

}  // namespace gpl

struct gpl_ctx {
  int device = -1;
  bool host_only = true;
  cudaStream_t stream = nullptr;
  bool own_stream = false;
  int sms = 148, smem_optin = 232448, l2_bytes = 126 * 1024 * 1024;
  double hbm_gbs = 6556.5;  // measured copy BW of this pool's B200s; gpl_set_option("hbm_gbs")
  std::map<std::string, gpl::Table> tables;
  uint64_t next_version = 1;
  std::vector<gpl::HashTable> hts;
  std::map<std::string, int> ht_by_name;
  std::string err;
  // device scratch: [0] tile counter, [1..MAXOPS] op_pass, [MAXOPS+1] error bits
  unsigned long long* d_scratch = nullptr;
  unsigned long long* d_partials = nullptr;
  size_t partials_cap = 0;
  long long* d_bounds = nullptr;  // zone restriction: binary-search result (2 rows)
  long long* d_minmax = nullptr;  // [kMinmaxSlots][3] column slots of pending loads
  size_t minmax_cap = 0;
  std::vector<gpl::PendingLoad> pending;  // loads whose min/max are not read back yet
  int mm_next = 0;                        // next free column slot
  cudaEvent_t mm_ev = nullptr;            // recorded after the last pending load's min/max D2H
  cudaStream_t mm_stream = nullptr;       // the min/max passes (overlap the next columns' copies)
  cudaEvent_t mm_col_ev[64] = {};         // "column i landed" (ctx stream -> mm_stream)
  cudaEvent_t ev0 = nullptr, ev1 = nullptr;
  // whole-query graphs: a second capture lane for build segments that do not
  // depend on each other (fork/join events, created on first use)
  cudaStream_t side = nullptr;
  cudaEvent_t fork_ev[8] = {};
  gpl::LastRun last;
  gpl::Options opt;
  uint64_t opt_version = 1;  // bumped by gpl_set_option (invalidates prepared plans)
  std::map<std::string, std::vector<double>> lambda;  // plan text -> per-op pass fraction (A9 "profile the first tile")
  std::map<std::string, gpl::RunProfile> profile;     // plan text -> first timed run after λ (consumer cost fit)
  // prepared-plan caches (keyed by segment text [+ tile_rows]); validated on
  // every use against table versions, hash-table refs and options
  std::map<std::string, std::shared_ptr<gpl::PreparedRun>> run_cache;
  std::map<std::string, gpl::PreparedBuild> build_cache;
  // gpl_run_query: whole-query CUDA graphs (builds + fused run), keyed by plan text + tile_rows
  std::map<std::string, cudaGraphExec_t> graphs;
  std::map<std::string, int> graph_kernels;  // kernel nodes of each recorded query graph
  std::map<std::tuple<int, int, int>, gpl::GammaCurve> gamma;  // (depth, stage rows, CTAs/SM) -> Γ(d)
  std::map<std::string, gpl::TunedShape> tuned;  // probe segment text -> measured-best shape
  std::map<std::string, std::vector<std::string>> plan_segs;  // gpl_run_query: plan text -> segments
  void* h_stage = nullptr;  // pinned host staging for one packed D2H of results
  unsigned int* h_err = nullptr;  // pinned word for error-bit reads (gpl_sync)
  long long* h_minmax = nullptr;  // pinned column min/max of pending loads ([kMinmaxSlots][3])
  unsigned long long* h_stage_dev = nullptr;  // device alias of h_stage (the fused kernel's result copy-out)
  size_t h_stage_cap = 0;
  // hash group-by (NEXT-4): aggregation table, result rows, selection scratch;
  // distinct groups of each plan's last run size the next table
  void* d_hagg = nullptr;
  size_t hagg_alloc = 0;
  unsigned long long* d_hres = nullptr;
  size_t hres_alloc = 0;
  unsigned long long* d_hcand = nullptr;
  size_t hcand_alloc = 0;
  void* d_sort = nullptr;  // full device sort (ORDER BY without LIMIT): scratch + sorted rows
  size_t sort_alloc = 0;
  std::map<std::string, std::pair<uint64_t, int64_t>> hagg_groups;  // plan text -> (distinct groups, fact rows) of its last run
  // A10 key decodes: table name -> (table version, key -> output value)
  std::map<std::string, std::pair<uint64_t, std::map<int32_t, int32_t>>> decode_maps;
  unsigned long long* d_kbe_bytes = nullptr;  // GPL (w/o CE): materialised bytes counted on the device
  // KBE scratch (gpl_run_plan_kbe)
  void* kbe_buf = nullptr;
  size_t kbe_cap = 0;
  // GPL (w/o CE): the tile loop captured once per (plan, tile rows) and replayed while the lowered
  // descriptor (pointers, sizes, shape), the scratch pool and the options are unchanged
  struct KbeGraph {
    cudaGraphExec_t exec = nullptr;
    std::vector<char> desc;
    void* buf = nullptr;
    size_t cap = 0;
    uint64_t opt_version = 0;
    double inter = 0;
  };
  std::map<std::string, KbeGraph> kbe_graphs;
};
