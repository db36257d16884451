// plan.h — plan-segment IR and parser (host).
//
// A query is a sequence of segments, each ending at a blocking kernel
// (§3.1, segmentation after [23]); here:
//   build segments: scan -> filter* -> probe* -> insert   (ends at hash build)
//   probe segment : scan -> filter* -> probe* -> where* -> group-by aggregate
// Grammar (one statement per line, '#' comments): DESIGN.md §4.
#pragma once
#include <cstdint>
#include <string>
#include <vector>

namespace gpl {

struct RefIR {
  enum Kind { COL, SLOT, YEARCOL, CONST } kind = CONST;
  std::string name;  // column or slot name
  int64_t c = 0;
};

struct FilterIR {
  std::string col;
  int kind = 0;  // F_RANGE / F_MASK / F_NE
  int64_t lo = INT64_MIN, hi = INT64_MAX;
  uint64_t mask = 0;
};

struct ProbeIR {
  std::string ht;
  int kind = 0;                   // P_INNER / P_SEMI / P_MARK
  std::vector<std::string> keys;  // 1 or 2 columns
  std::string out;                // slot name ("" none)
};

struct WhereIR {
  int kind = 0;  // R_EQ / R_PAIRS / R_RANGE / R_MASK
  std::string a, b;
  std::vector<std::pair<int64_t, int64_t>> pairs;
  int64_t lo = INT64_MIN, hi = INT64_MAX;
  uint64_t mask = 0;
};

struct GroupIR {
  RefIR ref;
  int64_t lo = 0, hi = 0;  // domain [lo, hi) (dense group-by)
};

// ORDER BY component of a hash group-by result
struct OrderIR {
  bool is_agg = true;  // agg index (0 = COUNT) or group-key index
  int idx = 0;
  bool desc = false;
};

// A10 finalize (gpl_fetch_result): map a group key's values through a loaded
// table, e.g. nation key -> n_name code ('decode key 0 nation n_nationkey -> n_name')
struct DecodeIR {
  int key = 0;
  std::string table, keycol, outcol;
};

// A10 derived column: scale * agg[num] / agg[den] as a double (Q8 mkt_share,
// Q14 promo_revenue); den = 0 -> NaN (SQL NULL)
struct RatioIR {
  double scale = 1.0;
  int num = 0, den = 0;
};

struct FactorIR {
  RefIR x;   // CONST => constant a
  int64_t a = 0;
  int b = 1;
};
struct TermIR {
  int sign = 1;
  std::vector<FactorIR> f;
};

struct AggIR {
  int kind = 0;  // A_COUNT / A_SUM / A_SUMIF / A_SUMIFEQ
  std::string slot;
  int64_t c = 0;
};

struct Segment {
  bool is_build = false;
  std::string name;   // build: hash table name
  std::string table;  // scanned table
  std::vector<FilterIR> filters;
  std::vector<ProbeIR> probes;
  // build
  std::vector<std::string> key;
  RefIR payload;  // CONST kind => none
  int hash = -1;  // -1 auto, H_MULT, H_ORDERED, 2 = direct
  bool multi = false;  // 'multi': the key is not unique; probes join every match (NEXT-4 fan-out)
  // partition segment (NEXT-4 partitioned hash join): 'partition NAME' ... 'key COL by HT' ['parts P']:
  // the scanned rows that pass its operators are range-partitioned by COL over HT's key domain into the
  // derived table NAME (COL + rowid), grouped by partition, which a later 'run NAME' segment probes
  bool is_partition = false;
  std::string by_ht;
  int nparts = 1024;
  int load_pct = 50;
  // probe segment
  std::vector<WhereIR> wheres;
  std::vector<GroupIR> groups;
  std::vector<TermIR> value;
  std::vector<AggIR> aggs;  // agg 0 is always COUNT
  // hash group-by over unbounded keys (NEXT-4): 'group hash A[, B]' (no
  // domain), then optional 'order ...' / 'limit K' run on the device
  bool hash_group = false;
  std::vector<OrderIR> order;  // dense groups: applied on the host by gpl_fetch_result (A10)
  int limit = 0;
  std::vector<DecodeIR> decodes;  // A10: group key decodes through loaded tables
  std::vector<RatioIR> ratios;    // A10: derived ratio columns
  int split_hint = -2;      // -2: auto
  std::string text;
};

// Parse one segment. Returns false with a message (line number included).
bool parse_segment(const std::string& text, Segment* out, std::string* err);

}  // namespace gpl
