// common.h — POD descriptors shared by the host lowering (plan.cpp) and the
// sm_100a kernels (build.cu, pipeline.cu, kbe.cu). No torch, no CUDA types.
#pragma once
#ifndef __CUDACC_RTC__
#include <cstdint>
#else  // NVRTC (plan-specialised JIT kernels): no host headers
typedef int int32_t;
typedef unsigned int uint32_t;
typedef long long int64_t;
typedef unsigned long long uint64_t;
#endif

namespace gpl {

constexpr int MAXC = 8;      // staged / scanned columns per segment
constexpr int MAXF = 4;      // filters
constexpr int MAXP = 4;      // probes
constexpr int MAXR = 3;      // where-residuals
constexpr int MAXG = 3;      // group-by dimensions
constexpr int MAXA = 4;      // aggregates (agg 0 = COUNT)
constexpr int MAXQ = 12;     // survivor-queue fields
constexpr int MAXHT = 8;     // hash tables referenced by one segment
constexpr int MAXTERM = 2;   // value = term +/- term
constexpr int MAXFACT = 3;   // factors per term
constexpr int MAXOPS = 16;   // op_pass counters
constexpr int RPL = 4;       // rows per lane per consumer iteration (128-row warp packets)
constexpr int MAXSP = 2;     // probes that may run in the stage phase (register slots)
constexpr int QCAP = 256;    // survivor-queue entries per warp (>= 127 + 128)
constexpr int kSmemTableMax = 32 * 1024;     // DIRECT tables up to this size are staged in smem
constexpr int kSmemTablesTotal = 48 * 1024;  // ... up to this total per CTA

constexpr uint32_t EMPTY32 = 0xFFFFFFFFu;
constexpr unsigned long long EMPTY64 = 0xFFFFFFFFFFFFFFFFull;

// Device error bits (latched, returned at fetch/sync).
enum : uint32_t { ERR_DOMAIN = 1u, ERR_DUPKEY = 2u, ERR_RESERVED_KEY = 4u, ERR_CAPACITY = 8u };

// ---- filters: x passes RANGE iff lo <= x <= hi; MASK iff 0 <= x < 64 and bit x of mask; NE iff x != lo
enum : int32_t { F_RANGE = 0, F_MASK = 1, F_NE = 2 };
struct Filt {
  int32_t kind, ref;  // ref: stage column (pipeline) / scanned column (build) / field (residual)
  int64_t lo, hi;
  uint64_t mask;
};

// ---- hash tables (open addressing, linear probing, power-of-two slots)
// Hashed kinds: open addressing, linear probing, power-of-two slots:
//   SET32 4 B {key}, MAP32 8 B {key, payload}, MAP64 16 B {key64, payload64}.
// DIRECT: direct-addressed array over a dense key domain [kmin, kmin+nslots)
//   (a collision-free perfect hash): width 0 = bitmap set, W_NIBBLE = 4-bit
//   cells (two per byte, the even cell in the low nibble; payload ranges of at
//   most 15 values: nation keys, years), else 1/2/4-byte cells; a cell holds
//   payload - pay_base + 1 (0 = empty).
// MULTI (non-unique build keys): CSR over a dense key
//   domain — slots = uint32 offsets[nslots + 1], pay = int32 payload[count];
//   key k's matches are pay[off[k - kmin] .. off[k - kmin + 1]) (fan-out join).
// PART: not a hash table — the output of a partition segment (a derived table), registered by name so
//   the query's segment bookkeeping (graphs, caches) treats it like a build.
enum : int32_t { HT_SET32 = 0, HT_MAP32 = 1, HT_MAP64 = 2, HT_DIRECT = 3, HT_MULTI = 4, HT_PART = 5 };
constexpr int32_t W_NIBBLE = 3;  // DIRECT cell width code of 4-bit cells (not a byte count)
enum : int32_t { H_MULT = 0, H_ORDERED = 1 };

// Device-resident header, written by the build's count and size kernels and
// read by every probing kernel's prologue (sizing is exact and on-device).
struct HTHeader {
  unsigned long long count;  // rows that reached the insert step
  long long kmin, kmax;      // inserted key range (ordered hash)
  unsigned long long mult;   // ordered hash: slot = ((key-kmin)*mult) >> 32
  uint32_t log2, mask;       // nslots = mask + 1 = 1 << log2
  // count-pass accumulators; the count kernel's last block publishes them
  // into the fields above and resets them (so no per-build init launch).
  unsigned long long acc_count;
  long long acc_kmin, acc_kmax;
  uint32_t done, pad;
};

struct HTRef {
  const void* slots;
  const HTHeader* hdr;
  int32_t kind, hash;
  // DIRECT only (host-decided): key base, cell count, payload base, cell width
  long long kmin;
  unsigned long long nslots;
  long long pay_base;
  int32_t width, pad;
  const void* pay;  // MULTI: the payload array (slots = offsets)
};

// ---- probes
enum : int32_t { P_INNER = 0, P_SEMI = 1, P_MARK = 2 };
struct Probe {
  int32_t ht;         // index into the segment's HTRef table
  int32_t kind;
  int32_t k1, k2;     // key refs (k2 = -1: single int32 key; else composite (k1<<32)|k2)
  int32_t out;        // ref receiving payload (INNER on MAP) or flag (MARK); -1 none
};

// ---- residual predicates on queue fields
enum : int32_t { R_EQ = 0, R_PAIRS = 1, R_RANGE = 2, R_MASK = 3 };
struct Resid {
  int32_t kind, a, b, npairs;
  int32_t pa[4], pb[4];
  int64_t lo, hi;
  uint64_t mask;
};

// ---- group-by: gid = sum_d (t(v_d) - lo_d) * stride_d, t = identity or year
enum : int32_t { G_ID = 0, G_YEAR = 1 };
struct GroupDim {
  int32_t field, transform;
  int32_t lo, size, stride, pad;
};

// ---- value expression: sum over terms of sign * prod(a + b * x_field)
struct Factor {
  int32_t field;  // -1: constant a
  int32_t b;      // +1 / -1
  int64_t a;
};
struct Term {
  int32_t sign, nfact;
  Factor f[MAXFACT];
};

// ---- aggregates
enum : int32_t { A_COUNT = 0, A_SUM = 1, A_SUMIF = 2, A_SUMIFEQ = 3 };
struct Agg {
  int32_t kind, field;
  int64_t c;
};
enum : int32_t { AGG_REG = 0, AGG_SMEM = 1, AGG_GLOBAL = 2, AGG_HASH = 3 };
enum : int32_t { SINK_AGG = 0, SINK_INSERT = 1, SINK_PCOUNT = 2, SINK_PSCATTER = 3 };

// ---- survivor-queue push: field <- stage column, stage-phase probe slot, or
// a value term computed in the stage phase (expression pushdown)
enum : int32_t { PUSH_COL = 0, PUSH_SREG = 1, PUSH_TERM = 2, PUSH_ROWID = 3 };
struct Push {
  int32_t kind, src;
};
// Stage-phase factor refs: >= 0 stage column, -1 constant, <= -2 stage slot (-(p+2)).
constexpr int32_t SREF_CONST = -1;

// Descriptor of the fused probe-segment pipeline (kernel parameter, by value).
struct PipeDesc {
  // staging (A3)
  long long nrows;
  const char* col[MAXC];
  int32_t colw[MAXC];
  int32_t coloff[MAXC];  // byte offset of column c inside one ring slot (-1: lazy)
  // late materialisation (the paper's k_reduce fetches
  // LINEITEM only for satisfied tuples): a lazy column is not staged by
  // TMA; its values are gathered from HBM for the rows that reach its first use
  int32_t lazy[MAXC];
  int32_t ncols, slot_bytes;
  // schedule (A2)
  long long tile_rows;
  int32_t stage_rows, depth, nwarps, flush_each_tile;
  int32_t npack;  // 128-row packets per consumer iteration (1 or 2: stage-phase probes of both in flight)
  int32_t min_blocks;  // CTAs per SM the configuration runs (JIT: __launch_bounds__ minimum, caps registers)
  // operator-specialised consumer warps (the paper's
  // per-operator kernels and work-group counts, Eq 8): the last
  // ndrain consumer warps only drain survivor packets that the stage warps
  // hand over through a 2*ndrain-slot shared-memory ring (0: every consumer
  // warp drains its own queue)
  int32_t ndrain;
  // stage phase (A4 + first probes)
  int32_t nfilt, nsprobe, nprobe, npush;
  Filt filt[MAXF];
  Probe probe[MAXP];     // [0, nsprobe): keys are stage columns; [nsprobe, nprobe): keys are fields
  Push push[MAXQ];       // push[i] fills queue field i
  int32_t qoff[MAXQ];    // byte offset of field f's array in a warp's queue (QCAP entries)
  int32_t qw[MAXQ];      // field width in bytes (4 or 8)
  int32_t qbytes;        // bytes of one warp's queue
  int32_t qlazy[MAXQ];   // >= 0: field f is lazy column qlazy[f], gathered by the drain via the row id
  int32_t qlazy_at[MAXQ];  // lazy field f is gathered right before queue probe qlazy_at[f] (nprobe: before
                           // the group-by / value / sink), only for the rows still alive there
  // 1: fields the drain produces (f >= npush: lazy gathers, queue-probe slots) live in registers of the
  // plan-specialised kernel; the warp queues hold only the pushed fields (0: every field in the queue)
  int32_t reg_fields;
  // AGG_SMEM: copies of the shared-memory group table, one per lane (32) when
  // it fits, else 1; kept as separate low / high 32-bit word arrays so a row's
  // add is two native 32-bit shared atomics (no 64-bit CAS loop)
  int32_t agg_lanes;
  // clustered probe: stage probe cl_probe reads a DIRECT table by a key column
  // (cl_col) sorted in the fact table, so one stage's keys span a narrow cell
  // range; the producer TMA-stages those cells (<= cl_cap bytes at slot offset
  // cl_off) beside the columns and the probe reads shared memory
  int32_t cl_probe, cl_col, cl_off, cl_cap;
  int32_t cl_kpr, cl_pad;  // clustered probe: staged keys per stage row (cell buffer = cl_kpr x stage rows)
  int32_t rowid_field;   // queue field holding the row id (-1: no lazy column)
  // fan-out probe (NEXT-4): queue-phase probe into a MULTI table; every match
  // of a row continues through the remaining operators (-1: none)
  int32_t fan_probe, fan_pad;
  int32_t term_field[MAXTERM];  // >= 0: term t was computed in the stage phase into this field
  Term sterm[MAXTERM];          // stage-phase form of pushed-down terms (stage refs)
  int32_t nfield, nresid, ngroup, ngroups_total;
  Resid resid[MAXR];
  GroupDim gdim[MAXG];
  int32_t nterm, nagg, agg_mode, nht;
  Term term[MAXTERM];
  Agg agg[MAXA];
  HTRef ht[MAXHT];
  // small DIRECT tables copied into shared memory at kernel start (-1: global)
  int32_t ht_smem_off[MAXHT];
  int32_t ht_smem_bytes[MAXHT];
  int32_t smem_tables_bytes;
  // smem layout
  int32_t off_queue, off_agg, off_ring, smem_bytes;
  // sink: SINK_AGG (probe segment: group-by aggregation) or SINK_INSERT (build
  // segment run through the same pipeline: insert key -> payload into a DIRECT
  // table; the blocking hash build of P:147 as the segment's last operator)
  int32_t sink;
  int32_t ins_kfield, ins_pfield, ins_ptransform, ins_width;  // queue fields, G_ID/G_YEAR, cell bytes (0 = bitmap)
  // stage-phase insert (every probe in the stage phase): key / payload stage
  // columns, or the payload's stage-probe slot; ins_kcol < 0: insert from the queue
  // ins_dense (clustered build): the key column is sorted and the domain is its [min, max], so each
  // packet writes its whole cell range — its rows' cells (0 when a row fails) and the key gaps between
  // them — with plain stores: no atomics and no clear pass (P:147's blocking build, B200 form)
  // ins_q: the insert runs in the queue phase (drain) from queue fields (queue-phase probes or
  // residuals before it); a dense build then zero-fills each packet's cell range in the stage phase
  // (ins_kcol: the staged key column) and the drain writes the surviving rows' cells
  int32_t ins_kcol, ins_pcol, ins_psreg, ins_dense, ins_q;
  long long ins_kmin, ins_pay_base;                            // run-time (table bases)
  unsigned long long ins_nslots;
  void* ins_slots;
  // hash group-by (AGG_HASH): open addressing, linear
  // probing over 2^hagg_log2 slots; hagg_keys holds ~key (0 = empty, so the
  // table clears with zeros), hagg_accs [slot][nagg] exact int64 sums;
  // hagg_count counts distinct groups (CAS winners)
  unsigned long long* hagg_keys;
  long long* hagg_accs;
  unsigned long long* hagg_count;
  int32_t hagg_log2, hagg_pad;
  // partition phase (NEXT-4 partitioned hash join): SINK_PCOUNT counts the rows of each
  // (partition, CTA) in a shared-memory histogram, SINK_PSCATTER writes (key, source row id) at the
  // CTA's own offsets (exclusive scan of the counts, partition-major), so the output is grouped by
  // partition with no global atomics. Partition of a key: (key - part_kmin) >> part_shift; keys outside
  // [part_kmin, part_kmin + nparts << part_shift) cannot join and are dropped. Both passes use static
  // tiles (CTA b takes tiles b, b + grid, ...) so a CTA sees the same rows twice.
  long long part_kmin;
  int32_t part_shift, nparts;
  unsigned* part_hist;   // [nparts][grid] counts, then (after the scan) offsets
  int* part_key_out;
  int* part_row_out;
  int32_t static_tiles, part_pad;
  long long part_row0;   // row id of the first scanned row (zone restriction offset)
  // rows to scan read from the device at kernel start (a partitioned table's row count; 0: nrows)
  const unsigned* nrows_dev;
  // outputs
  unsigned long long* partials;      // [ngroups_total][nagg] x (lo, hi)
  unsigned long long* tile_counter;  // zeroed before launch
  unsigned long long* op_pass;       // [MAXOPS]
  unsigned int* err;
};

// Result step of a hash group-by (blocking, after the pipeline): ORDER BY ...
// LIMIT k selection, or compaction of every group. Rows are [key, acc 0..nagg).
struct HaggResultDesc {
  const unsigned long long* keys;  // ~key per slot, 0 = empty
  const long long* accs;           // [slot][nagg]
  unsigned long long nslots;
  int32_t nagg, nkeys;             // key fields packed (k0 << 32 | k1) when nkeys == 2
  int32_t limit;                   // 0: every group (compaction)
  int32_t norder;
  int32_t ord_is_agg[3], ord_idx[3], ord_desc[3];
  unsigned long long* cand;        // selection scratch: [nblocks * limit] x (4 sort words, slot index)
  int32_t nblocks, pad;
  unsigned long long* rows;        // out: n_out rows of (1 + nagg) words (device)
  unsigned long long* small_out;   // out (limit): [n_groups, n_out, rows...] in the partials area
  unsigned long long* n_out;       // out (compaction): row counter (zeroed per run)
};

// Descriptor of one build segment (hash_build kernels).
enum : int32_t { PAY_NONE = 0, PAY_COL = 1, PAY_SLOT = 2, PAY_YEARCOL = 3 };
struct BuildDesc {
  long long nrows;
  const char* col[MAXC];
  int32_t colw[MAXC];
  int32_t ncols, nfilt, nprobe, k1, k2, pay_kind, pay_ref, nht;
  Filt filt[MAXF];
  Probe probe[MAXP];  // inner/semi probes into earlier tables; out = slot register 0..MAXP-1
  HTRef src[MAXHT];
  void* slots;        // destination table
  HTHeader* hdr;
  void* pay;          // MULTI: payload array
  unsigned int* cursor;  // MULTI: per-key counts, then scatter cursors [nslots + 1]
  void* scan_tmp;        // MULTI: device scan scratch
  unsigned long long scan_tmp_bytes;
  long long cap_slots;
  int32_t kind, hash, load_pct, width;  // width: DIRECT cell bytes (0 = bitmap)
  long long kmin, pay_base;             // DIRECT key / payload bases
  unsigned long long nslots;            // DIRECT cells
  unsigned int* err;
};

}  // namespace gpl
