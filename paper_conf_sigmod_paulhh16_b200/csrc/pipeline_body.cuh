// pipeline_body.cuh — A2-A8: the fused, warp-specialised, persistent
// probe-segment kernel body for sm_100a.
//
// GPL's segment = concurrently running kernels connected by channels, fed one
// tile at a time (§3.1, §3.3, §3.4,
// P:191-203 §3.5). The B200 re-expression is ONE kernel per segment:
//
//   producer warp (lane 0)                     consumer warps (W per CTA)
//   ----------------------                     -------------------------------------------
//   claim tile t = atomicAdd(counter)   A2     wait full[slot]
//   for each stage of the tile:                for each 128-row packet of the stage
//     wait empty[slot]                         (4 consecutive rows per lane):
//     cp.async.bulk every column       A3        filters (selection = map only)  A4
//       (TMA engine, L2 evict_first)             stage-phase probes (first `nsprobe`)     A5
//     arrive.expect_tx full[slot]                value terms computable here (pushdown)
//                                                ballot/popc compaction -> warp queue     A8
//                                                whenever >= 128 survivors are queued:
//                                                  remaining probes, where, group-by,   A5-A7
//                                                  exact int64 aggregation
//                                              arrive empty[slot]
//
// The ring of `depth` stages replaces the paper's "number of channels" n and
// the warp packet replaces its packet size p. Survivors travel
// through per-warp shared-memory queues carrying their values, so no operator
// writes an intermediate to HBM; the only global writes are the
// few-KB aggregate partials (int128) and counters.
//
// One source, two instantiations:
//   * generic (pipeline.cu, precompiled): the plan shape is read from the
//     kernel parameter `d` at run time;
//   * plan-specialised (jit.cpp, NVRTC at first use of a plan): the shape is a
//     constexpr descriptor, so every count, kind, width, offset and constant
//     folds into the code and every operator loop unrolls.
// `K` is the shape (GPL_SHAPE_OF(d)); `d` supplies the run-time fields only:
// column / table / output pointers, nrows, tile_rows.
//
// All shared-memory accesses use integer offsets into one __shared__ array so
// they compile to plain LDS/STS.
#pragma once
#include "device_common.cuh"

#ifndef GPL_SHAPE_OF
#define GPL_SHAPE_OF(d) (d)
#endif
#ifdef GPL_JIT
#define GPL_UNROLL _Pragma("unroll")
#define GPL_DRAIN_INLINE __forceinline__
#else
#define GPL_UNROLL
#define GPL_DRAIN_INLINE __noinline__
#endif

namespace gpl {
namespace pipe {

extern __shared__ __align__(128) unsigned char g_smem[];

constexpr int kMaxWarps = 17;  // 16 consumers + 1 producer
constexpr int kMaxThreads = kMaxWarps * 32;
constexpr int kMaxDepth = 8;
// fixed shared-memory region (see PipeDesc.off_*):
constexpr int kOffFull = 0;       // unsigned long long[kMaxDepth]
constexpr int kOffEmpty = 64;     // unsigned long long[kMaxDepth]
constexpr int kOffHdr = 128;      // int4[kMaxDepth]
constexpr int kOffHtp = 256;      // HTP[MAXHT]
constexpr int kOffHdr2 = 896;     // int4[kMaxDepth]: clustered-probe cell range (start lo, hi, bytes)
constexpr int kOffCnt = 1024;     // unsigned long long[kMaxWarps][MAXOPS]
// drain hand-off ring (ndrain > 0): a bounded multi-producer / multi-consumer
// queue of R slots. Slot s carries a sequence number: ticket t may fill it
// when seq == t and drain it when seq == t + 1 (then seq = t + R). Several
// stage warps hold tickets at once, so an mbarrier's phase parity could not
// tell ticket t from ticket t + 2R; the sequence numbers can.
constexpr int kMaxHand = 8;
constexpr int kOffHSeq = 3328;    // unsigned[kMaxHand]
constexpr int kOffHHdr = 3456;    // int[kMaxHand]: entries in the packet (-1: end)
constexpr int kOffHTick = 3488;   // unsigned[3]: producer ticket, consumer ticket, stage warps done
static_assert(kOffHtp + MAXHT * sizeof(HTP) <= kOffHdr2, "HTP region overflow");
static_assert(kOffHdr2 + kMaxDepth * 16 <= kOffCnt, "header region overflow");
static_assert(kOffCnt + kMaxWarps * MAXOPS * 8 <= kOffHSeq, "counter region overflow");
static_assert(kOffHTick + 12 <= 4096, "fixed region overflow");

template <class T>
__device__ __forceinline__ T& S(uint32_t off) {
  return *reinterpret_cast<T*>(g_smem + off);
}

// shared-space scalar loads at a shared-window address (see smem_base)
__device__ __forceinline__ uint32_t lds_u32(uint32_t sa) {
  uint32_t v;
  asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(sa));
  return v;
}
__device__ __forceinline__ uint32_t lds_u16(uint32_t sa) {
  unsigned short v;
  asm volatile("ld.shared.u16 %0, [%1];" : "=h"(v) : "r"(sa));
  return v;
}
__device__ __forceinline__ uint32_t lds_u8(uint32_t sa) {
  uint32_t v;
  asm volatile("ld.shared.u8 %0, [%1];" : "=r"(v) : "r"(sa));
  return v;
}

__device__ __forceinline__ long long lds_s64(uint32_t sa) {
  long long v;
  asm volatile("ld.shared.s64 %0, [%1];" : "=l"(v) : "r"(sa));
  return v;
}
__device__ __forceinline__ int lds_s32(uint32_t sa) {
  int v;
  asm volatile("ld.shared.s32 %0, [%1];" : "=r"(v) : "r"(sa));
  return v;
}
__device__ __forceinline__ void sts_32(uint32_t sa, int v) {
  asm volatile("st.shared.u32 [%0], %1;" ::"r"(sa), "r"(v));
}
__device__ __forceinline__ void sts_64(uint32_t sa, long long v) {
  asm volatile("st.shared.u64 [%0], %1;" ::"r"(sa), "l"(v));
}

__device__ __forceinline__ unsigned lanemask_lt() {
  unsigned m;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}

// Shared-space loads at g_smem + a: the shared-window address of g_smem is
// computed once per thread (smem_base) instead of being rematerialised from
// SR_CgaCtaId for every load of the hot loop (ncu: that S2R + LEA chain was
// the top stall of the stage phase). Volatile: never hoisted above the ring's
// mbarrier waits (which are volatile asm too).
__device__ __forceinline__ uint32_t smem_base() {
  return (uint32_t)__cvta_generic_to_shared(g_smem);
}
__device__ __forceinline__ int4 lds_v4(uint32_t sa) {
  int4 v;
  asm volatile("ld.shared.v4.s32 {%0, %1, %2, %3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(sa));
  return v;
}
__device__ __forceinline__ longlong2 lds_v2_64(uint32_t sa) {
  longlong2 v;
  asm volatile("ld.shared.v2.s64 {%0, %1}, [%2];" : "=l"(v.x), "=l"(v.y) : "r"(sa));
  return v;
}

// RPL consecutive rows (r0 % 4 == 0) of one staged column, widened to int64.
__device__ __forceinline__ void ld_rows(uint32_t a, int w, long long (&x)[RPL]) {
  const uint32_t sa = smem_base() + a;
  if (w == 4) {
    const int4 v = lds_v4(sa);
    x[0] = v.x; x[1] = v.y; x[2] = v.z; x[3] = v.w;
  } else {
    const longlong2 u = lds_v2_64(sa);
    const longlong2 v = lds_v2_64(sa + 16);
    x[0] = u.x; x[1] = u.y; x[2] = v.x; x[3] = v.y;
  }
}

// A 4-byte filter column evaluated in 32-bit arithmetic (dates, keys, codes):
// range as one unsigned compare of x - lo against hi - lo, bounds clamped to
// the int32 range (an empty clamp passes nothing).
__device__ __forceinline__ void filt_rows32(const Filt& F, uint32_t a, bool* p) {
  const int4 v = lds_v4(smem_base() + a);
  const int x[RPL] = {v.x, v.y, v.z, v.w};
  if (F.kind == F_RANGE) {
    const long long lo = F.lo < -2147483648LL ? -2147483648LL : F.lo;
    const long long hi = F.hi > 2147483647LL ? 2147483647LL : F.hi;
    const bool none = lo > hi;
    const unsigned lo32 = (unsigned)(int)(none ? 0 : lo), span = (unsigned)((none ? 0 : hi) - (none ? 0 : lo));
#pragma unroll
    for (int j = 0; j < RPL; j++) p[j] = p[j] && !none && ((unsigned)x[j] - lo32) <= span;
  } else if (F.kind == F_MASK) {
#pragma unroll
    for (int j = 0; j < RPL; j++) p[j] = p[j] && (unsigned)x[j] < 64u && ((F.mask >> x[j]) & 1ull);
  } else {
#pragma unroll
    for (int j = 0; j < RPL; j++) p[j] = p[j] && (long long)x[j] != F.lo;
  }
}

// RPL rows of column c for one lane: from the staged tile, or — for a lazy
// (late-materialised) column — gathered from HBM for the active rows only.
__device__ __forceinline__ void ld_col(const PipeDesc& d, const PipeDesc& K, int c, uint32_t sb, int r0,
                                       long long rowbase, const bool* act, long long (&x)[RPL]) {
  if (K.lazy[c]) {
#pragma unroll
    for (int j = 0; j < RPL; j++) x[j] = act[j] ? ld_col_global(d.col[c], K.colw[c], rowbase + r0 + j) : 0;
  } else {
    ld_rows(sb + K.coloff[c] + r0 * K.colw[c], K.colw[c], x);
  }
}

// RPL rows of a 32-bit key column (probe keys are validated 32-bit): staged
// (one 16-B shared load) or, for a lazy column, gathered for the active rows
__device__ __forceinline__ void ld_key32(const PipeDesc& d, const PipeDesc& K, int c, uint32_t sb, int r0,
                                         long long rowbase, const bool* act, uint32_t (&x)[RPL]) {
  if (K.lazy[c]) {
#pragma unroll
    for (int j = 0; j < RPL; j++) x[j] = act[j] ? __ldg((const uint32_t*)d.col[c] + rowbase + r0 + j) : 0u;
  } else {
    const int4 v = lds_v4(smem_base() + sb + K.coloff[c] + r0 * 4);
    x[0] = (uint32_t)v.x; x[1] = (uint32_t)v.y; x[2] = (uint32_t)v.z; x[3] = (uint32_t)v.w;
  }
}

// survivor-queue field access (shared-space loads/stores, see smem_base)
__device__ __forceinline__ long long qget(const PipeDesc& K, uint32_t qb, int f, int i) {
  const uint32_t a = smem_base() + qb + K.qoff[f];
  return K.qw[f] == 4 ? (long long)lds_s32(a + i * 4) : lds_s64(a + i * 8);
}
__device__ __forceinline__ void qput(const PipeDesc& K, uint32_t qb, int f, int i, long long v) {
  const uint32_t a = smem_base() + qb + K.qoff[f];
  if (K.qw[f] == 4) sts_32(a + i * 4, (int)v);
  else sts_64(a + i * 8, v);
}

// Probe RPL rows of one lane in table t: small DIRECT tables were staged in
// shared memory by the prologue (LDS, no L1/L2 round trip); the rest go to
// global memory (ht_probe_n: all RPL loads in flight).
template <int N>
__device__ __forceinline__ void probe_rows(const PipeDesc& K, const HTP& h, int t, const unsigned long long (&key)[N],
                                           const bool (&act)[N], bool (&hit)[N], long long (&pay)[N]) {
  const int kind = K.ht[t].kind, width = K.ht[t].width, so = K.ht_smem_off[t];
  if (kind == HT_DIRECT && so >= 0) {
    // branch-free: the cell index is clamped into the table and the loaded
    // value masked, so the 4 shared-memory loads issue back to back
    const uint32_t last = (uint32_t)(h.nslots - 1);
    const uint32_t sso = smem_base() + (uint32_t)so;
    uint32_t v[N];
#pragma unroll
    for (int j = 0; j < N; j++) {
      const unsigned long long idx = (unsigned long long)((long long)(int32_t)(uint32_t)key[j] - (long long)h.kmin);
      const bool in = act[j] && idx < h.nslots;
      const uint32_t i = in ? (uint32_t)idx : last;
      uint32_t x;
      if (width == 0) x = (lds_u32(sso + (i >> 5) * 4) >> (i & 31)) & 1u;
      else if (width == W_NIBBLE) x = (lds_u8(sso + (i >> 1)) >> ((i & 1) * 4)) & 0xFu;
      else if (width == 1) x = lds_u8(sso + i);
      else if (width == 2) x = lds_u16(sso + i * 2);
      else x = lds_u32(sso + i * 4);
      v[j] = in ? x : 0u;
    }
#pragma unroll
    for (int j = 0; j < N; j++) {
      hit[j] = v[j] != 0;
      pay[j] = width == 0 ? 1 : (long long)v[j] - 1 + h.pay_base;
    }
    return;
  }
  ht_probe_n<N>(h, kind, width, key, act, hit, pay);
}

// Clustered probe (DIRECT table, key column sorted in the fact table): the
// producer staged the cells of the stage's key range at smem byte `base`; they
// cover keys [k0, k0 + ncells). The column is sorted (checked at load), so
// every key of the stage lies in the staged range or outside the table's
// domain: one 32-bit subtract + compare + predicated LDS per row, no 64-bit
// index math and no global fallback (a stage whose range did not fit the slot
// probes the table in memory instead, see the caller).
template <int N>
__device__ __forceinline__ void probe_rows_cl(const PipeDesc& K, const HTP& h, int t, const unsigned long long (&key)[N],
                                              const bool (&act)[N], bool (&hit)[N], long long (&pay)[N], uint32_t base,
                                              uint32_t k0, uint32_t ncells) {
  const int width = K.ht[t].width;
  const uint32_t sbase = (uint32_t)__cvta_generic_to_shared(g_smem) + base;
  uint32_t x[N];
#pragma unroll
  for (int j = 0; j < N; j++) {
    const uint32_t o = (uint32_t)key[j] - k0;
    const bool in = act[j] && o < ncells;
    uint32_t v = 0;
    if (width == 0) v = in ? (lds_u32(sbase + (o >> 5) * 4) >> (o & 31)) & 1u : 0u;
    else if (width == W_NIBBLE) v = in ? (lds_u8(sbase + (o >> 1)) >> ((o & 1) * 4)) & 0xFu : 0u;
    else if (width == 1) v = in ? lds_u8(sbase + o) : 0u;
    else if (width == 2) v = in ? lds_u16(sbase + o * 2) : 0u;
    else v = in ? lds_u32(sbase + o * 4) : 0u;
    x[j] = v;
  }
#pragma unroll
  for (int j = 0; j < N; j++) {
    hit[j] = x[j] != 0;
    pay[j] = width == 0 ? 1 : (long long)x[j] - 1 + h.pay_base;
  }
}

__device__ __forceinline__ unsigned count4(const bool (&p)[RPL]) {
  return (unsigned)p[0] + (unsigned)p[1] + (unsigned)p[2] + (unsigned)p[3];
}
__device__ __forceinline__ bool any4(const bool (&p)[RPL]) { return p[0] | p[1] | p[2] | p[3]; }
// v added mod 2^64 to the counter whose low word is lo[i] and high word
// lo[words + i], with two native 32-bit shared atomics: the low word's carry
// (old + v.lo wrapped) goes into the high word. Concurrent adds are exact; the
// words are read only after the CTA's barrier.
__device__ __forceinline__ void smem_add_split(unsigned* lo, int words, int i, unsigned long long v) {
  const unsigned l = (unsigned)v, h = (unsigned)(v >> 32);
  const unsigned old = atomicAdd(lo + i, l);
  const unsigned up = h + (unsigned)(old + l < old);
  if (up) atomicAdd(lo + words + i, up);
}
// rows per lane of one consumer iteration: up to two packets in the
// plan-specialised kernel; the generic kernel keeps one (register budget)
#ifdef GPL_JIT
constexpr int NR = 2 * RPL;
#else
constexpr int NR = RPL;
#endif
constexpr int NPMAX = NR / RPL;
__device__ __forceinline__ unsigned count_n(const bool (&p)[NR]) {
  unsigned c = 0;
#pragma unroll
  for (int j = 0; j < NR; j++) c += (unsigned)p[j];
  return c;
}
__device__ __forceinline__ bool any_n(const bool (&p)[NR]) {
  bool a = false;
#pragma unroll
  for (int j = 0; j < NR; j++) a |= p[j];
  return a;
}

// Build segments: the blocking hash build as the pipeline's last
// operator, N rows of a lane at a time. DIRECT cells start at 0 (= empty):
// bitmap cells by atomicOr, 32-bit cells by atomicCAS, 1- and 2-byte cells by
// atomicOr into their word; a non-empty old cell is a duplicate key (FK->PK
// joins only). All N atomics are issued before any old value is examined, so
// their round trips overlap (one latency per call, not N).
template <int N>
__device__ __forceinline__ void insert_cells(const PipeDesc& d, const PipeDesc& K, const long long (&key)[N],
                                             const long long (&pay)[N], const bool (&act)[N]) {
  bool in[N];
  unsigned long long ci[N];
  bool bad = false;
#pragma unroll
  for (int j = 0; j < N; j++) {
    ci[j] = (unsigned long long)((long long)(int32_t)key[j] - d.ins_kmin);
    in[j] = act[j] && ci[j] < d.ins_nslots;
    bad |= act[j] && !in[j];
  }
  if (bad) atomicOr(d.err, ERR_CAPACITY);
  uint32_t old[N], m[N];
#pragma unroll
  for (int j = 0; j < N; j++) {
    old[j] = 0;
    m[j] = 0;
    if (!in[j]) continue;
    if (K.ins_width == 0) {
      m[j] = 1u << (ci[j] & 31);
      old[j] = atomicOr((uint32_t*)d.ins_slots + (ci[j] >> 5), m[j]);
      continue;
    }
    long long pv = pay[j];
    if (K.ins_ptransform == G_YEAR) pv = (int)pv / 10000;
    const uint32_t v = (uint32_t)(pv - d.ins_pay_base + 1);
    if (K.ins_width == 4) {
      m[j] = 0xFFFFFFFFu;
      old[j] = atomicCAS((uint32_t*)d.ins_slots + ci[j], 0u, v);
    } else if (K.ins_width == W_NIBBLE) {
      const unsigned long long byte = ci[j] >> 1;
      const uint32_t sh = (uint32_t)(byte & 3ull) * 8u + (uint32_t)(ci[j] & 1ull) * 4u;
      m[j] = 0xFu << sh;
      old[j] = atomicOr((uint32_t*)((char*)d.ins_slots + (byte & ~3ull)), v << sh);
    } else {
      const unsigned long long byte = ci[j] * (unsigned long long)K.ins_width;
      const uint32_t sh = (uint32_t)(byte & 3ull) * 8u;
      m[j] = (K.ins_width == 1 ? 0xFFu : 0xFFFFu) << sh;
      old[j] = atomicOr((uint32_t*)((char*)d.ins_slots + (byte & ~3ull)), v << sh);
    }
  }
  bool dup = false;
#pragma unroll
  for (int j = 0; j < N; j++) dup |= (old[j] & m[j]) != 0u;
  if (dup) atomicOr(d.err, ERR_DUPKEY);
}

// 4-bit cells: cell c is nibble (c & 1) of byte c >> 1; the word-level atomics
// touch only that nibble's bits, so they commute with every other cell's update
__device__ __forceinline__ uint32_t nibble_shift(long long c) {
  return (uint32_t)((c >> 1) & 3ll) * 8u + (uint32_t)(c & 1ll) * 4u;
}
__device__ __forceinline__ uint32_t* nibble_word(char* cells, long long c) {
  return (uint32_t*)(cells + ((c >> 1) & ~3ll));
}
__device__ __forceinline__ void nibble_or(char* cells, long long c, uint32_t v) {
  if (v) atomicOr(nibble_word(cells, c), (v & 0xFu) << nibble_shift(c));
}
__device__ __forceinline__ void nibble_clear(char* cells, long long c) {
  atomicAnd(nibble_word(cells, c), ~(0xFu << nibble_shift(c)));
}

// Dense (clustered) build: the cells of N qualifying rows by plain stores. The
// key column is strictly increasing, so no other row writes these cells; the
// packet's zero fill (the key gaps and failing rows) precedes them in the warp.
template <int N>
__device__ __forceinline__ void dense_cells(const PipeDesc& d, const PipeDesc& K, const long long (&key)[N],
                                            const long long (&pay)[N], const bool (&act)[N]) {
  char* cells = (char*)d.ins_slots;
#pragma unroll
  for (int j = 0; j < N; j++) {
    if (!act[j]) continue;
    long long pv = pay[j];
    if (K.ins_ptransform == G_YEAR) pv = (int)pv / 10000;
    const uint32_t v = (uint32_t)(pv - d.ins_pay_base + 1);
    const long long c = key[j] - d.ins_kmin;
    if (K.ins_width == W_NIBBLE) nibble_or(cells, c, v);  // (rows of one byte may sit in different lanes)
    else if (K.ins_width == 1) cells[c] = (char)v;
    else if (K.ins_width == 2) ((unsigned short*)cells)[c] = (unsigned short)v;
    else ((uint32_t*)cells)[c] = v;
  }
}

// A dense build's zero fill of one 128-row packet: the cells from its first
// row's key to the next packet's first key (the next stage's, at a stage end),
// aligned 16-B stores inside, byte stores at the edges it shares with its
// neighbours. Every cell of the domain is written exactly once per build.
// 4-bit cells: the packet owns the bytes whose two cells are both in its range;
// a byte it shares with a neighbouring packet (an odd first cell, an odd end)
// has its own nibble cleared by an atomic, never a byte store.
__device__ __forceinline__ void dense_zero_fill(const PipeDesc& d, const PipeDesc& K, uint32_t sb, int pb, int n,
                                                int ins_knext, int lane, long long* c0_out = nullptr,
                                                long long* c1_out = nullptr) {
  const uint32_t kcol_sa = smem_base() + sb + (uint32_t)K.coloff[K.ins_kcol];
  const int first = lds_s32(kcol_sa + (uint32_t)pb * 4u);
  const int next = pb + 128 < n ? lds_s32(kcol_sa + (uint32_t)(pb + 128) * 4u) : ins_knext;
  const int w = K.ins_width;
  char* cells = (char*)d.ins_slots;
  const long long c0 = (long long)first - d.ins_kmin, c1 = (long long)next - d.ins_kmin;  // cells [c0, c1)
  if (c0_out) *c0_out = c0;
  if (c1_out) *c1_out = c1;
  long long blo, bhi;
  if (w == W_NIBBLE) {
    blo = (c0 + 1) >> 1;
    bhi = c1 >> 1;
    if (lane == 0 && (c0 & 1)) nibble_clear(cells, c0);
    if (lane == 1 && (c1 & 1)) nibble_clear(cells, c1 - 1);
  } else {
    blo = c0 * w;
    bhi = c1 * w;
  }
  const long long alo = (blo + 15) & ~15ll, ahi = bhi & ~15ll;
  if (alo < ahi) {
    for (long long b = alo + lane * 16; b < ahi; b += 512) *(uint4*)(cells + b) = make_uint4(0u, 0u, 0u, 0u);
    for (long long b = blo + lane; b < alo; b += 32) cells[b] = 0;
    for (long long b = ahi + lane; b < bhi; b += 32) cells[b] = 0;
  } else {
    for (long long b = blo + lane; b < bhi; b += 32) cells[b] = 0;
  }
}

// Queue phase on up to RPL*32 queued survivors starting at qhead: lane `lane`
// owns entries qhead + j*32 + lane (j < RPL) that are < n. Remaining probes,
// where residuals, group-by and the exact aggregation (A5-A7).
// A fan-out probe (NEXT-4: inner join on a non-unique build key, MULTI table)
// expands each row into its matches: the warp loops over the match index m
// (up to the warp's largest match count); match m of every row writes its
// payload into the row's queue field and continues through the remaining
// probes, residuals and the sink, so no expanded row is ever materialised.
__device__ GPL_DRAIN_INLINE void drain(const PipeDesc& d, uint32_t qb, int qhead, int n, unsigned long long* cnt,
                                       long long* acc, int lane) {
  const PipeDesc& K = GPL_SHAPE_OF(d);
  const HTP* htp = &S<HTP>(kOffHtp);
  int idx[RPL];
  bool p[RPL];
#pragma unroll
  for (int j = 0; j < RPL; j++) {
    const int e = j * 32 + lane;
    idx[j] = (qhead + e) & (QCAP - 1);
    p[j] = e < n;
  }
  // Field access. Pushed fields (f < npush) live in the warp queue; the fields
  // the drain produces itself (lazy gathers, queue-probe slots) live in
  // registers of the plan-specialised kernel (reg_fields: f is a compile-time
  // constant there), else in the queue as well.
#ifdef GPL_JIT
  long long dv[MAXQ][RPL];
#define GPL_REGF(f) (K.reg_fields && (f) >= K.npush)
  auto fget = [&](int f, int j) -> long long { return GPL_REGF(f) ? dv[f][j] : qget(K, qb, f, idx[j]); };
  auto fput = [&](int f, int j, long long v) {
    if (GPL_REGF(f)) dv[f][j] = v;
    else qput(K, qb, f, idx[j], v);
  };
#undef GPL_REGF
#else
  auto fget = [&](int f, int j) -> long long { return qget(K, qb, f, idx[j]); };
  auto fput = [&](int f, int j, long long v) { qput(K, qb, f, idx[j], v); };
#endif
  // late materialisation: a lazy column is gathered right before its first
  // use (queue probe `at`, or nprobe = the group-by / value), for the rows
  // still alive there; all loads of a lane in flight together
  auto gather = [&](int at, const bool (&p)[RPL]) {
    if (K.rowid_field < 0) return;
    GPL_UNROLL
    for (int f = 0; f < K.nfield; f++) {
      const int c = K.qlazy[f];
      if (c < 0 || K.qlazy_at[f] != at) continue;
      long long v[RPL];
#pragma unroll
      for (int j = 0; j < RPL; j++)
        v[j] = p[j] ? ld_col_global(d.col[c], K.colw[c], (long long)(uint32_t)fget(K.rowid_field, j)) : 0;
#pragma unroll
      for (int j = 0; j < RPL; j++)
        if (p[j]) fput(f, j, v[j]);
    }
  };
  auto run_probes = [&](int lo, int hi, bool (&p)[RPL]) {
    GPL_UNROLL
    for (int pi = lo; pi < hi; pi++) {
      const int op = K.nfilt + pi;
      const Probe& P = K.probe[pi];
      if (__any_sync(0xffffffffu, any4(p))) {
        gather(pi, p);
        unsigned long long k[RPL];
#pragma unroll
        for (int j = 0; j < RPL; j++) {
          k[j] = (uint32_t)fget(P.k1, j);
          if (P.k2 >= 0) k[j] = (k[j] << 32) | (uint32_t)fget(P.k2, j);
        }
        bool hit[RPL];
        long long v[RPL];
        probe_rows<RPL>(K, htp[P.ht], P.ht, k, p, hit, v);
#pragma unroll
        for (int j = 0; j < RPL; j++) {
          if (P.kind == P_MARK) {
            if (p[j] && P.out >= 0) fput(P.out, j, hit[j] ? 1 : 0);
          } else {
            if (hit[j] && P.out >= 0) fput(P.out, j, v[j]);
            p[j] = hit[j];
          }
        }
      }
      const unsigned c = __reduce_add_sync(0xffffffffu, count4(p));
      if (lane == 0) cnt[op] += c;
    }
  };
  // residuals, the remaining lazy gathers, then the sink (insert or aggregate)
  auto tail = [&](bool (&p)[RPL]) {
    GPL_UNROLL
    for (int r = 0; r < K.nresid; r++) {
      const int op = K.nfilt + K.nprobe + r;
      const Resid& R = K.resid[r];
#pragma unroll
      for (int j = 0; j < RPL; j++) {
        if (!p[j]) continue;
        const long long a = fget(R.a, j);
        if (R.kind == R_EQ) {
          p[j] = a == fget(R.b, j);
        } else if (R.kind == R_PAIRS) {
          const long long b = fget(R.b, j);
          bool ok = false;
          GPL_UNROLL
          for (int i = 0; i < R.npairs; i++) ok |= (a == R.pa[i]) & (b == R.pb[i]);
          p[j] = ok;
        } else if (R.kind == R_RANGE) {
          p[j] = a >= R.lo && a <= R.hi;
        } else {
          p[j] = (unsigned long long)a < 64ull && ((R.mask >> a) & 1ull);
        }
      }
      const unsigned c = __reduce_add_sync(0xffffffffu, count4(p));
      if (lane == 0) cnt[op] += c;
    }
    if (!__any_sync(0xffffffffu, any4(p))) return;
    gather(K.nprobe, p);
    if (K.sink == SINK_INSERT) {
      long long kx[RPL], px[RPL];
#pragma unroll
      for (int j = 0; j < RPL; j++) {
        kx[j] = fget(K.ins_kfield, j);
        px[j] = K.ins_pfield >= 0 ? fget(K.ins_pfield, j) : 0;
      }
      if (K.ins_dense) {
        // dense build, queue-phase insert: the stage phase zero-filled this row's
        // packet range (same warp, ordered by the __syncwarp before the drain)
        dense_cells<RPL>(d, K, kx, px, p);
      } else {
        insert_cells<RPL>(d, K, kx, px, p);
      }
      return;
    }
    // the Listings' SELECT expression of row j (exact int64, bounded by the lowering)
    auto row_value = [&](int j) -> long long {
      long long val = 0;
      GPL_UNROLL
      for (int t = 0; t < K.nterm; t++) {
        if (K.term_field[t] >= 0) {
          val += fget(K.term_field[t], j);
          continue;
        }
        const Term& T = K.term[t];
        long long prod = T.sign;
        GPL_UNROLL
        for (int f = 0; f < T.nfact; f++) {
          const Factor& F = T.f[f];
          prod *= F.field < 0 ? F.a : F.a + (long long)F.b * fget(F.field, j);
        }
        val += prod;
      }
      return val;
    };
    auto agg_contrib = [&](int a, int j, long long val) -> long long {
      const Agg& A = K.agg[a];
      if (A.kind == A_SUM) return val;
      if (A.kind == A_SUMIF) return fget(A.field, j) != 0 ? val : 0;
      if (A.kind == A_SUMIFEQ) return fget(A.field, j) == A.c ? val : 0;
      return 1;
    };
    // dense group id over the GROUP BY dimensions; false outside the domain
    auto group_id = [&](int j, int& gid) -> bool {
      gid = 0;
      bool ok = true;
      GPL_UNROLL
      for (int g = 0; g < K.ngroup; g++) {
        const GroupDim& G = K.gdim[g];
        long long v = fget(G.field, j);
        if (G.transform == G_YEAR) v = (int)v / 10000;
        const long long o = v - G.lo;
        if ((unsigned long long)o >= (unsigned long long)G.size) ok = false;
        gid += (int)o * G.stride;
      }
      return ok;
    };
    if (K.agg_mode == AGG_SMEM) {
      // Shared-memory group table: sm_100 has no native 64-bit shared-memory add
      // (atom.shared.add.u64 is a CAS loop), so each add is two native 32-bit
      // atomics on the table's low / high word arrays (smem_add_split); with
      // lane-private copies (agg_lanes = 32) the lanes of a warp never hit the
      // same word, so dense groups do not serialise a warp. The
      // copies are summed mod 2^64 at the flush (exact: the lowering bounds
      // every partial by rows x max|value| < 4.6e18).
      const int L = K.agg_lanes, words = K.ngroups_total * K.nagg * L;
      unsigned* lo = &S<unsigned>(K.off_agg);
#pragma unroll
      for (int j = 0; j < RPL; j++) {
        if (!p[j]) continue;
        int gid = 0;
        if (!group_id(j, gid)) {
          atomicOr(d.err, ERR_DOMAIN);
          continue;
        }
        const long long val = row_value(j);
        GPL_UNROLL
        for (int a = 0; a < K.nagg; a++) {
          const long long c = agg_contrib(a, j, val);
          if (c != 0) smem_add_split(lo, words, (gid * K.nagg + a) * L + (L == 32 ? lane : 0), (unsigned long long)c);
        }
      }
      return;
    }
#pragma unroll
    for (int j = 0; j < RPL; j++) {
      if (!p[j]) continue;
      long long hslot = -1;  // AGG_HASH: the group's slot
      if (K.agg_mode == AGG_HASH) {
        // hash group-by over unbounded keys (NEXT-4): the packed key finds or
        // claims its slot (open addressing, linear probing); slots hold ~key
        unsigned long long key = 0;
        GPL_UNROLL
        for (int g = 0; g < K.ngroup; g++) {
          long long v = fget(K.gdim[g].field, j);
          if (K.gdim[g].transform == G_YEAR) v = (int)v / 10000;
          key = (key << 32) | (unsigned long long)(unsigned)v;
        }
        if (key == ~0ull) {
          atomicOr(d.err, ERR_RESERVED_KEY);
          continue;
        }
        const unsigned long long st = ~key, mask = (1ull << d.hagg_log2) - 1ull;
        // an overfull table stops early instead of walking every slot: no new
        // group is claimed past 7/8 load, and a probe gives up after 2^14
        // steps; both latch ERR_CAPACITY and the host re-runs with a larger table
        const unsigned long long fill_limit = mask + 1ull - ((mask + 1ull) >> 3);
        const unsigned long long max_steps = mask < 16383ull ? mask : 16383ull;
        unsigned long long h = (key * 0x9E3779B97F4A7C15ull) >> (64 - d.hagg_log2);
        for (unsigned long long step = 0; step <= max_steps; step++, h = (h + 1) & mask) {
          unsigned long long cur = __ldcg(d.hagg_keys + h);
          if (cur == 0ull) {
            if (__ldcg(d.hagg_count) >= fill_limit) break;
            cur = atomicCAS(d.hagg_keys + h, 0ull, st);
            if (cur == 0ull) {
              gred_add_u64(d.hagg_count, 1ull);
              cur = st;
            }
          }
          if (cur == st) {
            hslot = (long long)h;
            break;
          }
        }
        if (hslot < 0) {  // table full: latched, the host re-runs with a larger table
          atomicOr(d.err, ERR_CAPACITY);
          continue;
        }
      }
      int gid = 0;
      if (K.agg_mode != AGG_HASH && !group_id(j, gid)) {
        atomicOr(d.err, ERR_DOMAIN);
        continue;
      }
      const long long val = row_value(j);
      GPL_UNROLL
      for (int a = 0; a < K.nagg; a++) {
        const long long c = agg_contrib(a, j, val);
        if (K.agg_mode == AGG_REG) acc[a] += c;
        else if (c != 0) {
          if (K.agg_mode == AGG_HASH) gred_add_u64((unsigned long long*)d.hagg_accs + hslot * K.nagg + a, (unsigned long long)c);
          else atomic_add_i128(d.partials + 2 * (gid * K.nagg + a), c);
        }
      }
    }
  };
  if (K.fan_probe < 0) {
    run_probes(K.nsprobe, K.nprobe, p);
    tail(p);
    return;
  }
  run_probes(K.nsprobe, K.fan_probe, p);
  {
    const Probe& P = K.probe[K.fan_probe];
    const HTP& h = htp[P.ht];
    const uint32_t* off = (const uint32_t*)h.slots;
    gather(K.fan_probe, p);
    uint32_t beg[RPL], end[RPL];
    int mx = 0;
    unsigned tot = 0;
#pragma unroll
    for (int j = 0; j < RPL; j++) {
      const unsigned long long ix =
          (unsigned long long)((long long)(int32_t)(uint32_t)fget(P.k1, j) - (long long)h.kmin);
      const bool in = p[j] && ix < h.nslots;
      beg[j] = in ? __ldg(off + ix) : 0u;
      end[j] = in ? __ldg(off + ix + 1) : 0u;
      mx = max(mx, (int)(end[j] - beg[j]));
      tot += end[j] - beg[j];
    }
    mx = __reduce_max_sync(0xffffffffu, (unsigned)mx);
    const unsigned c = __reduce_add_sync(0xffffffffu, tot);  // output rows of the join
    if (lane == 0) cnt[K.nfilt + K.fan_probe] += c;
    for (int m = 0; m < mx; m++) {
      bool q[RPL];
#pragma unroll
      for (int j = 0; j < RPL; j++) {
        q[j] = beg[j] + (uint32_t)m < end[j];
        if (q[j] && P.out >= 0) fput(P.out, j, (long long)__ldg((const int*)h.pay + beg[j] + m));
      }
      run_probes(K.fan_probe + 1, K.nprobe, q);
      tail(q);
    }
  }
}

__device__ __forceinline__ void flush_reg(const PipeDesc& d, long long (&acc)[MAXA], int lane) {
  const PipeDesc& K = GPL_SHAPE_OF(d);
#pragma unroll
  for (int a = 0; a < MAXA; a++) {
    if (a < K.nagg) {
      // (in 128 bits: each lane's accumulator is exact, the warp's sum may not fit int64)
      unsigned long long lo;
      long long hi;
      warp_sum_i128(acc[a], lo, hi);
      if (lane == 0 && (lo | (unsigned long long)hi) != 0) atomic_add_i128_wide(d.partials + 2 * a, lo, hi);
      acc[a] = 0;
    }
  }
}

__device__ __forceinline__ void pipeline_body(const PipeDesc& d) {
  const PipeDesc& K = GPL_SHAPE_OF(d);
  unsigned long long* full = &S<unsigned long long>(kOffFull);
  unsigned long long* empty = &S<unsigned long long>(kOffEmpty);
  int4* hdr = &S<int4>(kOffHdr);
  int4* hdr2 = &S<int4>(kOffHdr2);  // clustered probe: staged cell range per slot
  HTP* htp = &S<HTP>(kOffHtp);
  unsigned long long* cnt_all = &S<unsigned long long>(kOffCnt);
  unsigned long long* stab = &S<unsigned long long>(K.off_agg);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int W = K.nwarps;          // consumer warps (the producer is warp W)
  const int Ws = W - K.ndrain;      // stage warps (the rest only drain hand-off packets)
  const int R = 2 * K.ndrain;       // hand-off ring slots

  if (threadIdx.x == 0) {
    for (int i = 0; i < K.depth; i++) {
      mbar_init(&full[i], 1);
      mbar_init(&empty[i], (uint32_t)Ws);
    }
    for (int i = 0; i < R; i++) S<unsigned>(kOffHSeq + 4 * i) = (unsigned)i;
    S<unsigned>(kOffHTick) = S<unsigned>(kOffHTick + 4) = S<unsigned>(kOffHTick + 8) = 0u;
    fence_mbar_init();
  }
  // (PDL) everything above overlaps the previous kernel's tail; tables,
  // counters and columns it may write are read only after this wait
  grid_dep_wait();
  grid_dep_launch_dependents();
  if (threadIdx.x < K.nht) htp[threadIdx.x] = load_htp(d.ht[threadIdx.x]);
  GPL_UNROLL
  for (int t = 0; t < K.nht; t++) {  // stage small DIRECT tables into shared memory
    if (K.ht_smem_off[t] >= 0) {
      const uint4* src = (const uint4*)d.ht[t].slots;
      for (int j = threadIdx.x; j < K.ht_smem_bytes[t] / 16; j += blockDim.x)
        S<uint4>(K.ht_smem_off[t] + j * 16) = __ldg(src + j);
    }
  }
  for (int i = threadIdx.x; i < kMaxWarps * MAXOPS; i += blockDim.x) cnt_all[i] = 0;
  if (K.agg_mode == AGG_SMEM && K.sink == SINK_AGG)  // low + high word arrays of every copy
    for (int i = threadIdx.x; i < K.ngroups_total * K.nagg * K.agg_lanes; i += blockDim.x) stab[i] = 0;
  // partition phase: per-CTA counts (zeroed) or write cursors (this CTA's offsets after the scan)
  if (K.sink == SINK_PCOUNT || K.sink == SINK_PSCATTER) {
    unsigned* pc = &S<unsigned>(K.off_agg);
    for (int i = threadIdx.x; i < K.nparts; i += blockDim.x)
      pc[i] = K.sink == SINK_PCOUNT ? 0u : d.part_hist[(size_t)i * gridDim.x + blockIdx.x];
  }
  __syncthreads();

  if (warp == W) {
    // ------------------------------------------------------------ producer
    if (lane == 0) {
      const unsigned long long pol = policy_evict_first();
      uint32_t slot = 0, phase = 0;
      // Stages are visited in order; the next stage is computed (and the tile
      // after it claimed) while the current one is issued, so the claim's
      // global-atomic round trip and — for a clustered probe — the loads of
      // the next stage's first/last key overlap the current stage's copies.
      const long long S = K.stage_rows;
      // rows to scan: a partitioned table's row count lives on the device
      const long long NROWS = d.nrows_dev ? (long long)*(const volatile unsigned*)d.nrows_dev : d.nrows;
      // Stage cursors: A is issued now, B next, C after B. Tiles are claimed
      // dynamically (atomicAdd), or statically for the partition phase (tile
      // b, b + grid, ...: both passes give a CTA the same rows); `tq` is the
      // tile claimed for after C's, so a claim's latency is hidden behind the
      // stages still ahead. Stage keys a clustered probe or a dense build needs
      // (first / last / next row) are loaded for B one iteration ahead, and C's
      // are prefetched into L2 two iterations ahead, so those loads hit L2 and
      // never stall the producer on an HBM round trip (ncu: that stall capped
      // the producer at ~1 stage per microsecond per CTA).
      const bool need_keys = K.cl_probe >= 0 || K.ins_dense;
      const int* kcol = K.cl_probe >= 0 ? (const int*)d.col[K.cl_col]
                        : K.ins_dense ? (const int*)d.col[K.ins_kcol] : nullptr;
      auto claim = [&](unsigned long long prev) -> unsigned long long {
        return K.static_tiles ? prev + gridDim.x : atomicAdd(d.tile_counter, 1ull);
      };
      auto stage_n = [&](unsigned long long tt, long long so) -> int {  // rows of stage (tile tt, offset so)
        const long long r0 = (long long)tt * d.tile_rows;
        if (r0 >= NROWS) return 0;
        const long long rn = min(d.tile_rows, NROWS - r0);
        return so < rn ? (int)min(S, rn - so) : 0;
      };
      unsigned long long ta = K.static_tiles ? (unsigned long long)blockIdx.x : atomicAdd(d.tile_counter, 1ull);
      long long sa = 0;
      unsigned long long tq = claim(ta);
      // advance a cursor by one stage (crossing into the queued tile)
      auto advance = [&](unsigned long long& tt, long long& so) {
        const long long r0 = (long long)tt * d.tile_rows;
        const long long rn = r0 < NROWS ? min(d.tile_rows, NROWS - r0) : 0;
        if (so + S < rn) {
          so += S;
        } else {
          tt = tq;
          so = 0;
          tq = claim(tq);
        }
      };
      unsigned long long tb = ta, tc;
      long long sb_ = sa, sc;
      advance(tb, sb_);
      tc = tb;
      sc = sb_;
      advance(tc, sc);
      auto row_of = [&](unsigned long long tt, long long so) { return (long long)tt * d.tile_rows + so; };
      // keys of A (current) and B (next)
      int klo = 0, khi = 0, knx = 0, klo_b = 0, khi_b = 0, knx_b = 0;
      const int kend = (int)(d.ins_kmin + (long long)d.ins_nslots);  // dense build: one past the domain
      auto load_keys = [&](unsigned long long tt, long long so, int& lo, int& hi, int& nx) {
        const int nn = stage_n(tt, so);
        if (!need_keys || nn <= 0) return;
        const long long r = row_of(tt, so);
        lo = __ldg(kcol + r);
        hi = __ldg(kcol + r + nn - 1);
        if (K.ins_dense) nx = r + nn < NROWS ? __ldg(kcol + r + nn) : kend;
      };
      auto prefetch_keys = [&](unsigned long long tt, long long so) {
        const int nn = stage_n(tt, so);
        if (!need_keys || nn <= 0) return;
        const long long r = row_of(tt, so);
        asm volatile("prefetch.global.L2 [%0];" ::"l"(kcol + r));
        asm volatile("prefetch.global.L2 [%0];" ::"l"(kcol + r + nn - 1));
        if (K.ins_dense && r + nn < NROWS) asm volatile("prefetch.global.L2 [%0];" ::"l"(kcol + r + nn));
      };
      load_keys(ta, sa, klo, khi, knx);
      load_keys(tb, sb_, klo_b, khi_b, knx_b);
      prefetch_keys(tc, sc);
      for (;;) {
        const int n = stage_n(ta, sa);
        if (n <= 0) break;
        const long long row = row_of(ta, sa);
        const long long rn = min(d.tile_rows, NROWS - (long long)ta * d.tile_rows);
        const bool last_of_tile = sa + S >= rn;
        const int knext = knx;
        mbar_wait(&empty[slot], phase ^ 1u);
        hdr[slot] = make_int4((int)(row & 0xffffffff), (int)(row >> 32), n, last_of_tile ? 1 : 0);
        uint32_t bytes = 0;
        GPL_UNROLL
        for (int c = 0; c < K.ncols; c++)
          if (!K.lazy[c]) bytes += ((uint32_t)n * K.colw[c] + 15u) & ~15u;
        // clustered probe: the table cells of [klo, khi] (16-B aligned), when
        // they fit the slot's cell buffer; else the consumers probe HBM/L2
        long long cl_start = 0;
        uint32_t cl_size = 0;
        if (K.cl_probe >= 0) {
          const HTP& H = htp[K.probe[K.cl_probe].ht];
          long long clo = (long long)klo - (long long)H.kmin, chi = (long long)khi - (long long)H.kmin;
          clo = max(clo, 0ll);
          chi = min(chi, (long long)H.nslots - 1);
          if (clo <= chi) {
            const int w = K.ht[K.probe[K.cl_probe].ht].width;
            const long long blo = w == 0 ? (clo >> 5) * 4 : w == W_NIBBLE ? clo >> 1 : clo * w;
            const long long bhi = w == 0 ? ((chi >> 5) + 1) * 4 : w == W_NIBBLE ? (chi >> 1) + 1 : (chi + 1) * w;
            cl_start = blo & ~15ll;
            const long long sz = ((bhi + 15) & ~15ll) - cl_start;
            if (sz <= K.cl_cap) cl_size = (uint32_t)sz;
          }
          hdr2[slot] = make_int4((int)(cl_start & 0xffffffff), (int)(cl_start >> 32), (int)cl_size, knext);
          bytes += cl_size;
        } else if (K.ins_dense) {
          hdr2[slot] = make_int4(0, 0, 0, knext);
        }
        mbar_arrive_expect_tx(&full[slot], bytes);
        unsigned char* dst = g_smem + K.off_ring + (unsigned long long)slot * K.slot_bytes;
        GPL_UNROLL
        for (int c = 0; c < K.ncols; c++)
          if (!K.lazy[c])
            bulk_g2s(dst + K.coloff[c], d.col[c] + row * K.colw[c], ((uint32_t)n * K.colw[c] + 15u) & ~15u,
                     &full[slot], pol);
        if (cl_size)
          bulk_g2s(dst + K.cl_off, (const char*)htp[K.probe[K.cl_probe].ht].slots + cl_start, cl_size, &full[slot],
                   policy_evict_last());
        if (++slot == (uint32_t)K.depth) { slot = 0; phase ^= 1u; }
        // A <- B (its keys were loaded an iteration ago), B <- C (prefetched into
        // L2 an iteration ago: load its keys now), C <- the stage after C (prefetch)
        ta = tb;
        sa = sb_;
        klo = klo_b;
        khi = khi_b;
        knx = knx_b;
        tb = tc;
        sb_ = sc;
        load_keys(tb, sb_, klo_b, khi_b, knx_b);
        advance(tc, sc);
        prefetch_keys(tc, sc);
      }
      mbar_wait(&empty[slot], phase ^ 1u);
      hdr[slot] = make_int4(0, 0, -1, 0);
      mbar_arrive(&full[slot]);
    }
    return;
  }

  // -------------------------------------------------------------- consumers
  unsigned long long* cnt = cnt_all + warp * MAXOPS;
  const uint32_t qb = (uint32_t)K.off_queue + (uint32_t)warp * (uint32_t)K.qbytes;
  long long acc[MAXA] = {0, 0, 0, 0};
  int qhead = 0, qcount = 0;
  uint32_t slot = 0, phase = 0;
#ifdef GPL_JIT
  // stage-phase probe tables' parameters live in registers for the kernel's
  // lifetime (the specialised kernel has registers to spare; the generic one
  // reads them from shared memory)
  HTP hsp[MAXSP];
#pragma unroll
  for (int sp = 0; sp < MAXSP; sp++) hsp[sp] = htp[sp < K.nsprobe ? K.probe[sp].ht : 0];
#define GPL_SP_HTP(sp) hsp[sp]
#else
#define GPL_SP_HTP(sp) htp[K.probe[sp].ht]
#endif
  // drain hand-off ring (ndrain > 0): slot s's packet lives after the stage
  // warps' queues, in the same field layout as a warp queue
  const uint32_t hq0 = (uint32_t)K.off_queue + (uint32_t)Ws * (uint32_t)K.qbytes;
  // stage warp: hand n queued survivors (from qhead) to the drain warps (n < 0: end token)
  auto seq_wait = [&](int hs, unsigned want) {  // lane 0 spins, then the warp proceeds (acquire)
    if (lane == 0) {
      volatile unsigned* q = &S<unsigned>(kOffHSeq + 4 * hs);
      while (*q != want) __nanosleep(32);
      __threadfence_block();
    }
    __syncwarp();
  };
  auto seq_set = [&](int hs, unsigned v) {  // the warp's writes are visible before the slot moves on (release)
    __syncwarp();
    if (lane == 0) {
      __threadfence_block();
      *(volatile unsigned*)&S<unsigned>(kOffHSeq + 4 * hs) = v;
    }
  };
  auto hand_off = [&](int head, int n) {
    unsigned t = 0;
    if (lane == 0) t = atomicAdd(&S<unsigned>(kOffHTick), 1u);
    t = __shfl_sync(0xffffffffu, t, 0);
    const int hs = (int)(t % (unsigned)R);
    seq_wait(hs, t);
    const uint32_t hb = hq0 + (uint32_t)hs * (uint32_t)K.qbytes;
    GPL_UNROLL
    for (int e = 0; e < K.npush; e++) {
      const uint32_t src = qb + K.qoff[e], dst = hb + K.qoff[e];
      for (int i = lane; i < n; i += 32) {
        const int si = (head + i) & (QCAP - 1);
        if (K.qw[e] == 4) S<int>(dst + i * 4) = S<int>(src + si * 4);
        else S<long long>(dst + i * 8) = S<long long>(src + si * 8);
      }
    }
    if (lane == 0) S<int>(kOffHHdr + 4 * hs) = n;
    seq_set(hs, t + 1u);
  };
  if (K.ndrain > 0 && warp >= Ws) {
    // ------------------------------------------------ drain warps (NEXT-1)
    // the queue phase (remaining probes, residuals, aggregation / insert) of
    // the packets the stage warps hand over, in ticket order
    for (;;) {
      unsigned t = 0;
      if (lane == 0) t = atomicAdd(&S<unsigned>(kOffHTick + 4), 1u);
      t = __shfl_sync(0xffffffffu, t, 0);
      const int hs = (int)(t % (unsigned)R);
      seq_wait(hs, t + 1u);
      const int n = S<int>(kOffHHdr + 4 * hs);
      if (n < 0) break;
      drain(d, hq0 + (uint32_t)hs * (uint32_t)K.qbytes, 0, n, cnt, acc, lane);
      if (K.flush_each_tile) flush_reg(d, acc, lane);
      seq_set(hs, t + (unsigned)R);
    }
  } else {
  unsigned lc[MAXF + MAXSP];  // stage-phase pass counts of this lane's rows (filters, stage probes)
#pragma unroll
  for (int i = 0; i < MAXF + MAXSP; i++) lc[i] = 0;
  // rows this warp queued = the pass count of the last stage-phase operator
  const bool kQueueCounts = !(K.sink != SINK_AGG && K.ins_kcol >= 0 && !K.ins_q);  // (a stage-phase sink queues nothing)
  unsigned long long queued = 0;
  for (;;) {
    mbar_wait(&full[slot], phase);
    const int4 h = hdr[slot];
    const int n = h.z;
    if (n < 0) break;
    const uint32_t sb = (uint32_t)K.off_ring + slot * (uint32_t)K.slot_bytes;
    const long long rowbase = ((long long)h.y << 32) | (long long)(uint32_t)h.x;  // lazy-column gathers
    // dense build: the first key after this stage in row order
    const int ins_knext = K.ins_dense ? hdr2[slot].w : 0;
    // clustered probe: the staged cells cover keys [cl_k0, cl_k0 + cl_ncells)
    uint32_t cl_k0 = 0, cl_ncells = 0;
    int cl_size = 0;
    if (K.cl_probe >= 0) {
      const int4 h2 = hdr2[slot];
      const long long cl_start = ((long long)h2.y << 32) | (long long)(uint32_t)h2.x;
      cl_size = h2.z;
      const int w = K.ht[K.probe[K.cl_probe].ht].width;
      const HTP& H = GPL_SP_HTP(K.cl_probe);
      cl_k0 = (uint32_t)((long long)H.kmin + (w == 0 ? cl_start * 8 : w == W_NIBBLE ? cl_start * 2 : cl_start / (w > 0 ? w : 1)));
      // (the 16-B rounded range may reach past the domain's last cell: those
      // bytes are zero — the build clears them — so such keys miss)
      cl_ncells = w == 0 ? (uint32_t)cl_size * 8u
                  : w == W_NIBBLE ? (uint32_t)cl_size * 2u : (uint32_t)cl_size / (uint32_t)(w > 0 ? w : 1);
    }
    const int nit = (n + 127) >> 7;
    bool released = false;
    // Each iteration takes npk (1 or 2) of the warp's 128-row packets,
    // it0 and it0 + W: their filters and stage-phase probes run in lockstep so
    // a lane keeps up to NR = 8 independent probe loads in flight (the
    // stage-phase probe latency is a warp's critical path); compaction and the
    // queue then proceed packet by packet.
    const int npk = K.npack < NPMAX ? K.npack : NPMAX;
    for (int it0 = warp; it0 < nit; it0 += npk * Ws) {
      int r0q[NPMAX];
      bool live[NPMAX];
#pragma unroll
      for (int q = 0; q < NPMAX; q++) {
        r0q[q] = ((it0 + q * Ws) << 7) + (lane << 2);
        live[q] = q == 0 || (q < npk && it0 + q * Ws < nit);  // (packet 0: the loop condition)
      }
      bool p[NR];
#pragma unroll
      for (int q = 0; q < NPMAX; q++)
#pragma unroll
        for (int j = 0; j < RPL; j++) p[q * RPL + j] = live[q] && r0q[q] + j < n;
      // A4 selection: predicates on staged columns, 4 rows per lane per packet
      GPL_UNROLL
      for (int f = 0; f < K.nfilt; f++) {
        const Filt& F = K.filt[f];
#pragma unroll
        for (int q = 0; q < NPMAX; q++) {
          if (!live[q]) continue;  // (a packet past the stage must not be read: smem bounds)
          if (K.colw[F.ref] == 4) {
            filt_rows32(F, sb + K.coloff[F.ref] + r0q[q] * 4, p + q * RPL);
          } else {
            long long x[RPL];
            ld_rows(sb + K.coloff[F.ref] + r0q[q] * K.colw[F.ref], K.colw[F.ref], x);
#pragma unroll
            for (int j = 0; j < RPL; j++) p[q * RPL + j] = p[q * RPL + j] && filt_pass(F, x[j]);
          }
        }
        // per-lane pass count, reduced once after the last stage (the last stage-phase
        // operator is counted by the compaction instead: its survivors are the queued rows)
        if (!(kQueueCounts && K.nsprobe == 0 && f == K.nfilt - 1)) lc[f] += count_n(p);
      }
      // A5 stage-phase probes (keys from the stage; all NR loads in flight together)
      long long sreg[MAXSP][NR];
#pragma unroll
      for (int sp = 0; sp < MAXSP; sp++) {
#pragma unroll
        for (int j = 0; j < NR; j++) sreg[sp][j] = 0;
        if (sp < K.nsprobe) {
          const Probe& P = K.probe[sp];
          // (with no operator before it every row of a live packet is active)
          if ((sp == 0 && K.nfilt == 0) || __any_sync(0xffffffffu, any_n(p))) {
            unsigned long long k[NR];
#pragma unroll
            for (int q = 0; q < NPMAX; q++) {
              uint32_t k1[RPL];
              if (live[q]) {
                ld_key32(d, K, P.k1, sb, r0q[q], rowbase, p + q * RPL, k1);
              } else {
#pragma unroll
                for (int j = 0; j < RPL; j++) k1[j] = 0u;
              }
#pragma unroll
              for (int j = 0; j < RPL; j++) k[q * RPL + j] = k1[j];
              if (P.k2 >= 0 && live[q]) {
                uint32_t k2[RPL];
                ld_key32(d, K, P.k2, sb, r0q[q], rowbase, p + q * RPL, k2);
#pragma unroll
                for (int j = 0; j < RPL; j++) k[q * RPL + j] = (k[q * RPL + j] << 32) | k2[j];
              }
            }
            bool hit[NR];
            long long v[NR];
            if (sp == K.cl_probe && cl_size > 0)
              probe_rows_cl<NR>(K, GPL_SP_HTP(sp), P.ht, k, p, hit, v, sb + (uint32_t)K.cl_off, cl_k0, cl_ncells);
            else
              probe_rows<NR>(K, GPL_SP_HTP(sp), P.ht, k, p, hit, v);
#pragma unroll
            for (int j = 0; j < NR; j++) {
              if (P.kind == P_MARK) {
                sreg[sp][j] = hit[j] ? 1 : 0;
              } else {
                sreg[sp][j] = v[j];
                p[j] = hit[j];
              }
            }
          }
          if (!(kQueueCounts && sp == K.nsprobe - 1)) lc[K.nfilt + sp] += count_n(p);
        }
      }
      if ((K.sink == SINK_PCOUNT || K.sink == SINK_PSCATTER) && K.ins_kcol >= 0) {
        // partition phase (NEXT-4 partitioned hash join): the rows that
        // passed the segment's operators go to their key range's partition
        unsigned* pc = &S<unsigned>(K.off_agg);
#pragma unroll
        for (int q = 0; q < NPMAX; q++) {
          if (!live[q]) continue;
          uint32_t k4[RPL];
          ld_key32(d, K, K.ins_kcol, sb, r0q[q], rowbase, p + q * RPL, k4);
#pragma unroll
          for (int j = 0; j < RPL; j++) {
            const uint32_t pid = (uint32_t)((long long)(int32_t)k4[j] - d.part_kmin) >> K.part_shift;
            const bool in = p[q * RPL + j] && (long long)(int32_t)k4[j] >= d.part_kmin && pid < (uint32_t)K.nparts;
            if (!in) continue;
            if (K.sink == SINK_PCOUNT) {
              atomicAdd(pc + pid, 1u);
            } else {
              const unsigned pos = atomicAdd(pc + pid, 1u);
              d.part_key_out[pos] = (int)k4[j];
              d.part_row_out[pos] = (int)(d.part_row0 + rowbase + r0q[q] + j);
            }
          }
        }
#pragma unroll
        for (int q = 0; q < NPMAX; q++)
          if (live[q] && it0 + q * Ws + Ws >= nit) {
            __syncwarp();
            if (lane == 0) mbar_arrive(&empty[slot]);
            released = true;
          }
        continue;
      }
      if (K.sink == SINK_INSERT && K.ins_q && K.ins_dense) {
        // dense build with a queue-phase insert: zero-fill every live packet's
        // cell range now; the drain writes the cells of the rows that survive
#pragma unroll
        for (int q = 0; q < NPMAX; q++)
          if (live[q]) dense_zero_fill(d, K, sb, (it0 + q * Ws) << 7, n, ins_knext, lane);
        __syncwarp();  // the zero fill is ordered before this warp's drains
      }
      if (K.sink == SINK_INSERT && K.ins_kcol >= 0 && !K.ins_q) {
        // build segment with every probe in the stage phase: insert straight
        // from the staged tile (no survivor queue), all rows' atomics in flight
        long long kx[NR], px[NR];
#pragma unroll
        for (int q = 0; q < NPMAX; q++) {
          long long k4[RPL], p4[RPL];
          if (live[q]) {
            ld_rows(sb + K.coloff[K.ins_kcol] + r0q[q] * K.colw[K.ins_kcol], K.colw[K.ins_kcol], k4);
            if (K.ins_pcol >= 0) ld_rows(sb + K.coloff[K.ins_pcol] + r0q[q] * K.colw[K.ins_pcol], K.colw[K.ins_pcol], p4);
          } else {
#pragma unroll
            for (int j = 0; j < RPL; j++) k4[j] = p4[j] = 0;
          }
#pragma unroll
          for (int j = 0; j < RPL; j++) {
            kx[q * RPL + j] = k4[j];
            px[q * RPL + j] = K.ins_pcol >= 0 ? p4[j]
                              : K.ins_psreg == 0 ? sreg[0][q * RPL + j] : K.ins_psreg == 1 ? sreg[1][q * RPL + j] : 0;
          }
        }
        if (K.ins_dense) {
          // clustered (dense) build: the packet owns the cells from its first
          // row's key to the next packet's first key (the next stage's, at a
          // stage end); it zero-fills that range (aligned 16-B stores, byte
          // stores at the edges it shares with its neighbours) and then writes
          // the cells of its qualifying rows. The key column is strictly
          // increasing (checked at load), so no key repeats and every cell of
          // the domain is written exactly once per build: no atomics, no clear
          // pass, no duplicate check.
#pragma unroll
          for (int q = 0; q < NPMAX; q++) {
            if (!live[q]) continue;
            long long c0, c1;
            dense_zero_fill(d, K, sb, (it0 + q * Ws) << 7, n, ins_knext, lane, &c0, &c1);
            const int w = K.ins_width;
            char* cells = (char*)d.ins_slots;
            __syncwarp();  // the zero fill is ordered before the cells below (same warp)
            if (w == W_NIBBLE) {
              // 4-bit cells: the row of a byte's even cell writes the whole byte
              // (its value | the next row's when that row holds the odd cell),
              // the row of an odd cell only when the even cell has no row; the
              // two bytes shared with the neighbouring packets take atomics
              long long c[RPL];
              uint32_t v[RPL];
              bool ok[RPL];
#pragma unroll
              for (int j = 0; j < RPL; j++) {
                ok[j] = r0q[q] + j < n;
                c[j] = kx[q * RPL + j] - d.ins_kmin;
                long long pv = px[q * RPL + j];
                if (K.ins_ptransform == G_YEAR) pv = (int)pv / 10000;
                v[j] = p[q * RPL + j] ? (uint32_t)(pv - d.ins_pay_base + 1) & 0xFu : 0u;
              }
              const long long cn = __shfl_down_sync(0xffffffffu, c[0], 1), cp = __shfl_up_sync(0xffffffffu, c[RPL - 1], 1);
              const uint32_t vn = __shfl_down_sync(0xffffffffu, v[0], 1);
              const bool okn = __shfl_down_sync(0xffffffffu, ok[0], 1) && lane < 31;
              const bool okp = __shfl_up_sync(0xffffffffu, ok[RPL - 1], 1) && lane > 0;
#pragma unroll
              for (int j = 0; j < RPL; j++) {
                if (!ok[j]) continue;
                const long long cj = c[j];
                if ((cj & 1) == 0) {
                  if (cj + 1 == c1) {
                    nibble_or(cells, cj, v[j]);  // shared with the next packet
                  } else {
                    const bool hn = j < RPL - 1 ? ok[j + 1] && c[j + 1] == cj + 1 : okn && cn == cj + 1;
                    const uint32_t b = v[j] | ((hn ? (j < RPL - 1 ? v[j + 1] : vn) : 0u) << 4);
                    if (b) cells[cj >> 1] = (char)b;
                  }
                } else if (cj == c0) {
                  nibble_or(cells, cj, v[j]);  // shared with the previous packet
                } else {
                  const bool hp = j > 0 ? c[j - 1] == cj - 1 : okp && cp == cj - 1;
                  if (!hp && v[j]) cells[cj >> 1] = (char)(v[j] << 4);
                }
              }
              continue;
            }
#pragma unroll
            for (int j = 0; j < RPL; j++) {
              if (!p[q * RPL + j]) continue;
              long long pv = px[q * RPL + j];
              if (K.ins_ptransform == G_YEAR) pv = (int)pv / 10000;
              const uint32_t v = (uint32_t)(pv - d.ins_pay_base + 1);
              const long long c = kx[q * RPL + j] - d.ins_kmin;
              if (w == 1) cells[c] = (char)v;
              else if (w == 2) ((unsigned short*)cells)[c] = (unsigned short)v;
              else ((uint32_t*)cells)[c] = v;
            }
          }
        }
        // the ring slot is no longer read: release it before the atomics' round trip
#pragma unroll
        for (int q = 0; q < NPMAX; q++)
          if (live[q] && it0 + q * Ws + Ws >= nit) {
            __syncwarp();
            if (lane == 0) mbar_arrive(&empty[slot]);
            released = true;
          }
        if (!K.ins_dense) insert_cells<NR>(d, K, kx, px, p);
        continue;
      }
      // A8 compaction into the warp's survivor queue (the on-chip channel), packet by packet
#pragma unroll
      for (int q = 0; q < NPMAX; q++) {
        if (!live[q]) break;
        const int r0 = r0q[q];
        int base = qcount;
        int pos[RPL];
        // a packet with no survivor (most packets of a selective stage phase:
        // Q9's 0.005%) skips the per-row ballots with one vote
        const bool any_q = __any_sync(0xffffffffu, p[q * RPL] | p[q * RPL + 1] | p[q * RPL + 2] | p[q * RPL + 3]);
        if (any_q) {
#pragma unroll
        for (int j = 0; j < RPL; j++) {
          const unsigned m = __ballot_sync(0xffffffffu, p[q * RPL + j]);
          pos[j] = (qhead + base + __popc(m & lanemask_lt())) & (QCAP - 1);
          base += __popc(m);
        }
        queued += (unsigned)(base - qcount);
        }
        if (base != qcount) {
          uint32_t ra4[RPL], ra8[RPL];  // a queued row's entry: queue base + position x width
          {
            const uint32_t qs = smem_base() + qb;
#pragma unroll
            for (int j = 0; j < RPL; j++) {
              ra4[j] = qs + (uint32_t)pos[j] * 4u;
              ra8[j] = qs + (uint32_t)pos[j] * 8u;
            }
          }
          // late materialisation: when the queue is entered straight after the filters
          // (scattered survivors, e.g. Q14's date window), the lazy columns the drain
          // gathers first are prefetched into L2 as their rows are queued, so the drain's
          // dependent gather is an L2 hit, not an HBM round trip (measured: Q14 SF 100
          // 0.79 -> 0.69 ms; after a clustered probe the survivors share sectors and the
          // prefetch only costs instructions, so it is off there)
          if (K.rowid_field >= 0 && K.push[K.rowid_field].kind == PUSH_ROWID && K.nsprobe == 0 && K.nfilt > 0) {
            GPL_UNROLL
            for (int f = 0; f < K.nfield; f++) {
              const int c = K.qlazy[f];
              if (c < 0 || K.qlazy_at[f] != K.nsprobe) continue;
#pragma unroll
              for (int j = 0; j < RPL; j++)
                if (p[q * RPL + j])
                  asm volatile("prefetch.global.L2 [%0];" ::"l"(d.col[c] + (rowbase + r0 + j) * K.colw[c]));
            }
          }
          GPL_UNROLL
          for (int e = 0; e < K.npush; e++) {
            const Push& E = K.push[e];
            const uint32_t qa = qb + K.qoff[e];
            long long v[RPL];
            if (E.kind == PUSH_COL) {
              ld_col(d, K, E.src, sb, r0, rowbase, p + q * RPL, v);
            } else if (E.kind == PUSH_ROWID) {  // for the drain's lazy-column gather
#pragma unroll
              for (int j = 0; j < RPL; j++) v[j] = rowbase + r0 + j;
            } else if (E.kind == PUSH_SREG) {
#pragma unroll
              for (int j = 0; j < RPL; j++) v[j] = E.src == 0 ? sreg[0][q * RPL + j] : sreg[1][q * RPL + j];
            } else {  // pushed-down value term: sign * prod(a + b * x)
              const Term& T = K.sterm[E.src];
#pragma unroll
              for (int j = 0; j < RPL; j++) v[j] = T.sign;
              GPL_UNROLL
              for (int f = 0; f < T.nfact; f++) {
                const Factor& F = T.f[f];
                long long x[RPL];
                if (F.field >= 0) {
                  ld_col(d, K, F.field, sb, r0, rowbase, p + q * RPL, x);
                } else {
#pragma unroll
                  for (int j = 0; j < RPL; j++)
                    x[j] = F.field == SREF_CONST ? 0 : (F.field == -2 ? sreg[0][q * RPL + j] : sreg[1][q * RPL + j]);
                }
#pragma unroll
                for (int j = 0; j < RPL; j++) v[j] *= F.a + (long long)F.b * x[j];
              }
            }
            // (row addresses computed once per packet; the field offset is a
            // compile-time immediate of the store in the plan-specialised kernel)
            (void)qa;
            if (K.qw[e] == 4) {
#pragma unroll
              for (int j = 0; j < RPL; j++)
                if (p[q * RPL + j]) sts_32(ra4[j] + (uint32_t)K.qoff[e], (int)v[j]);
            } else {
#pragma unroll
              for (int j = 0; j < RPL; j++)
                if (p[q * RPL + j]) sts_64(ra8[j] + (uint32_t)K.qoff[e], v[j]);
            }
          }
          qcount = base;
        }
        if (it0 + q * Ws + Ws >= nit) {
          // the warp's last packet of this stage is in the queue: release the
          // ring slot BEFORE draining (the drain reads only the queue), so the
          // producer's next copy overlaps the drain's probe/insert latency
          __syncwarp();
          if (lane == 0) mbar_arrive(&empty[slot]);
          released = true;
        }
        if (qcount >= RPL * 32) {
          __syncwarp();
          if (K.ndrain > 0) hand_off(qhead, RPL * 32);
          else drain(d, qb, qhead, RPL * 32, cnt, acc, lane);
          __syncwarp();
          qhead = (qhead + RPL * 32) & (QCAP - 1);
          qcount -= RPL * 32;
        }
      }
    }
    if (!released) {
      __syncwarp();
      if (lane == 0) mbar_arrive(&empty[slot]);
    }
    if (K.flush_each_tile && h.w) flush_reg(d, acc, lane);
    if (++slot == (uint32_t)K.depth) { slot = 0; phase ^= 1u; }
  }
  GPL_UNROLL
  for (int op = 0; op < K.nfilt + K.nsprobe; op++) {
    if (kQueueCounts && op == K.nfilt + K.nsprobe - 1) {
      if (lane == 0) cnt[op] += queued;
      continue;
    }
    const unsigned c = __reduce_add_sync(0xffffffffu, lc[op]);
    if (lane == 0) cnt[op] += c;
  }
  if (qcount > 0) {
    __syncwarp();
    if (K.ndrain > 0) hand_off(qhead, qcount);
    else drain(d, qb, qhead, qcount, cnt, acc, lane);
  }
  if (K.ndrain > 0) {  // the last stage warp to finish sends one end token per drain warp
    unsigned done = 0;
    if (lane == 0) done = atomicAdd(&S<unsigned>(kOffHTick + 8), 1u);
    done = __shfl_sync(0xffffffffu, done, 0);
    if (done == (unsigned)(Ws - 1))
      for (int e = 0; e < K.ndrain; e++) hand_off(0, -1);
  }
  }  // stage warps
  __syncwarp();
  if (K.agg_mode == AGG_REG) flush_reg(d, acc, lane);
  if (lane == 0) {
    const int nops = K.nfilt + K.nprobe + K.nresid;
    for (int o = 0; o < nops; o++)
      if (cnt[o]) atomicAdd(d.op_pass + o, cnt[o]);
  }
  if (K.sink == SINK_PCOUNT) {  // this CTA's count of every partition (partition-major for the scan)
    named_bar_sync(1, (uint32_t)W * 32u);
    const unsigned* pc = &S<unsigned>(K.off_agg);
    for (int i = threadIdx.x; i < K.nparts; i += W * 32) d.part_hist[(size_t)i * gridDim.x + blockIdx.x] = pc[i];
  }
  if (K.agg_mode == AGG_SMEM && K.sink == SINK_AGG) {
    named_bar_sync(1, (uint32_t)W * 32u);
    const int L = K.agg_lanes, words = K.ngroups_total * K.nagg * L;
    const unsigned* lo = &S<unsigned>(K.off_agg);
    for (int i = threadIdx.x; i < K.ngroups_total * K.nagg; i += W * 32) {
      unsigned long long t = 0;  // the copies' sum mod 2^64
      for (int l = 0; l < L; l++)
        t += (unsigned long long)lo[i * L + l] | ((unsigned long long)lo[words + i * L + l] << 32);
      if (t != 0) atomic_add_i128(d.partials + 2 * i, (long long)t);
    }
  }
}

}  // namespace pipe
}  // namespace gpl
