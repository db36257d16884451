// device_common.cuh — device helpers shared by the build, pipeline and KBE
// kernels: hash-table addressing/probing, exact int128 accumulation, PTX
// wrappers for mbarrier / bulk-async copies / L2 cache policies (sm_90+, used
// here for sm_100a).
#pragma once
#ifndef __CUDACC_RTC__
#include <cstdint>
#endif

#include "common.h"

namespace gpl {

// ---------------------------------------------------------------- hash tables
// Per-kernel copy of a table's parameters (from HTRef + its device header).
struct HTP {
  const void* slots;
  unsigned long long kmin, mult;  // hashed: ordered-hash base/multiplier; DIRECT: key base
  unsigned long long nslots;      // DIRECT cells
  long long pay_base;             // DIRECT payload base
  uint32_t mask, shift;
  int32_t kind, hash, width, pad;
  const void* pay;                // MULTI payload array
};

__device__ __forceinline__ HTP load_htp(const HTRef& r) {
  HTP p;
  p.slots = r.slots;
  p.kind = r.kind;
  p.hash = r.hash;
  p.width = r.width;
  p.pad = 0;
  p.pay = r.pay;
  if (r.kind == HT_DIRECT || r.kind == HT_MULTI) {
    p.kmin = (unsigned long long)r.kmin;
    p.nslots = r.nslots;
    p.pay_base = r.pay_base;
    p.mult = 0;
    p.mask = 0;
    p.shift = 0;
    return p;
  }
  const HTHeader* h = r.hdr;
  p.mask = h->mask;
  const uint32_t log2 = h->log2;
  p.shift = (r.kind == HT_MAP64 ? 64u : 32u) - log2;
  p.kmin = (unsigned long long)h->kmin;
  p.mult = h->mult;
  p.nslots = 0;
  p.pay_base = 0;
  return p;
}

// DIRECT probe: one load, no chain. key is the int32 key zero-extended.
__device__ __forceinline__ bool direct_probe(const HTP& h, unsigned long long key, long long* payload) {
  const unsigned long long idx = (unsigned long long)((long long)(int32_t)(uint32_t)key - (long long)h.kmin);
  if (idx >= h.nslots) return false;
  if (h.width == 0) {
    const uint32_t w = __ldg((const uint32_t*)h.slots + (idx >> 5));
    *payload = 1;
    return (w >> (idx & 31)) & 1u;
  }
  uint32_t v;
  if (h.width == W_NIBBLE) v = ((uint32_t)__ldg((const unsigned char*)h.slots + (idx >> 1)) >> ((idx & 1) * 4)) & 0xFu;
  else if (h.width == 1) v = __ldg((const unsigned char*)h.slots + idx);
  else if (h.width == 2) v = __ldg((const unsigned short*)h.slots + idx);
  else v = __ldg((const uint32_t*)h.slots + idx);
  *payload = (long long)v - 1 + h.pay_base;
  return v != 0;
}

// Home slot. MULT: Fibonacci (multiplicative) hashing on the high bits.
// ORDERED: monotone range scaling, so keys arriving in order (lineitem is
// clustered by orderkey) touch consecutive slots.
__device__ __forceinline__ uint32_t ht_home(const HTP& h, unsigned long long key) {
  if (h.hash == H_ORDERED) return (uint32_t)(((key - h.kmin) * h.mult) >> 32) & h.mask;
  if (h.kind == HT_MAP64) return (uint32_t)((key * 0x9E3779B97F4A7C15ull) >> h.shift);
  return ((uint32_t)key * 0x9E3779B1u) >> h.shift;
}

// Linear probing. Returns true on hit; MAP kinds also return the payload.
__device__ __forceinline__ bool ht_probe(const HTP& h, unsigned long long key, long long* payload) {
  if (h.kind == HT_DIRECT) return direct_probe(h, key, payload);
  uint32_t i = ht_home(h, key);
  if (h.kind == HT_MAP32) {
    if ((uint32_t)key == EMPTY32) return false;
    const unsigned long long* s = (const unsigned long long*)h.slots;
    for (;;) {
      const unsigned long long v = __ldg(s + i);
      const uint32_t k = (uint32_t)v;
      if (k == (uint32_t)key) { *payload = (long long)(int32_t)(uint32_t)(v >> 32); return true; }
      if (k == EMPTY32) return false;
      i = (i + 1) & h.mask;
    }
  } else if (h.kind == HT_SET32) {
    if ((uint32_t)key == EMPTY32) return false;
    const uint32_t* s = (const uint32_t*)h.slots;
    for (;;) {
      const uint32_t k = __ldg(s + i);
      if (k == (uint32_t)key) { *payload = 1; return true; }
      if (k == EMPTY32) return false;
      i = (i + 1) & h.mask;
    }
  } else {
    if (key == EMPTY64) return false;
    const ulonglong2* s = (const ulonglong2*)h.slots;
    for (;;) {
      const ulonglong2 v = __ldg(s + i);
      if (v.x == key) { *payload = (long long)v.y; return true; }
      if (v.x == EMPTY64) return false;
      i = (i + 1) & h.mask;
    }
  }
}

// Probe R keys of one lane with their loads in flight together (ILP): each
// round issues one slot load per still-active row, then resolves them.
// `kind` and `width` are passed separately so that a plan-specialised (JIT)
// kernel sees them as compile-time constants.
template <int R>
__device__ __forceinline__ void ht_probe_n(const HTP& h, const int kind, const int width,
                                           const unsigned long long (&key)[R], const bool (&act)[R], bool (&hit)[R],
                                           long long (&pay)[R]) {
  if (kind == HT_DIRECT) {  // one load per row; dispatch on the cell width once
    unsigned long long idx[R];
    bool in[R];
#pragma unroll
    for (int j = 0; j < R; j++) {
      idx[j] = (unsigned long long)((long long)(int32_t)(uint32_t)key[j] - (long long)h.kmin);
      in[j] = act[j] && idx[j] < h.nslots;
    }
    uint32_t v[R];
    if (width == 0) {
#pragma unroll
      for (int j = 0; j < R; j++) v[j] = in[j] ? (__ldg((const uint32_t*)h.slots + (idx[j] >> 5)) >> (idx[j] & 31)) & 1u : 0u;
#pragma unroll
      for (int j = 0; j < R; j++) { hit[j] = v[j] != 0; pay[j] = 1; }
      return;
    }
    if (width == W_NIBBLE) {
#pragma unroll
      for (int j = 0; j < R; j++)
        v[j] = in[j] ? ((uint32_t)__ldg((const unsigned char*)h.slots + (idx[j] >> 1)) >> ((idx[j] & 1) * 4)) & 0xFu : 0u;
    } else if (width == 1) {
#pragma unroll
      for (int j = 0; j < R; j++) v[j] = in[j] ? (uint32_t)__ldg((const unsigned char*)h.slots + idx[j]) : 0u;
    } else if (width == 2) {
#pragma unroll
      for (int j = 0; j < R; j++) v[j] = in[j] ? (uint32_t)__ldg((const unsigned short*)h.slots + idx[j]) : 0u;
    } else {
#pragma unroll
      for (int j = 0; j < R; j++) v[j] = in[j] ? __ldg((const uint32_t*)h.slots + idx[j]) : 0u;
    }
#pragma unroll
    for (int j = 0; j < R; j++) {
      hit[j] = v[j] != 0;
      pay[j] = (long long)v[j] - 1 + h.pay_base;
    }
    return;
  }
  uint32_t pos[R];
  bool live[R];
  bool any = false;
#pragma unroll
  for (int j = 0; j < R; j++) {
    hit[j] = false;
    pay[j] = 0;
    live[j] = act[j] && (kind == HT_MAP64 ? key[j] != EMPTY64 : (uint32_t)key[j] != EMPTY32);
    pos[j] = ht_home(h, key[j]);
    any |= live[j];
  }
  if (kind == HT_MAP32) {
    const unsigned long long* s = (const unsigned long long*)h.slots;
    while (any) {
      unsigned long long v[R];
#pragma unroll
      for (int j = 0; j < R; j++) v[j] = live[j] ? __ldg(s + pos[j]) : 0ull;
      any = false;
#pragma unroll
      for (int j = 0; j < R; j++) {
        if (!live[j]) continue;
        const uint32_t k = (uint32_t)v[j];
        if (k == (uint32_t)key[j]) { hit[j] = true; pay[j] = (long long)(int32_t)(uint32_t)(v[j] >> 32); live[j] = false; }
        else if (k == EMPTY32) live[j] = false;
        else { pos[j] = (pos[j] + 1) & h.mask; any = true; }
      }
    }
  } else if (kind == HT_SET32) {
    const uint32_t* s = (const uint32_t*)h.slots;
    while (any) {
      uint32_t v[R];
#pragma unroll
      for (int j = 0; j < R; j++) v[j] = live[j] ? __ldg(s + pos[j]) : 0u;
      any = false;
#pragma unroll
      for (int j = 0; j < R; j++) {
        if (!live[j]) continue;
        if (v[j] == (uint32_t)key[j]) { hit[j] = true; pay[j] = 1; live[j] = false; }
        else if (v[j] == EMPTY32) live[j] = false;
        else { pos[j] = (pos[j] + 1) & h.mask; any = true; }
      }
    }
  } else {
    const ulonglong2* s = (const ulonglong2*)h.slots;
    while (any) {
      ulonglong2 v[R];
#pragma unroll
      for (int j = 0; j < R; j++) v[j] = live[j] ? __ldg(s + pos[j]) : make_ulonglong2(0ull, 0ull);
      any = false;
#pragma unroll
      for (int j = 0; j < R; j++) {
        if (!live[j]) continue;
        if (v[j].x == key[j]) { hit[j] = true; pay[j] = (long long)v[j].y; live[j] = false; }
        else if (v[j].x == EMPTY64) live[j] = false;
        else { pos[j] = (pos[j] + 1) & h.mask; any = true; }
      }
    }
  }
}

// ------------------------------------------------------------ exact int128
// p[0] = low word, p[1] = high word (two's complement). Adds a signed int64.
// Correct under concurrency: the low word wraps exactly once per carry seen
// by the atomic that caused it.
// 64-bit atomics on GLOBAL memory spelled out (a generic-address atomicAdd
// also compiles a shared-memory CAS-loop branch that never runs here).
__device__ __forceinline__ unsigned long long gatom_add_u64(unsigned long long* p, unsigned long long v) {
  unsigned long long old;
  asm volatile("atom.global.add.u64 %0, [%1], %2;" : "=l"(old) : "l"(p), "l"(v) : "memory");
  return old;
}
__device__ __forceinline__ void gred_add_u64(unsigned long long* p, unsigned long long v) {
  asm volatile("red.global.add.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

__device__ __forceinline__ void atomic_add_i128(unsigned long long* p, long long v) {
  const unsigned long long lo = (unsigned long long)v;
  const unsigned long long old = gatom_add_u64(p, lo);
  const unsigned long long carry = (old + lo) < old ? 1ull : 0ull;
  const unsigned long long hi = (v < 0 ? ~0ull : 0ull) + carry;
  if (hi) gred_add_u64(p + 1, hi);
}

// The 128-bit sum of the lanes' int64 values (exact at any magnitude), and its
// atomic addition into an int128 counter {lo, hi}.
__device__ __forceinline__ void warp_sum_i128(long long v, unsigned long long& lo, long long& hi) {
  lo = (unsigned long long)v;
  hi = v < 0 ? -1ll : 0ll;
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    const unsigned long long l2 = __shfl_xor_sync(0xffffffffu, lo, o);
    const long long h2 = __shfl_xor_sync(0xffffffffu, hi, o);
    const unsigned long long s = lo + l2;
    hi += h2 + (s < lo ? 1ll : 0ll);
    lo = s;
  }
}
__device__ __forceinline__ void atomic_add_i128_wide(unsigned long long* p, unsigned long long lo, long long hi) {
  const unsigned long long old = gatom_add_u64(p, lo);
  const unsigned long long h = (unsigned long long)hi + ((old + lo) < old ? 1ull : 0ull);
  if (h) gred_add_u64(p + 1, h);
}

__device__ __forceinline__ long long warp_sum_i64(long long v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}

// ------------------------------------------------------------- PTX wrappers
__device__ __forceinline__ uint32_t smem_addr(const void* p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(unsigned long long* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_addr(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_mbar_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void fence_proxy_async_smem() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(unsigned long long* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_addr(bar)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_arrive(unsigned long long* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_addr(bar)) : "memory");
}
__device__ __forceinline__ void mbar_wait(unsigned long long* bar, uint32_t parity) {
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "GPL_WAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      "@!p bra GPL_WAIT_%=;\n"
      "}\n" ::"r"(smem_addr(bar)),
      "r"(parity)
      : "memory");
}
// 1-D bulk async copy global -> shared (TMA engine), completes on `bar` by
// transaction bytes; L2 cache hint `policy`.
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, unsigned long long* bar,
                                         unsigned long long policy) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;" ::"r"(
          smem_addr(dst)),
      "l"(src), "r"(bytes), "r"(smem_addr(bar)), "l"(policy)
      : "memory");
}
__device__ __forceinline__ unsigned long long policy_evict_last() {
  unsigned long long p;
  asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ unsigned long long policy_evict_first() {
  unsigned long long p;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}
// Programmatic dependent launch: a kernel launched with programmatic stream
// serialization may start while its predecessor drains; it must wait here
// before touching anything the predecessor writes (a no-op otherwise).
__device__ __forceinline__ void grid_dep_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
// Allow the next kernel in the stream to be scheduled (it still waits in
// grid_dep_wait for this grid's completion and memory flush).
__device__ __forceinline__ void grid_dep_launch_dependents() {
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
}
__device__ __forceinline__ void named_bar_sync(uint32_t id, uint32_t nthreads) {
  asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(nthreads) : "memory");
}

// Typed column read (4- or 8-byte column) widened to int64.
__device__ __forceinline__ long long ld_col_global(const char* base, int w, long long row) {
  return w == 4 ? (long long)__ldg((const int*)base + row) : __ldg((const long long*)base + row);
}

__device__ __forceinline__ bool filt_pass(const Filt& f, long long x) {
  if (f.kind == F_RANGE) return x >= f.lo && x <= f.hi;
  if (f.kind == F_MASK) return (unsigned long long)x < 64ull && ((f.mask >> x) & 1ull);
  return x != f.lo;
}

}  // namespace gpl
