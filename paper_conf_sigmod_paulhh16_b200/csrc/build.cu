// build.cu — A1 build segment: scan a build relation through its filters and
// probes into earlier hash tables, then insert key -> payload into an
// open-addressing, linear-probing, power-of-two table (load <= load_pct).
//
// Paper: "We implement the simple hash join with two phases, i.e., hash build
// and hash probe ... it requires a blocking barrier after hash build"
// (§3.2). The barrier is stream order: every later segment is
// enqueued after this one. Hash tables are the only materialised segment
// output.
//
// Sizing is exact and stays on the device: a count pass accumulates the
// number of qualifying rows and their key range into the table's header; its
// last block computes nslots = next_pow2(count * 100 / load_pct) and the
// ordered-hash multiplier. The clear and insert kernels read the header, so
// the whole build is asynchronous (no host round trip).
#include <algorithm>
#include <climits>

#include <cub/cub.cuh>

#include "device_common.cuh"
#include "kernels.h"

namespace gpl {
namespace {

constexpr int kThreads = 256;

// Evaluate BR consecutive build rows at once (row0 % BR == 0): filters,
// probes into earlier tables (a miss drops the row: inner / semi join), key
// and payload. The filter columns are read with one 16-B vector load per
// BR = 4 rows and every probe of the BR rows is issued before any is needed,
// so one thread keeps BR independent memory round trips in flight (the build
// is latency-bound otherwise). Rows past nrows read the zero padding of the
// column store (64-row padded copies; borrowed columns hold >= 4-row multiples).
// Measured on B200 (Q5 SF1 builds): BR = 1 with one row per thread is faster
// than BR = 4 (5.4/19.7/5.0 us vs 9.0/25.6/8.7 us): the per-row chains are
// predicated control flow that does not overlap, and fewer threads are
// resident. Kept selectable for experiments.
#ifndef GPL_BUILD_BR
#define GPL_BUILD_BR 1
#endif
constexpr int BR = GPL_BUILD_BR;
__device__ __forceinline__ void ld4_global(const char* col, int w, long long row0, long long (&x)[BR]) {
  if (BR != 4) {
#pragma unroll
    for (int j = 0; j < BR; j++) x[j] = ld_col_global(col, w, row0 + j);
  } else if (w == 4) {
    const int4 v = __ldg((const int4*)col + (row0 >> 2));
    x[0] = v.x; x[1] = v.y; x[2] = v.z; x[3] = v.w;
  } else {
    const longlong2 a = __ldg((const longlong2*)col + (row0 >> 1));
    const longlong2 b = __ldg((const longlong2*)col + (row0 >> 1) + 1);
    x[0] = a.x; x[1] = a.y; x[2] = b.x; x[3] = b.y;
  }
}
__device__ __forceinline__ void build_rows(const BuildDesc& d, const HTP* src, long long row0, long long stride,
                                           bool (&ok)[BR], unsigned long long (&key)[BR], long long (&pay)[BR]) {
  (void)stride;
#pragma unroll
  for (int j = 0; j < BR; j++) ok[j] = row0 + j < d.nrows;
  for (int f = 0; f < d.nfilt; f++) {
    const Filt& F = d.filt[f];
    long long x[BR];
    ld4_global(d.col[F.ref], d.colw[F.ref], row0, x);
#pragma unroll
    for (int j = 0; j < BR; j++) ok[j] = ok[j] && filt_pass(F, x[j]);
  }
  long long slot[MAXP][BR];
#pragma unroll
  for (int p = 0; p < MAXP; p++) {
#pragma unroll
    for (int j = 0; j < BR; j++) slot[p][j] = 0;
    if (p < d.nprobe) {
      const Probe& P = d.probe[p];
      unsigned long long k[BR];
#pragma unroll
      for (int j = 0; j < BR; j++) {
        k[j] = ok[j] ? (uint32_t)ld_col_global(d.col[P.k1], d.colw[P.k1], row0 + j) : 0u;
        if (P.k2 >= 0 && ok[j]) k[j] = (k[j] << 32) | (uint32_t)ld_col_global(d.col[P.k2], d.colw[P.k2], row0 + j);
      }
      bool hit[BR];
      long long v[BR];
      const HTP& H = src[P.ht];
      ht_probe_n<BR>(H, H.kind, H.width, k, ok, hit, v);
#pragma unroll
      for (int j = 0; j < BR; j++) {
        ok[j] = ok[j] && hit[j];  // inner / semi: a miss drops the row
        slot[p][j] = v[j];
      }
    }
  }
#pragma unroll
  for (int j = 0; j < BR; j++) {
    const long long row = row0 + j;
    key[j] = 0;
    pay[j] = 0;
    if (!ok[j]) continue;
    unsigned long long k = (uint32_t)ld_col_global(d.col[d.k1], d.colw[d.k1], row);
    if (d.k2 >= 0) k = (k << 32) | (uint32_t)ld_col_global(d.col[d.k2], d.colw[d.k2], row);
    key[j] = k;
    if (d.pay_kind == PAY_COL) pay[j] = ld_col_global(d.col[d.pay_ref], d.colw[d.pay_ref], row);
    else if (d.pay_kind == PAY_YEARCOL) pay[j] = (int)ld_col_global(d.col[d.pay_ref], d.colw[d.pay_ref], row) / 10000;
    else if (d.pay_kind == PAY_SLOT) {
      long long s = slot[0][j];
#pragma unroll
      for (int p = 1; p < MAXP; p++) s = d.pay_ref == p ? slot[p][j] : s;
      pay[j] = s;
    }
  }
}

__device__ __forceinline__ void finalize_header(HTHeader* h, unsigned long long count, long long kmin,
                                                long long kmax, long long cap_slots, int load_pct) {
  unsigned long long need = (count * 100ull + (unsigned long long)load_pct - 1) / (unsigned long long)load_pct;
  uint32_t log2 = 4;
  while ((1ull << log2) < need) log2++;
  while ((1ll << log2) > cap_slots && log2 > 4) log2--;
  const unsigned long long nslots = 1ull << log2;
  if (count == 0) { kmin = 0; kmax = 0; }
  const unsigned long long range = (unsigned long long)(kmax - kmin) + 1ull;
  h->count = count;
  h->kmin = kmin;
  h->kmax = kmax;
  h->mult = (nslots << 32) / range;
  h->log2 = log2;
  h->mask = (uint32_t)(nslots - 1);
}

__global__ void header_init_kernel(HTHeader* h) {
  h->acc_count = 0;
  h->acc_kmin = LLONG_MAX;
  h->acc_kmax = LLONG_MIN;
  h->done = 0;
  h->count = 0;
  h->kmin = h->kmax = 0;
  h->mult = 1ull << 32;
  h->log2 = 4;
  h->mask = 15;
}

__global__ void __launch_bounds__(kThreads) build_count_kernel(const __grid_constant__ BuildDesc d) {
  __shared__ HTP src[MAXHT];
  __shared__ unsigned long long s_cnt;
  __shared__ long long s_min, s_max;
  if (threadIdx.x < d.nht) src[threadIdx.x] = load_htp(d.src[threadIdx.x]);
  if (threadIdx.x == 0) { s_cnt = 0; s_min = LLONG_MAX; s_max = LLONG_MIN; }
  __syncthreads();
  unsigned long long cnt = 0;
  long long mn = LLONG_MAX, mx = LLONG_MIN;
  const long long stride = (long long)gridDim.x * blockDim.x;
  for (long long row = ((long long)blockIdx.x * blockDim.x + threadIdx.x) * BR; row < d.nrows; row += stride * BR) {
    bool ok[BR];
    unsigned long long k[BR];
    long long pay[BR];
    build_rows(d, src, row, stride, ok, k, pay);
#pragma unroll
    for (int j = 0; j < BR; j++)
      if (ok[j]) {
        cnt++;
        mn = min(mn, (long long)k[j]);
        mx = max(mx, (long long)k[j]);
      }
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    cnt += __shfl_xor_sync(0xffffffffu, cnt, o);
    mn = min(mn, __shfl_xor_sync(0xffffffffu, mn, o));
    mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, o));
  }
  if ((threadIdx.x & 31) == 0 && cnt) {
    atomicAdd(&s_cnt, cnt);
    atomicMin(&s_min, mn);
    atomicMax(&s_max, mx);
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    HTHeader* h = d.hdr;
    if (s_cnt) {
      atomicAdd(&h->acc_count, s_cnt);
      atomicMin(&h->acc_kmin, s_min);
      atomicMax(&h->acc_kmax, s_max);
    }
    __threadfence();
    const uint32_t prev = atomicAdd(&h->done, 1u);
    if (prev == gridDim.x - 1) {  // last block: publish the exact size
      __threadfence();
      const unsigned long long c = atomicAdd(&h->acc_count, 0ull);
      const long long lo = atomicMin(&h->acc_kmin, LLONG_MAX);
      const long long hi = atomicMax(&h->acc_kmax, LLONG_MIN);
      finalize_header(h, c, lo, hi, d.cap_slots, d.load_pct);
      h->acc_count = 0;
      h->acc_kmin = LLONG_MAX;
      h->acc_kmax = LLONG_MIN;
      h->done = 0;
      __threadfence();
    }
  }
}

__global__ void __launch_bounds__(kThreads) build_clear_kernel(const __grid_constant__ BuildDesc d, int has_known,
                                                                const __grid_constant__ HTHeader known) {
  uint32_t mask;
  if (has_known) {
    mask = known.mask;
    if (blockIdx.x == 0 && threadIdx.x == 0) {
      HTHeader* h = d.hdr;
      h->count = known.count;
      h->kmin = known.kmin;
      h->kmax = known.kmax;
      h->mult = known.mult;
      h->log2 = known.log2;
      h->mask = known.mask;
    }
  } else {
    mask = d.hdr->mask;
  }
  const int slot_bytes = d.kind == HT_SET32 ? 4 : d.kind == HT_MAP32 ? 8 : 16;
  const unsigned long long n16 = ((unsigned long long)mask + 1ull) * slot_bytes / 16ull;
  uint4* p = (uint4*)d.slots;
  const uint4 ones = make_uint4(~0u, ~0u, ~0u, ~0u);
  for (unsigned long long i = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; i < n16;
       i += (unsigned long long)gridDim.x * blockDim.x)
    p[i] = ones;
}

__global__ void __launch_bounds__(kThreads) build_insert_kernel(const __grid_constant__ BuildDesc d) {
  __shared__ HTP src[MAXHT];
  __shared__ HTP dst;
  if (threadIdx.x < d.nht) src[threadIdx.x] = load_htp(d.src[threadIdx.x]);
  if (threadIdx.x == 0 && d.kind != HT_DIRECT) {
    HTRef r{};
    r.slots = d.slots;
    r.hdr = d.hdr;
    r.kind = d.kind;
    r.hash = d.hash;
    dst = load_htp(r);
  }
  __syncthreads();
  const long long stride = (long long)gridDim.x * blockDim.x;
  for (long long row0 = ((long long)blockIdx.x * blockDim.x + threadIdx.x) * BR; row0 < d.nrows; row0 += stride * BR) {
   bool okv[BR];
   unsigned long long keyv[BR];
   long long payv[BR];
   build_rows(d, src, row0, stride, okv, keyv, payv);
   if (d.kind == HT_DIRECT) {
    // one atomic per row, all BR in flight: bitmap / 32-bit cells by
    // atomicOr / atomicCAS; 1- and 2-byte cells by atomicOr into their word
    // (cells start at 0 = empty, so OR sets exactly the cell; a non-zero old
    // cell means a duplicate key)
#pragma unroll
    for (int j = 0; j < BR; j++) {
      if (!okv[j]) continue;
      const unsigned long long idx = (unsigned long long)((long long)(int32_t)(uint32_t)keyv[j] - d.kmin);
      if (idx >= d.nslots) { atomicOr(d.err, ERR_CAPACITY); continue; }
      if (d.width == 0) {
        const uint32_t bit = 1u << (idx & 31);
        if (atomicOr((uint32_t*)d.slots + (idx >> 5), bit) & bit) atomicOr(d.err, ERR_DUPKEY);
      } else {
        const uint32_t v = (uint32_t)(payv[j] - d.pay_base + 1);
        if (d.width == 4) {
          if (atomicCAS((uint32_t*)d.slots + idx, 0u, v) != 0u) atomicOr(d.err, ERR_DUPKEY);
        } else if (d.width == W_NIBBLE) {
          const unsigned long long byte = idx >> 1;
          uint32_t* w = (uint32_t*)((char*)d.slots + (byte & ~3ull));
          const uint32_t sh = (uint32_t)(byte & 3ull) * 8u + (uint32_t)(idx & 1ull) * 4u;
          if (atomicOr(w, v << sh) & (0xFu << sh)) atomicOr(d.err, ERR_DUPKEY);
        } else {
          const unsigned long long byte = idx * (unsigned long long)d.width;
          uint32_t* w = (uint32_t*)((char*)d.slots + (byte & ~3ull));
          const uint32_t sh = (uint32_t)(byte & 3ull) * 8u;
          const uint32_t m = (d.width == 1 ? 0xFFu : 0xFFFFu) << sh;
          if (atomicOr(w, v << sh) & m) atomicOr(d.err, ERR_DUPKEY);
        }
      }
    }
    continue;
   }
   for (int j = 0; j < BR; j++) {
    if (!okv[j]) continue;
    const unsigned long long key = keyv[j];
    const long long pay = payv[j];
    uint32_t i = ht_home(dst, key);
    if (d.kind == HT_MAP32) {
      if ((uint32_t)key == EMPTY32) { atomicOr(d.err, ERR_RESERVED_KEY); continue; }
      unsigned long long* s = (unsigned long long*)d.slots;
      const unsigned long long nv = ((unsigned long long)(uint32_t)(int32_t)pay << 32) | (uint32_t)key;
      for (;;) {
        const unsigned long long old = atomicCAS(s + i, EMPTY64, nv);
        if (old == EMPTY64) break;
        if ((uint32_t)old == (uint32_t)key) { atomicOr(d.err, ERR_DUPKEY); break; }
        i = (i + 1) & dst.mask;
      }
    } else if (d.kind == HT_SET32) {
      if ((uint32_t)key == EMPTY32) { atomicOr(d.err, ERR_RESERVED_KEY); continue; }
      uint32_t* s = (uint32_t*)d.slots;
      for (;;) {
        const uint32_t old = atomicCAS(s + i, EMPTY32, (uint32_t)key);
        if (old == EMPTY32) break;
        if (old == (uint32_t)key) { atomicOr(d.err, ERR_DUPKEY); break; }
        i = (i + 1) & dst.mask;
      }
    } else {
      if (key == EMPTY64) { atomicOr(d.err, ERR_RESERVED_KEY); continue; }
      ulonglong2* s = (ulonglong2*)d.slots;
      for (;;) {
        const unsigned long long old = atomicCAS(&s[i].x, EMPTY64, key);
        if (old == EMPTY64) { s[i].y = (unsigned long long)pay; break; }
        if (old == key) { atomicOr(d.err, ERR_DUPKEY); break; }
        i = (i + 1) & dst.mask;
      }
    }
   }
  }
}

__global__ void minmax_init_kernel(long long* out) {
  out[0] = LLONG_MAX;
  out[1] = LLONG_MIN;
  out[2] = 0;  // descents: rows i with v[i] > v[i+1]
}

__global__ void __launch_bounds__(kThreads) minmax_kernel(const char* col, int w, long long n, long long* out) {
  long long mn = LLONG_MAX, mx = LLONG_MIN;
  unsigned long long desc = 0;
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
    const long long v = ld_col_global(col, w, i);
    mn = min(mn, v);
    mx = max(mx, v);
    if (i + 1 < n && v > ld_col_global(col, w, i + 1)) desc++;
  }
  if (desc) atomicAdd((unsigned long long*)&out[2], desc);
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    mn = min(mn, __shfl_xor_sync(0xffffffffu, mn, o));
    mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, o));
  }
  if ((threadIdx.x & 31) == 0) {
    atomicMin(&out[0], mn);
    atomicMax(&out[1], mx);
  }
}

// one table's columns at once (A0 load): blockIdx.y = column
struct MinmaxCols {
  const char* col[64];
  int w[64];
  long long* out;  // [ncols][4]: min, max, descents, equal neighbours
};

__global__ void minmax_init_cols_kernel(long long* out, int ncols) {
  const int c = threadIdx.x;
  if (c < ncols) {
    out[4 * c] = LLONG_MAX;
    out[4 * c + 1] = LLONG_MIN;
    out[4 * c + 2] = 0;
    out[4 * c + 3] = 0;
  }
}

__global__ void __launch_bounds__(kThreads) minmax_cols_kernel(MinmaxCols a, long long n) {
  const int c = blockIdx.y;
  const char* col = a.col[c];
  const int w = a.w[c];
  long long* out = a.out + 4 * c;
  long long mn = LLONG_MAX, mx = LLONG_MIN;
  unsigned long long desc = 0, eq = 0;
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
    const long long v = ld_col_global(col, w, i);
    mn = min(mn, v);
    mx = max(mx, v);
    if (i + 1 < n) {
      const long long u = ld_col_global(col, w, i + 1);
      desc += v > u;
      eq += v == u;
    }
  }
  if (desc) atomicAdd((unsigned long long*)&out[2], desc);
  if (eq) atomicAdd((unsigned long long*)&out[3], eq);
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    mn = min(mn, __shfl_xor_sync(0xffffffffu, mn, o));
    mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, o));
  }
  if ((threadIdx.x & 31) == 0) {
    atomicMin(&out[0], mn);
    atomicMax(&out[1], mx);
  }
}

// MULTI tables (NEXT-4 fan-out joins, non-unique build key): CSR build.
// Count pass: per-key match counts (a key outside the declared domain latches
// ERR_CAPACITY; the domain comes from the key column's min/max, so it cannot
// happen unless the column changed under a borrowed pointer).
__global__ void __launch_bounds__(kThreads) multi_count_kernel(const __grid_constant__ BuildDesc d) {
  __shared__ HTP src[MAXHT];
  if (threadIdx.x < d.nht) src[threadIdx.x] = load_htp(d.src[threadIdx.x]);
  __syncthreads();
  const long long stride = (long long)gridDim.x * blockDim.x;
  for (long long row = ((long long)blockIdx.x * blockDim.x + threadIdx.x) * BR; row < d.nrows; row += stride * BR) {
    bool ok[BR];
    unsigned long long k[BR];
    long long pay[BR];
    build_rows(d, src, row, stride, ok, k, pay);
#pragma unroll
    for (int j = 0; j < BR; j++) {
      if (!ok[j]) continue;
      const unsigned long long ix = (unsigned long long)((long long)(int32_t)(uint32_t)k[j] - d.kmin);
      if (ix >= d.nslots) atomicOr(d.err, ERR_CAPACITY);
      else atomicAdd(d.cursor + ix, 1u);
    }
  }
}

// Scatter pass: each qualifying row takes the next position of its key's
// range (the order inside a key's range is arbitrary: a join output is a set)
__global__ void __launch_bounds__(kThreads) multi_scatter_kernel(const __grid_constant__ BuildDesc d) {
  __shared__ HTP src[MAXHT];
  if (threadIdx.x < d.nht) src[threadIdx.x] = load_htp(d.src[threadIdx.x]);
  __syncthreads();
  const long long stride = (long long)gridDim.x * blockDim.x;
  for (long long row = ((long long)blockIdx.x * blockDim.x + threadIdx.x) * BR; row < d.nrows; row += stride * BR) {
    bool ok[BR];
    unsigned long long k[BR];
    long long pay[BR];
    build_rows(d, src, row, stride, ok, k, pay);
#pragma unroll
    for (int j = 0; j < BR; j++) {
      if (!ok[j]) continue;
      const unsigned long long ix = (unsigned long long)((long long)(int32_t)(uint32_t)k[j] - d.kmin);
      if (ix >= d.nslots) continue;
      const unsigned pos = atomicAdd(d.cursor + ix, 1u);
      ((int*)d.pay)[pos] = (int)pay[j];
    }
  }
}

// Row range [lower_bound(lo), upper_bound(hi)) of a non-decreasing column.
__global__ void sorted_bounds_kernel(const char* col, int w, long long n, long long lo, long long hi, long long* out) {
  long long a = 0, b = n;  // first row with v >= lo
  while (a < b) {
    const long long m = (a + b) / 2;
    if (ld_col_global(col, w, m) < lo) a = m + 1;
    else b = m;
  }
  out[0] = a;
  b = n;  // first row with v > hi (from the lower bound on)
  while (a < b) {
    const long long m = (a + b) / 2;
    if (ld_col_global(col, w, m) <= hi) a = m + 1;
    else b = m;
  }
  out[1] = a;
}

// partition phase: the live row count = last offset + last count
__global__ void part_total_kernel(const unsigned* hist, const unsigned* offs, size_t n, unsigned* total) {
  *total = n ? offs[n - 1] + hist[n - 1] : 0u;
}

}  // namespace

size_t part_scan_tmp_bytes(size_t n) {
  size_t tmp = 0;
  cub::DeviceScan::ExclusiveSum(nullptr, tmp, (unsigned*)nullptr, (unsigned*)nullptr, (int)n);
  return tmp;
}

cudaError_t launch_part_scan(const unsigned* hist, unsigned* offs, size_t n, unsigned* total, void* tmp, size_t tmp_bytes,
                             cudaStream_t s) {
  size_t tb = tmp_bytes;
  cudaError_t e = cub::DeviceScan::ExclusiveSum(tmp, tb, hist, offs, (int)n, s);
  if (e != cudaSuccess) return e;
  part_total_kernel<<<1, 1, 0, s>>>(hist, offs, n, total);
  return cudaGetLastError();
}

cudaError_t launch_sorted_bounds(const void* col, int w, long long n, long long lo, long long hi, long long* out,
                                 cudaStream_t s) {
  sorted_bounds_kernel<<<1, 1, 0, s>>>((const char*)col, w, n, lo, hi, out);
  return cudaGetLastError();
}

size_t multi_scan_tmp_bytes(unsigned long long nslots) {
  size_t tmp = 0;
  cub::DeviceScan::ExclusiveSum(nullptr, tmp, (unsigned*)nullptr, (unsigned*)nullptr, (int)(nslots + 1));
  return tmp;
}

// MULTI build: counts -> exclusive scan into the offsets (slots) -> cursors =
// offsets -> scatter. Five stream-ordered steps, no host round trip.
static cudaError_t launch_build_multi(const BuildDesc& d, int num_sms, cudaStream_t s) {
  const size_t nb = (size_t)(d.nslots + 1) * 4;
  cudaError_t e = cudaMemsetAsync(d.cursor, 0, nb, s);
  if (e != cudaSuccess) return e;
  long long work = d.nrows > 0 ? d.nrows : 1;
  int grid = (int)std::min<long long>((work + kThreads * BR - 1) / (kThreads * BR), (long long)num_sms * 8);
  if (grid < 1) grid = 1;
  if (d.nrows > 0) multi_count_kernel<<<grid, kThreads, 0, s>>>(d);
  size_t tmp = (size_t)d.scan_tmp_bytes;
  e = cub::DeviceScan::ExclusiveSum(d.scan_tmp, tmp, d.cursor, (unsigned*)d.slots, (int)(d.nslots + 1), s);
  if (e != cudaSuccess) return e;
  e = cudaMemcpyAsync(d.cursor, d.slots, (size_t)d.nslots * 4, cudaMemcpyDeviceToDevice, s);
  if (e != cudaSuccess) return e;
  if (d.nrows > 0) multi_scatter_kernel<<<grid, kThreads, 0, s>>>(d);
  return cudaGetLastError();
}

cudaError_t launch_minmax_cols(const char* const* cols, const int* widths, int ncols, long long n, long long* out,
                               cudaStream_t s) {
  if (ncols < 1 || ncols > 64) return cudaErrorInvalidValue;
  minmax_init_cols_kernel<<<1, 64, 0, s>>>(out, ncols);
  if (n > 0) {
    MinmaxCols a;
    for (int c = 0; c < ncols; c++) {
      a.col[c] = cols[c];
      a.w[c] = widths[c];
    }
    a.out = out;
    const int gx = (int)std::min<long long>((n + kThreads - 1) / kThreads, std::max(1, 148 * 8 / ncols));
    minmax_cols_kernel<<<dim3(gx, ncols), kThreads, 0, s>>>(a, n);
  }
  return cudaGetLastError();
}

cudaError_t launch_header_init(HTHeader* hdr, cudaStream_t s) {
  header_init_kernel<<<1, 1, 0, s>>>(hdr);
  return cudaGetLastError();
}

cudaError_t launch_build(const BuildDesc& d, bool trivial, const HTHeader& known, int num_sms, cudaStream_t s) {
  long long work = d.nrows > 0 ? d.nrows : 1;
  int grid = (int)std::min<long long>((work + kThreads * BR - 1) / (kThreads * BR), (long long)num_sms * 8);
  if (grid < 1) grid = 1;
  if (d.kind == HT_MULTI) return launch_build_multi(d, num_sms, s);
  if (d.kind == HT_DIRECT) {  // host-sized: clear + insert, no count pass
    cudaError_t e = cudaMemsetAsync(d.slots, 0, direct_bytes(d.width, d.nslots), s);
    if (e != cudaSuccess) return e;
    if (d.nrows > 0) build_insert_kernel<<<grid, kThreads, 0, s>>>(d);
    return cudaGetLastError();
  }
  if (!trivial) build_count_kernel<<<grid, kThreads, 0, s>>>(d);
  long long clear_blocks = std::min<long long>((d.cap_slots * 16 / 16 + kThreads - 1) / kThreads, (long long)num_sms * 8);
  if (trivial) {
    const int sb = d.kind == HT_SET32 ? 4 : d.kind == HT_MAP32 ? 8 : 16;
    clear_blocks = std::min<long long>(((long long)(known.mask + 1ull) * sb / 16 + kThreads - 1) / kThreads,
                                       (long long)num_sms * 8);
  }
  if (clear_blocks < 1) clear_blocks = 1;
  build_clear_kernel<<<(int)clear_blocks, kThreads, 0, s>>>(d, trivial ? 1 : 0, known);
  if (d.nrows > 0) build_insert_kernel<<<grid, kThreads, 0, s>>>(d);
  return cudaGetLastError();
}

cudaError_t launch_minmax(const void* col, int width, long long n, long long* out, cudaStream_t s) {
  minmax_init_kernel<<<1, 1, 0, s>>>(out);
  if (n > 0) {
    int grid = (int)std::min<long long>((n + kThreads - 1) / kThreads, 148LL * 8);
    minmax_kernel<<<grid, kThreads, 0, s>>>((const char*)col, width, n, out);
  }
  return cudaGetLastError();
}

}  // namespace gpl
