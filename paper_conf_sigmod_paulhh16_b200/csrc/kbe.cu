// kbe.cu — the paper's kernel-based execution (KBE) baseline (PAPER.md
// P:89-95 §2.2, Fig 7): every operator runs as separate kernels
// over the WHOLE input and materialises its output in global memory before
// the next operator starts:
//   selection  = map (predicate flags) -> prefix sum -> scatter   (GDB [13])
//   hash probe = map (probe; flags + payload column) -> prefix sum -> scatter
//   where      = map -> prefix sum -> scatter
//   aggregate  = one reduction kernel over the final materialised rows
// As in KBE systems, the host reads each operator's output cardinality to
// size the next buffers (one D2H per operator). Same lowered plan, same hash
// tables and the same exact arithmetic as the fused pipeline, so results are
// bit-identical; the materialised bytes are counted for config 5
// (intermediate HBM bytes normalised to the input, Figs 3/17/18).
#include <cub/cub.cuh>

#include <vector>

#include "device_common.cuh"
#include "kernels.h"

namespace gpl {
namespace {

constexpr int kThreads = 256;

struct Field {
  char* ptr = nullptr;
  int w = 8;
  bool owned = false;
};

__device__ __forceinline__ long long ldf(const char* p, int w, long long i) {
  return w == 4 ? (long long)((const int*)p)[i] : ((const long long*)p)[i];
}
__device__ __forceinline__ void stf(char* p, int w, long long i, long long v) {
  if (w == 4) ((int*)p)[i] = (int)v;
  else ((long long*)p)[i] = v;
}

// map: all filters of the segment on the staged columns -> flags
__global__ void kbe_filter_map(const __grid_constant__ PipeDesc d, long long n, int* flags) {
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
    bool p = true;
    for (int f = 0; f < d.nfilt; f++) {
      const Filt& F = d.filt[f];
      p = p && filt_pass(F, ld_col_global(d.col[F.ref], d.colw[F.ref], i));
    }
    flags[i] = p ? 1 : 0;
  }
}

// value term from staged columns (expression materialised as a column)
__device__ __forceinline__ long long stage_term(const PipeDesc& d, const Term& T, long long i) {
  long long v = T.sign;
  for (int f = 0; f < T.nfact; f++) {
    const Factor& F = T.f[f];
    const long long x = F.field >= 0 ? ld_col_global(d.col[F.field], d.colw[F.field], i) : 0;
    v *= F.a + (long long)F.b * x;
  }
  return v;
}

__global__ void kbe_term_map(const __grid_constant__ PipeDesc d, int t, long long n, long long* out) {
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x)
    out[i] = stage_term(d, d.sterm[t], i);
}

struct FieldSet {
  char* ptr[MAXQ];
  int w[MAXQ];
  int n;
};

// scatter: compact every live field by flags/positions. Pushed-down terms
// with no array yet are evaluated from the staged columns (first operator).
__global__ void kbe_scatter(const __grid_constant__ PipeDesc d, long long n, const int* flags, const int* pos,
                            FieldSet in, FieldSet out, int first, const long long* nptr) {
  if (nptr) n = min(n, *nptr);
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
    if (!flags[i]) continue;
    const long long o = pos[i];
    for (int f = 0; f < out.n; f++) {
      if (!out.ptr[f]) continue;
      long long v;
      if (in.ptr[f]) v = ldf(in.ptr[f], in.w[f], i);
      else if (first && d.push[f].kind == PUSH_TERM) v = stage_term(d, d.sterm[d.push[f].src], i);
      else continue;
      stf(out.ptr[f], out.w[f], o, v);
    }
  }
}

__global__ void kbe_probe_map(const __grid_constant__ PipeDesc d, int pi, long long n, FieldSet fs, int* flags,
                              char* payload, int pw, const long long* nptr) {
  if (nptr) n = min(n, *nptr);
  const Probe& P = d.probe[pi];
  const HTP h = load_htp(d.ht[P.ht]);
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
    unsigned long long k = (uint32_t)ldf(fs.ptr[P.k1], fs.w[P.k1], i);
    if (P.k2 >= 0) k = (k << 32) | (uint32_t)ldf(fs.ptr[P.k2], fs.w[P.k2], i);
    long long v = 0;
    const bool hit = ht_probe(h, k, &v);
    flags[i] = hit ? 1 : 0;
    if (payload) stf(payload, pw, i, P.kind == P_MARK ? (hit ? 1 : 0) : v);
  }
}

__global__ void kbe_resid_map(const __grid_constant__ PipeDesc d, int r, long long n, FieldSet fs, int* flags,
                              const long long* nptr) {
  if (nptr) n = min(n, *nptr);
  const Resid& R = d.resid[r];
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
    const long long a = ldf(fs.ptr[R.a], fs.w[R.a], i);
    bool p;
    if (R.kind == R_EQ) p = a == ldf(fs.ptr[R.b], fs.w[R.b], i);
    else if (R.kind == R_PAIRS) {
      const long long b = ldf(fs.ptr[R.b], fs.w[R.b], i);
      p = false;
      for (int k = 0; k < R.npairs; k++) p |= (a == R.pa[k]) & (b == R.pb[k]);
    } else if (R.kind == R_RANGE) p = a >= R.lo && a <= R.hi;
    else p = (unsigned long long)a < 64ull && ((R.mask >> a) & 1ull);
    flags[i] = p ? 1 : 0;
  }
}

// output cardinality of a compaction; device-sized mode also accumulates the
// materialised bytes (positions + live output fields) on the device
__global__ void kbe_total(const int* flags, const int* pos, long long n, long long* total, unsigned long long* bytes,
                          const long long* nprev, int in_row_bytes, int out_w) {
  const long long live_in = nprev ? *nprev : n;  // (read before *total is overwritten: same word)
  const long long t = n ? (long long)pos[n - 1] + flags[n - 1] : 0;
  *total = t;
  if (bytes) *bytes += (unsigned long long)(live_in * in_row_bytes + t * (long long)out_w);
}

// aggregate over the final materialised rows: per-block shared table, then
// exact int128 global atomics (same arithmetic as the fused pipeline)
__global__ void kbe_aggregate(const __grid_constant__ PipeDesc d, long long n, FieldSet fs, unsigned long long* partials,
                              const long long* nptr) {
  if (nptr) n = min(n, *nptr);
  extern __shared__ unsigned long long tab[];
  const int G = d.ngroups_total, A = d.nagg;
  const bool use_smem = G * A <= 4096;
  if (use_smem)
    for (int i = threadIdx.x; i < G * A; i += blockDim.x) tab[i] = 0;
  __syncthreads();
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
    int gid = 0;
    bool ok = true;
    for (int g = 0; g < d.ngroup; g++) {
      const GroupDim& GD = d.gdim[g];
      long long v = ldf(fs.ptr[GD.field], fs.w[GD.field], i);
      if (GD.transform == G_YEAR) v = (int)v / 10000;
      const long long o = v - GD.lo;
      if ((unsigned long long)o >= (unsigned long long)GD.size) ok = false;
      gid += (int)o * GD.stride;
    }
    if (!ok) {
      atomicOr(d.err, ERR_DOMAIN);
      continue;
    }
    long long val = 0;
    for (int t = 0; t < d.nterm; t++) {
      if (d.term_field[t] >= 0) {
        val += ldf(fs.ptr[d.term_field[t]], fs.w[d.term_field[t]], i);
        continue;
      }
      const Term& T = d.term[t];
      long long prod = T.sign;
      for (int f = 0; f < T.nfact; f++) {
        const Factor& F = T.f[f];
        prod *= F.field < 0 ? F.a : F.a + (long long)F.b * ldf(fs.ptr[F.field], fs.w[F.field], i);
      }
      val += prod;
    }
    for (int a = 0; a < A; a++) {
      const Agg& Ag = d.agg[a];
      long long c = 1;
      if (Ag.kind == A_SUM) c = val;
      else if (Ag.kind == A_SUMIF) c = ldf(fs.ptr[Ag.field], fs.w[Ag.field], i) != 0 ? val : 0;
      else if (Ag.kind == A_SUMIFEQ) c = ldf(fs.ptr[Ag.field], fs.w[Ag.field], i) == Ag.c ? val : 0;
      if (c == 0) continue;
      if (use_smem) atomicAdd(&tab[gid * A + a], (unsigned long long)c);
      else atomic_add_i128(partials + 2 * (gid * A + a), c);
    }
  }
  __syncthreads();
  if (use_smem)
    for (int i = threadIdx.x; i < G * A; i += blockDim.x)
      if (tab[i]) atomic_add_i128(partials + 2 * i, (long long)tab[i]);
}

int grid_for(long long n, int sms) {
  long long g = (n + kThreads - 1) / kThreads;
  if (g > (long long)sms * 8) g = (long long)sms * 8;
  return (int)(g < 1 ? 1 : g);
}

}  // namespace

size_t kbe_pool_bytes(const PipeDesc& d, bool device_sized) {
  // upper bound: flags + positions + two generations of every field + payloads + scan temp
  size_t per_row = 8;
  size_t fw = 0;
  for (int f = 0; f < d.nfield; f++) fw += (size_t)d.qw[f];
  per_row += 2 * fw;
  per_row += 8 * (size_t)(d.nprobe + d.nresid + d.nfilt + 2) * 2;
  // device-sized (GPL w/o CE): every operator's outputs are allocated at the full capacity
  if (device_sized) per_row = (size_t)(d.nprobe + d.nresid + (d.nfilt > 0 ? 1 : 0) + 1) * (24 + fw) + 16;
  size_t tmp = 0;
  cub::DeviceScan::ExclusiveSum(nullptr, tmp, (int*)nullptr, (int*)nullptr, (int)(d.nrows > 0 ? d.nrows : 1));
  return per_row * (size_t)(d.nrows + 64) + 4 * (tmp + 4096) + (1 << 20);
}

// KBE over d.nrows rows. device_bytes == nullptr: the paper's KBE — the host
// reads every operator's output cardinality (one D2H + synchronise per
// operator) to size the next buffers. device_bytes != nullptr: the same
// kernel sequence with every buffer sized for d.nrows (an operator's output is
// never larger than its input) and the cardinalities kept on the device (the
// kernels read them): no host round trip, so GPL (w/o CE) can run tile after
// tile asynchronously; the materialised bytes accumulate in
// *device_bytes.
cudaError_t run_kbe(const PipeDesc& d, int sms, cudaStream_t s, void* pool, size_t pool_bytes, double* inter_bytes,
                    unsigned long long* device_bytes) {
  double bytes = 0;
  cudaError_t e = cudaSuccess;
  size_t used = 0;
  const bool dev = device_bytes != nullptr;
  // bump allocation from a per-context pool (sized once by kbe_pool_bytes), so
  // the baseline pays for materialisation, not for the allocator
  auto alloc = [&](size_t b) -> char* {
    b = (b + 255) & ~(size_t)255;
    if (b < 256) b = 256;
    if (used + b > pool_bytes) {
      if (e == cudaSuccess) e = cudaErrorMemoryAllocation;
      return nullptr;
    }
    char* p = (char*)pool + used;
    used += b;
    return p;
  };
  long long* d_total = (long long*)alloc(sizeof(long long));
  long long n = d.nrows;          // host: the row count (KBE) / the capacity (device-sized)
  const long long cap = d.nrows;
  const long long* nptr = nullptr;  // device-sized: the live row count on the device (null: n rows)
  FieldSet fs{};
  fs.n = d.nfield;
  for (int f = 0; f < d.nfield; f++) {
    fs.w[f] = d.qw[f];
    fs.ptr[f] = (f < d.npush && d.push[f].kind == PUSH_COL) ? (char*)d.col[d.push[f].src] : nullptr;
  }
  // compact all live fields by a flags array (prefix sum + scatter); returns new n
  auto compact = [&](int* flags, bool first, int pay_w) -> long long {
    int* pos = (int*)alloc(sizeof(int) * (size_t)(n > 0 ? n : 1));
    size_t tmp = 0;
    cub::DeviceScan::ExclusiveSum(nullptr, tmp, flags, pos, (int)n, s);
    void* t = alloc(tmp);
    if (e != cudaSuccess) return 0;
    if (n > 0) cub::DeviceScan::ExclusiveSum(t, tmp, flags, pos, (int)n, s);
    int out_w = 0;
    for (int f = 0; f < fs.n; f++)
      if (fs.ptr[f] || (first && f < d.npush && d.push[f].kind == PUSH_TERM)) out_w += fs.w[f];
    long long total = 0;
    if (dev) {
      // the count stays on the device; buffers sized for the capacity
      // flags + positions (8 B) + the map's payload column per live input row, then the compacted fields
      kbe_total<<<1, 1, 0, s>>>(flags, pos, n, d_total, device_bytes, nptr, 8 + pay_w, out_w);
      total = n;
    } else {
      kbe_total<<<1, 1, 0, s>>>(flags, pos, n, d_total, nullptr, nullptr, 0, 0);
      if (e == cudaSuccess) e = cudaMemcpyAsync(&total, d_total, sizeof(total), cudaMemcpyDeviceToHost, s);
      if (e == cudaSuccess) e = cudaStreamSynchronize(s);  // KBE sizes the next operator's output here
      bytes += 4.0 * n + (double)total * out_w;  // positions + the compacted live fields (flags/payloads: the maps)
    }
    FieldSet out = fs;
    for (int f = 0; f < fs.n; f++) {
      const bool live = fs.ptr[f] || (first && f < d.npush && d.push[f].kind == PUSH_TERM);
      out.ptr[f] = live ? alloc((size_t)(total > 0 ? total : 1) * fs.w[f]) : nullptr;
    }
    // (the scatter walks the whole input capacity: flags beyond the live rows are 0, and the
    // count word already holds this operator's OUTPUT count)
    if (n > 0) kbe_scatter<<<grid_for(n, sms), kThreads, 0, s>>>(d, n, flags, pos, fs, out, first ? 1 : 0, nullptr);
    fs = out;
    if (dev) nptr = d_total;  // every later kernel reads the live count
    return total;
  };
  // device-sized mode: a map writes flags only for the live rows; the rest of
  // the capacity must read as 0 for the scan
  auto flags_for = [&]() -> int* {
    int* f = (int*)alloc(sizeof(int) * (size_t)(n > 0 ? n : 1));
    if (dev && nptr && f && n > 0 && e == cudaSuccess) e = cudaMemsetAsync(f, 0, sizeof(int) * (size_t)n, s);
    return f;
  };
  // selection: map -> prefix sum -> scatter
  if (d.nfilt > 0) {
    int* flags = flags_for();
    if (n > 0) kbe_filter_map<<<grid_for(n, sms), kThreads, 0, s>>>(d, n, flags);
    if (!dev) bytes += 4.0 * n;
    n = compact(flags, true, 0);
  } else {
    for (int f = 0; f < d.npush; f++)
      if (d.push[f].kind == PUSH_TERM) {  // expression materialised as a column
        fs.ptr[f] = alloc(sizeof(long long) * (size_t)(n > 0 ? n : 1));
        if (n > 0) kbe_term_map<<<grid_for(n, sms), kThreads, 0, s>>>(d, d.push[f].src, n, (long long*)fs.ptr[f]);
        bytes += 8.0 * n;
      }
  }
  // probes: map (flags + payload) -> prefix sum -> scatter
  for (int p = 0; p < d.nprobe && e == cudaSuccess; p++) {
    const Probe& P = d.probe[p];
    int* flags = flags_for();
    char* pay = nullptr;
    int pw = 8;
    if (P.out >= 0) {
      pw = fs.w[P.out];
      pay = alloc((size_t)(n > 0 ? n : 1) * pw);
      fs.ptr[P.out] = pay;
      if (!dev) bytes += (double)n * pw;
    }
    if (n > 0) kbe_probe_map<<<grid_for(n, sms), kThreads, 0, s>>>(d, p, n, fs, flags, pay, pw, nptr);
    if (!dev) bytes += 4.0 * n;
    if (P.kind != P_MARK) n = compact(flags, false, P.out >= 0 ? pw : 0);
  }
  for (int r = 0; r < d.nresid && e == cudaSuccess; r++) {
    int* flags = flags_for();
    if (n > 0) kbe_resid_map<<<grid_for(n, sms), kThreads, 0, s>>>(d, r, n, fs, flags, nptr);
    if (!dev) bytes += 4.0 * n;
    n = compact(flags, false, 0);
  }
  if (e == cudaSuccess && n > 0) {
    const size_t sm = (size_t)d.ngroups_total * d.nagg <= 4096 ? (size_t)d.ngroups_total * d.nagg * 8 : 0;
    kbe_aggregate<<<grid_for(n, sms), kThreads, sm, s>>>(d, n, fs, d.partials, nptr);
  }
  (void)cap;
  *inter_bytes = bytes;
  if (e != cudaSuccess) return e;
  return cudaGetLastError();
}

}  // namespace gpl
