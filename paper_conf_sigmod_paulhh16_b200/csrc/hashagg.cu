// hashagg.cu — result step of a hash group-by: the
// blocking operator after the fused pipeline (ORDER BY is blocking).
//
//   * ORDER BY ... LIMIT k: a two-phase device selection. Phase A: every CTA
//     walks its slice of the hash-aggregation table in coalesced chunks and
//     keeps its k best groups in a shared-memory tile: a group is admitted
//     only if it beats the current k-th best, and the tile is bitonic-sorted
//     only when its free room runs low (so after the first sort almost every
//     group is rejected by one comparison). Phase B: one CTA runs the same
//     selection over the CTAs' candidates and writes the k rows in order — to
//     the device row buffer and to the run's result words, so the copy-out
//     kernel brings them back with the counters (no extra D2H).
//   * no LIMIT: every occupied slot is compacted into the row buffer; the
//     full ORDER BY (else key order) is then a device sort of the compacted
//     rows at fetch (sort_hagg_rows: one stable LSD radix-sort pass per sort
//     word, least significant word first, then a gather): a blocking full
//     sort on the GPU, no host sort.
// A row is [packed key, acc 0 .. nagg-1] (8-byte words). Ordering: the plan's
// components (aggregate or key field, asc/desc), then the full key ascending,
// so the first k rows are unique.
#include <algorithm>

#include <cub/cub.cuh>

#include "kernels.h"
#include "device_common.cuh"

namespace gpl {
namespace {

constexpr int kThreads = 256;
constexpr unsigned kNone = 0xFFFFFFFFu;
constexpr unsigned long long kSign = 1ull << 63;

// Selection tile of T entries: the k best so far in [0, k), new candidates
// appended after them.
constexpr int kSmallK = 32;  // k <= 32: compaction by k rounds of block arg-min, else bitonic sort

template <int T>
struct SelSmem {
  unsigned long long w[4][T];  // sort words (lexicographic, ascending = better)
  unsigned idx[T];             // slot index (kNone = padding / taken)
  unsigned long long thr[4];   // the current k-th best (admission threshold)
  int fill, have_thr;
  // small-k selection: the rounds' winners and the per-warp arg-min scratch
  unsigned long long selw[4][kSmallK];
  unsigned selidx[kSmallK];
  unsigned long long redw[4][kThreads / 32];
  int redpos[kThreads / 32];
  int nsel;
};

__device__ __forceinline__ int key_field(unsigned long long key, int nkeys, int i) {
  return nkeys == 2 ? (int)(unsigned)(i == 0 ? key >> 32 : key) : (int)(unsigned)key;
}

// The sort words of slot s (order components, then the full key ascending,
// then zeros); returns false when the slot is empty.
__device__ __forceinline__ bool words_of(const HaggResultDesc& D, unsigned long long s, unsigned long long (&w)[4]) {
  const unsigned long long st = __ldcg(D.keys + s);
  if (st == 0ull) return false;
  const unsigned long long key = ~st;
  unsigned long long kw;  // full key ascending (signed fields)
  if (D.nkeys == 2)
    kw = ((unsigned long long)((unsigned)key_field(key, 2, 0) ^ 0x80000000u) << 32) |
         (unsigned long long)((unsigned)key_field(key, 2, 1) ^ 0x80000000u);
  else
    kw = (unsigned long long)(long long)key_field(key, 1, 0) ^ kSign;
#pragma unroll
  for (int c = 0; c < 4; c++) {
    if (c < D.norder) {
      const long long v = D.ord_is_agg[c] ? __ldcg(D.accs + s * D.nagg + D.ord_idx[c])
                                          : (long long)key_field(key, D.nkeys, D.ord_idx[c]);
      const unsigned long long u = (unsigned long long)v ^ kSign;
      w[c] = D.ord_desc[c] ? ~u : u;
    } else {
      w[c] = c == D.norder ? kw : 0ull;
    }
  }
  return true;
}

__device__ __forceinline__ bool less4(const unsigned long long (&a)[4], const unsigned long long (&b)[4]) {
#pragma unroll
  for (int c = 0; c < 4; c++)
    if (a[c] != b[c]) return a[c] < b[c];
  return false;
}

template <int T>
__device__ __forceinline__ bool less_at(const SelSmem<T>& m, int i, int j) {
#pragma unroll
  for (int c = 0; c < 4; c++)
    if (m.w[c][i] != m.w[c][j]) return m.w[c][i] < m.w[c][j];
  return m.idx[i] < m.idx[j];
}

template <int T>
__device__ void bitonic_sort(SelSmem<T>& m) {
  for (int k = 2; k <= T; k <<= 1)
    for (int j = k >> 1; j > 0; j >>= 1) {
      for (int i = threadIdx.x; i < T; i += blockDim.x) {
        const int p = i ^ j;
        if (p > i) {
          const bool up = (i & k) == 0;
          if (less_at(m, p, i) == up) {
#pragma unroll
            for (int c = 0; c < 4; c++) {
              const unsigned long long t = m.w[c][i];
              m.w[c][i] = m.w[c][p];
              m.w[c][p] = t;
            }
            const unsigned t = m.idx[i];
            m.idx[i] = m.idx[p];
            m.idx[p] = t;
          }
        }
      }
      __syncthreads();
    }
}

// The k best of tile entries [0, n) moved to [0, k) in order (k <= kSmallK):
// k rounds of a block-wide arg-min (warp shuffles, then one warp over the
// per-warp winners); a winner is marked taken (idx = kNone). Much cheaper
// than sorting the tile when k is small.
template <int T>
__device__ void select_small(SelSmem<T>& m, int n, int K) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
  if (threadIdx.x == 0) m.nsel = 0;
  for (int r = 0; r < K; r++) {
    unsigned long long b[4] = {~0ull, ~0ull, ~0ull, ~0ull};
    int bp = -1;
    for (int i = threadIdx.x; i < n; i += blockDim.x) {
      if (m.idx[i] == kNone) continue;
      const unsigned long long x[4] = {m.w[0][i], m.w[1][i], m.w[2][i], m.w[3][i]};
      if (bp < 0 || less4(x, b)) {
#pragma unroll
        for (int c = 0; c < 4; c++) b[c] = x[c];
        bp = i;
      }
    }
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) {
      unsigned long long o[4];
#pragma unroll
      for (int c = 0; c < 4; c++) o[c] = __shfl_down_sync(0xffffffffu, b[c], off);
      const int op = __shfl_down_sync(0xffffffffu, bp, off);
      if (op >= 0 && (bp < 0 || less4(o, b))) {
#pragma unroll
        for (int c = 0; c < 4; c++) b[c] = o[c];
        bp = op;
      }
    }
    if (lane == 0) {
#pragma unroll
      for (int c = 0; c < 4; c++) m.redw[c][warp] = b[c];
      m.redpos[warp] = bp;
    }
    __syncthreads();
    if (warp == 0) {
      unsigned long long x[4] = {~0ull, ~0ull, ~0ull, ~0ull};
      int xp = -1;
      if (lane < nw) {
#pragma unroll
        for (int c = 0; c < 4; c++) x[c] = m.redw[c][lane];
        xp = m.redpos[lane];
      }
#pragma unroll
      for (int off = 16; off > 0; off >>= 1) {
        unsigned long long o[4];
#pragma unroll
        for (int c = 0; c < 4; c++) o[c] = __shfl_down_sync(0xffffffffu, x[c], off);
        const int op = __shfl_down_sync(0xffffffffu, xp, off);
        if (op >= 0 && (xp < 0 || less4(o, x))) {
#pragma unroll
          for (int c = 0; c < 4; c++) x[c] = o[c];
          xp = op;
        }
      }
      if (lane == 0 && xp >= 0) {
        const int t = m.nsel++;
#pragma unroll
        for (int c = 0; c < 4; c++) m.selw[c][t] = x[c];
        m.selidx[t] = m.idx[xp];
        m.idx[xp] = kNone;
      }
    }
    __syncthreads();
  }
  const int ns = m.nsel;
  for (int i = threadIdx.x; i < T; i += blockDim.x) {
    if (i < ns) {
#pragma unroll
      for (int c = 0; c < 4; c++) m.w[c][i] = m.selw[c][i];
      m.idx[i] = m.selidx[i];
    } else {
#pragma unroll
      for (int c = 0; c < 4; c++) m.w[c][i] = ~0ull;
      m.idx[i] = kNone;
    }
  }
  __syncthreads();
}

template <int T>
__device__ __forceinline__ void set_pad(SelSmem<T>& m, int i) {
#pragma unroll
  for (int c = 0; c < 4; c++) m.w[c][i] = ~0ull;
  m.idx[i] = kNone;
}

// Keep the k best of the input range in m.idx[0..k) (sorted, best first).
// from_cand: the input is D.cand entries [lo..hi) (phase A's winners with
// their sort words: 5 words each, idx kNone = none), else the hash slots. One coalesced chunk of blockDim positions per
// step; the tile is sorted only when its free room could not take another
// chunk (or at the end).
template <int T>
__device__ void select_k(const HaggResultDesc& D, SelSmem<T>& m, unsigned long long lo, unsigned long long hi,
                         bool from_cand) {
  const int K = D.limit;
  for (int i = threadIdx.x; i < T; i += blockDim.x) set_pad(m, i);
  if (threadIdx.x == 0) {
    m.fill = 0;
    m.have_thr = 0;
  }
  __syncthreads();
  const int room = T - K;  // >= blockDim (the launcher picks T from k)
  for (unsigned long long base = lo; base < hi; base += blockDim.x) {
    const unsigned long long pos = base + threadIdx.x;
    if (pos < hi) {
      unsigned long long s = pos;
      unsigned long long w[4];
      bool ok;
      if (from_cand) {  // coalesced: the words travel with the candidate
        const unsigned long long* e = D.cand + pos * 5;
        s = e[4];
        ok = s != kNone;
#pragma unroll
        for (int c = 0; c < 4; c++) w[c] = e[c];
      } else {
        ok = words_of(D, s, w);
      }
      if (ok) {
        bool admit = true;
        if (m.have_thr) {
          const unsigned long long th[4] = {m.thr[0], m.thr[1], m.thr[2], m.thr[3]};
          admit = less4(w, th);
        }
        if (admit) {
          const int at = K + atomicAdd(&m.fill, 1);
#pragma unroll
          for (int c = 0; c < 4; c++) m.w[c][at] = w[c];
          m.idx[at] = (unsigned)s;
        }
      }
    }
    __syncthreads();
    const int fill = m.fill;  // uniform
    if (fill > 0 && (fill > room - (int)blockDim.x || base + blockDim.x >= hi)) {
      if (K <= kSmallK) {
        select_small(m, K + fill, K);  // [0, K) best, the rest padding
      } else {
        bitonic_sort(m);
        // entries [K, T) are dropped: reset them
        for (int i = K + threadIdx.x; i < T; i += blockDim.x) set_pad(m, i);
      }
      // record the threshold (the k-th best)
      if (threadIdx.x == 0) {
        m.fill = 0;
        if (m.idx[K - 1] != kNone) {
          m.have_thr = 1;
#pragma unroll
          for (int c = 0; c < 4; c++) m.thr[c] = m.w[c][K - 1];
        }
      }
    }
    __syncthreads();
  }
}

template <int T>
__global__ void __launch_bounds__(kThreads) select_phase_a(const __grid_constant__ HaggResultDesc D) {
  __shared__ SelSmem<T> m;
  const unsigned long long per = (D.nslots + gridDim.x - 1) / gridDim.x;
  const unsigned long long lo = per * blockIdx.x, hi = min(D.nslots, lo + per);
  select_k<T>(D, m, lo, lo < hi ? hi : lo, false);
  unsigned long long* out = D.cand + (unsigned long long)blockIdx.x * D.limit * 5;
  for (int i = threadIdx.x; i < D.limit * 5; i += blockDim.x) {
    const int e = i / 5, c = i % 5;
    out[i] = c < 4 ? m.w[c][e] : (unsigned long long)m.idx[e];
  }
}

template <int T>
__global__ void __launch_bounds__(kThreads) select_phase_b(const __grid_constant__ HaggResultDesc D,
                                                           const unsigned long long* hagg_count) {
  __shared__ SelSmem<T> m;
  select_k<T>(D, m, 0, (unsigned long long)D.nblocks * D.limit, true);
  int n = 0;
  for (int i = 0; i < D.limit; i++) n += m.idx[i] != kNone;
  const int W = 1 + D.nagg;
  for (int i = threadIdx.x; i < n * W; i += blockDim.x) {
    const int r = i / W, c = i % W;
    const unsigned long long s = m.idx[r];
    const unsigned long long v = c == 0 ? ~__ldcg(D.keys + s) : (unsigned long long)__ldcg(D.accs + s * D.nagg + (c - 1));
    D.rows[i] = v;
    D.small_out[2 + i] = v;
  }
  if (threadIdx.x == 0) {
    D.small_out[0] = __ldcg(hagg_count);
    D.small_out[1] = (unsigned long long)n;
  }
}

__global__ void __launch_bounds__(kThreads) compact_groups(const __grid_constant__ HaggResultDesc D) {
  const int W = 1 + D.nagg;
  for (unsigned long long s = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; s < D.nslots;
       s += (unsigned long long)gridDim.x * blockDim.x) {
    const unsigned long long st = __ldcg(D.keys + s);
    if (st == 0ull) continue;
    const unsigned long long r = atomicAdd(D.n_out, 1ull);
    D.rows[r * W] = ~st;
    for (int a = 0; a < D.nagg; a++) D.rows[r * W + 1 + a] = (unsigned long long)__ldcg(D.accs + s * D.nagg + a);
  }
}

// ---- full device sort of compacted rows (ORDER BY without LIMIT)

// Sort word c of the rows in permutation order (the same words as words_of,
// read from a compacted row [key, acc...] instead of a table slot).
__global__ void __launch_bounds__(kThreads) sort_word_kernel(const __grid_constant__ HaggResultDesc D,
                                                              const unsigned long long* rows, const unsigned* perm,
                                                              unsigned long long n, int c, unsigned long long* out) {
  const int W = 1 + D.nagg;
  for (unsigned long long i = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (unsigned long long)gridDim.x * blockDim.x) {
    const unsigned r = perm ? perm[i] : (unsigned)i;
    const unsigned long long key = rows[(unsigned long long)r * W];
    unsigned long long w;
    if (c < D.norder) {
      const long long v = D.ord_is_agg[c] ? (long long)rows[(unsigned long long)r * W + 1 + D.ord_idx[c]]
                                          : (long long)key_field(key, D.nkeys, D.ord_idx[c]);
      const unsigned long long u = (unsigned long long)v ^ kSign;
      w = D.ord_desc[c] ? ~u : u;
    } else if (D.nkeys == 2) {
      w = ((unsigned long long)((unsigned)key_field(key, 2, 0) ^ 0x80000000u) << 32) |
          (unsigned long long)((unsigned)key_field(key, 2, 1) ^ 0x80000000u);
    } else {
      w = (unsigned long long)(long long)key_field(key, 1, 0) ^ kSign;
    }
    out[i] = w;
  }
}

__global__ void __launch_bounds__(kThreads) iota_kernel(unsigned* p, unsigned long long n) {
  for (unsigned long long i = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (unsigned long long)gridDim.x * blockDim.x)
    p[i] = (unsigned)i;
}

__global__ void __launch_bounds__(kThreads) gather_rows_kernel(const unsigned long long* rows, const unsigned* perm,
                                                                unsigned long long n, int W, unsigned long long* out) {
  for (unsigned long long i = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; i < n * (unsigned long long)W;
       i += (unsigned long long)gridDim.x * blockDim.x) {
    const unsigned long long r = i / (unsigned long long)W, w = i % (unsigned long long)W;
    out[i] = rows[(unsigned long long)perm[r] * W + w];
  }
}

struct SortTmp {
  unsigned long long *ka, *kb;
  unsigned *pa, *pb;
  void* cub;
  size_t cub_bytes;
};

SortTmp carve(void* tmp, unsigned long long n) {
  SortTmp t;
  char* p = (char*)tmp;
  auto take = [&](size_t b) {
    char* q = p;
    p += (b + 255) / 256 * 256;
    return q;
  };
  t.ka = (unsigned long long*)take(n * 8);
  t.kb = (unsigned long long*)take(n * 8);
  t.pa = (unsigned*)take(n * 4);
  t.pb = (unsigned*)take(n * 4);
  t.cub_bytes = 0;
  cub::DeviceRadixSort::SortPairs(nullptr, t.cub_bytes, (unsigned long long*)nullptr, (unsigned long long*)nullptr,
                                  (unsigned*)nullptr, (unsigned*)nullptr, (int)n);
  t.cub = take(t.cub_bytes);
  return t;
}

}  // namespace

size_t sort_hagg_tmp_bytes(unsigned long long n) {
  auto r = [](size_t b) { return (b + 255) / 256 * 256; };
  size_t cb = 0;
  cub::DeviceRadixSort::SortPairs(nullptr, cb, (unsigned long long*)nullptr, (unsigned long long*)nullptr,
                                  (unsigned*)nullptr, (unsigned*)nullptr, (int)n);
  return 2 * r(n * 8) + 2 * r(n * 4) + r(cb);
}

cudaError_t sort_hagg_rows(const HaggResultDesc& D, const unsigned long long* rows, unsigned long long n,
                           unsigned long long* out, void* tmp, int num_sms, cudaStream_t s) {
  if (n == 0) return cudaSuccess;
  SortTmp t = carve(tmp, n);
  const int grid = (int)std::min<unsigned long long>((n + kThreads - 1) / kThreads, (unsigned long long)num_sms * 8);
  iota_kernel<<<grid, kThreads, 0, s>>>(t.pa, n);
  // least significant word first: the full key, then the ORDER BY components from last to first;
  // each pass is a stable radix sort of (word, row) pairs
  for (int c = D.norder; c >= 0; c--) {
    sort_word_kernel<<<grid, kThreads, 0, s>>>(D, rows, t.pa, n, c, t.ka);
    size_t cb = t.cub_bytes;
    cudaError_t e = cub::DeviceRadixSort::SortPairs(t.cub, cb, t.ka, t.kb, t.pa, t.pb, (int)n, 0, 64, s);
    if (e != cudaSuccess) return e;
    std::swap(t.pa, t.pb);
  }
  gather_rows_kernel<<<grid, kThreads, 0, s>>>(rows, t.pa, n, 1 + D.nagg, out);
  return cudaGetLastError();
}

int hagg_select_blocks(unsigned long long nslots, int num_sms) {
  // one slice per CTA, >= 1K slots each, at most 2 CTAs per SM
  const unsigned long long b = (nslots + 1023) / 1024;
  return (int)(b < 1 ? 1 : b > (unsigned long long)(2 * num_sms) ? 2 * num_sms : b);
}

cudaError_t launch_hagg_result(const HaggResultDesc& D, const unsigned long long* hagg_count, int num_sms,
                               cudaStream_t s) {
  if (D.limit > 0) {
    // tile: room for the k best plus one chunk of candidates (k <= 512)
    if (D.limit <= 512 - kThreads) {
      select_phase_a<512><<<D.nblocks, kThreads, 0, s>>>(D);
      select_phase_b<512><<<1, kThreads, 0, s>>>(D, hagg_count);
    } else {
      select_phase_a<1024><<<D.nblocks, kThreads, 0, s>>>(D);
      select_phase_b<1024><<<1, kThreads, 0, s>>>(D, hagg_count);
    }
  } else {
    const unsigned long long b = (D.nslots + kThreads - 1) / kThreads;
    compact_groups<<<(int)(b < 1 ? 1 : b > (unsigned long long)(4 * num_sms) ? 4 * num_sms : b), kThreads, 0, s>>>(D);
  }
  return cudaGetLastError();
}

}  // namespace gpl
