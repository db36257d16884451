// pipeline.cu — A2-A8: the fused, warp-specialised, persistent probe-segment
// kernel for sm_100a.
//
// GPL's segment = concurrently running kernels connected by channels, fed one
// tile at a time (§3.1, §3.3, §3.4,
// P:191-203 §3.5). The B200 re-expression is ONE kernel per segment:
//
//   producer warp (lane 0)                     consumer warps (W per CTA)
//   ----------------------                     -------------------------------------------
//   claim tile t = atomicAdd(counter)   A2     wait full[slot]
//   for each stage of the tile:                for each 32-row packet of the stage:
//     wait empty[slot]                           filters (selection = map only)  A4
//     cp.async.bulk every column       A3        stage-phase probes (first `nsprobe`)     A5
//       (TMA engine, L2 evict_first)             ballot/popc compaction -> warp queue     A8
//     arrive.expect_tx full[slot]                whenever >= 32 survivors are queued:
//                                                  remaining probes, where, group-by,   A5-A7
//                                                  exact int64 aggregation
//                                              arrive empty[slot]
//
// The ring of `depth` stages replaces the paper's "number of channels" n and
// a 32-row warp packet replaces its packet size p. Survivors travel
// through per-warp shared-memory queues carrying their values, so no
// operator writes an intermediate to HBM; the only global writes
// are the few-KB aggregate partials (int128) and counters.
#include <climits>

#include "device_common.cuh"
#include "kernels.h"

namespace gpl {
namespace {

constexpr int kMaxWarps = 17;  // 16 consumers + 1 producer
constexpr int kMaxThreads = kMaxWarps * 32;
constexpr int kMaxDepth = 8;
// fixed shared-memory region (see PipeDesc.off_*):
constexpr int kOffFull = 0;       // unsigned long long[kMaxDepth]
constexpr int kOffEmpty = 64;     // unsigned long long[kMaxDepth]
constexpr int kOffHdr = 128;      // int4[kMaxDepth]
constexpr int kOffHtp = 256;      // HTP[MAXHT]
constexpr int kOffCnt = 1024;     // unsigned long long[kMaxWarps][MAXOPS]
static_assert(kOffHtp + MAXHT * sizeof(HTP) <= kOffCnt, "HTP region overflow");

__device__ __forceinline__ unsigned lanemask_lt() {
  unsigned m;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}

__device__ __forceinline__ long long ld_stage(const PipeDesc& d, const char* sb, int c, int r) {
  const char* p = sb + d.coloff[c];
  return d.colw[c] == 4 ? (long long)((const int*)p)[r] : ((const long long*)p)[r];
}

__device__ __forceinline__ long long sel4(const long long (&s)[MAXP], int i) {
  long long v = s[0];
#pragma unroll
  for (int k = 1; k < MAXP; k++) v = (i == k) ? s[k] : v;
  return v;
}

// Queue phase on one packet of up to 32 queued survivors: lane `lane` owns
// queue entry `idx` (valid iff `pass`). Runs the remaining probes, the where
// residuals, the group-by and the aggregation (A5-A7).
__device__ __forceinline__ void drain(const PipeDesc& d, const HTP* htp, long long* q, int idx, bool pass,
                                      unsigned long long* cnt, long long (&acc)[MAXA], unsigned long long* stab,
                                      int lane) {
  int op = d.nfilt + d.nsprobe;
  for (int p = d.nsprobe; p < d.nprobe; p++, op++) {
    const Probe& P = d.probe[p];
    if (__any_sync(0xffffffffu, pass)) {
      if (pass) {
        unsigned long long k = (uint32_t)q[P.k1 * QCAP + idx];
        if (P.k2 >= 0) k = (k << 32) | (uint32_t)q[P.k2 * QCAP + idx];
        long long v = 0;
        const bool hit = ht_probe(htp[P.ht], k, &v);
        if (P.kind == P_MARK) {
          q[P.out * QCAP + idx] = hit ? 1 : 0;
        } else {
          pass = hit;
          if (hit && P.out >= 0) q[P.out * QCAP + idx] = v;
        }
      }
    }
    const unsigned m = __ballot_sync(0xffffffffu, pass);
    if (lane == 0) cnt[op] += __popc(m);
  }
  for (int r = 0; r < d.nresid; r++, op++) {
    const Resid& R = d.resid[r];
    if (pass) {
      const long long a = q[R.a * QCAP + idx];
      if (R.kind == R_EQ) {
        pass = a == q[R.b * QCAP + idx];
      } else if (R.kind == R_PAIRS) {
        const long long b = q[R.b * QCAP + idx];
        bool ok = false;
        for (int i = 0; i < R.npairs; i++) ok |= (a == R.pa[i]) & (b == R.pb[i]);
        pass = ok;
      } else if (R.kind == R_RANGE) {
        pass = a >= R.lo && a <= R.hi;
      } else {
        pass = (unsigned long long)a < 64ull && ((R.mask >> a) & 1ull);
      }
    }
    const unsigned m = __ballot_sync(0xffffffffu, pass);
    if (lane == 0) cnt[op] += __popc(m);
  }
  if (!__any_sync(0xffffffffu, pass)) return;
  int gid = 0;
  if (pass) {
    for (int g = 0; g < d.ngroup; g++) {
      const GroupDim& G = d.gdim[g];
      long long v = q[G.field * QCAP + idx];
      if (G.transform == G_YEAR) v = (int)v / 10000;
      const long long o = v - G.lo;
      if ((unsigned long long)o >= (unsigned long long)G.size) {
        atomicOr(d.err, ERR_DOMAIN);
        pass = false;
      }
      gid += (int)o * G.stride;
    }
  }
  long long val = 0;
  for (int t = 0; t < d.nterm; t++) {
    const Term& T = d.term[t];
    long long prod = T.sign;
    for (int f = 0; f < T.nfact; f++) {
      const Factor& F = T.f[f];
      const long long x = F.field < 0 ? F.a : F.a + (long long)F.b * q[F.field * QCAP + idx];
      prod *= x;
    }
    val += prod;
  }
  if (!pass) return;
  if (d.agg_mode == AGG_REG) {
#pragma unroll
    for (int a = 0; a < MAXA; a++) {
      if (a < d.nagg) {
        const Agg& A = d.agg[a];
        long long c = 1;
        if (A.kind == A_SUM) c = val;
        else if (A.kind == A_SUMIF) c = q[A.field * QCAP + idx] != 0 ? val : 0;
        else if (A.kind == A_SUMIFEQ) c = q[A.field * QCAP + idx] == A.c ? val : 0;
        acc[a] += c;
      }
    }
  } else {
    for (int a = 0; a < d.nagg; a++) {
      const Agg& A = d.agg[a];
      long long c = 1;
      if (A.kind == A_SUM) c = val;
      else if (A.kind == A_SUMIF) c = q[A.field * QCAP + idx] != 0 ? val : 0;
      else if (A.kind == A_SUMIFEQ) c = q[A.field * QCAP + idx] == A.c ? val : 0;
      if (c == 0) continue;
      if (d.agg_mode == AGG_SMEM) atomicAdd(&stab[gid * d.nagg + a], (unsigned long long)c);
      else atomic_add_i128(d.partials + 2 * (gid * d.nagg + a), c);
    }
  }
}

__device__ __forceinline__ void flush_reg(const PipeDesc& d, long long (&acc)[MAXA], int lane) {
#pragma unroll
  for (int a = 0; a < MAXA; a++) {
    if (a < d.nagg) {
      const long long s = warp_sum_i64(acc[a]);
      if (lane == 0 && s != 0) atomic_add_i128(d.partials + 2 * a, s);
      acc[a] = 0;
    }
  }
}

__global__ void __launch_bounds__(kMaxThreads, 1) pipeline_kernel(const __grid_constant__ PipeDesc d) {
  extern __shared__ __align__(128) unsigned char smem[];
  unsigned long long* full = (unsigned long long*)(smem + kOffFull);
  unsigned long long* empty = (unsigned long long*)(smem + kOffEmpty);
  int4* hdr = (int4*)(smem + kOffHdr);
  HTP* htp = (HTP*)(smem + kOffHtp);
  unsigned long long* cnt_all = (unsigned long long*)(smem + kOffCnt);
  unsigned long long* stab = (unsigned long long*)(smem + d.off_agg);
  char* ring = (char*)(smem + d.off_ring);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int W = d.nwarps;

  if (threadIdx.x == 0) {
    for (int i = 0; i < d.depth; i++) {
      mbar_init(&full[i], 1);
      mbar_init(&empty[i], (uint32_t)W);
    }
    fence_mbar_init();
  }
  if (threadIdx.x < d.nht) htp[threadIdx.x] = load_htp(d.ht[threadIdx.x]);
  for (int i = threadIdx.x; i < kMaxWarps * MAXOPS; i += blockDim.x) cnt_all[i] = 0;
  if (d.agg_mode == AGG_SMEM)
    for (int i = threadIdx.x; i < d.ngroups_total * d.nagg; i += blockDim.x) stab[i] = 0;
  __syncthreads();

  if (warp == W) {
    // ------------------------------------------------------------ producer
    if (lane == 0) {
      const unsigned long long pol = policy_evict_first();
      uint32_t slot = 0, phase = 0;
      for (;;) {
        const unsigned long long t = atomicAdd(d.tile_counter, 1ull);
        const long long r0 = (long long)t * d.tile_rows;
        if (r0 >= d.nrows) break;
        const long long rn = min(d.tile_rows, d.nrows - r0);
        for (long long s0 = 0; s0 < rn; s0 += d.stage_rows) {
          const int n = (int)min((long long)d.stage_rows, rn - s0);
          mbar_wait(&empty[slot], phase ^ 1u);
          const long long row = r0 + s0;
          hdr[slot] = make_int4((int)(row & 0xffffffff), (int)(row >> 32), n, (s0 + d.stage_rows >= rn) ? 1 : 0);
          uint32_t bytes = 0;
          for (int c = 0; c < d.ncols; c++) bytes += ((uint32_t)n * d.colw[c] + 15u) & ~15u;
          mbar_arrive_expect_tx(&full[slot], bytes);
          char* dst = ring + (size_t)slot * d.slot_bytes;
          for (int c = 0; c < d.ncols; c++)
            bulk_g2s(dst + d.coloff[c], d.col[c] + row * d.colw[c], ((uint32_t)n * d.colw[c] + 15u) & ~15u,
                     &full[slot], pol);
          if (++slot == (uint32_t)d.depth) { slot = 0; phase ^= 1u; }
        }
      }
      mbar_wait(&empty[slot], phase ^ 1u);
      hdr[slot] = make_int4(0, 0, -1, 0);
      mbar_arrive(&full[slot]);
    }
    return;
  }

  // -------------------------------------------------------------- consumers
  unsigned long long* cnt = cnt_all + warp * MAXOPS;
  long long* q = (long long*)(smem + d.off_queue) + (size_t)warp * d.nfield * QCAP;
  long long acc[MAXA] = {0, 0, 0, 0};
  int qhead = 0, qcount = 0;
  uint32_t slot = 0, phase = 0;
  for (;;) {
    mbar_wait(&full[slot], phase);
    const int4 h = hdr[slot];
    const int n = h.z;
    if (n < 0) break;
    const char* sb = ring + (size_t)slot * d.slot_bytes;
    const int npk = (n + 31) >> 5;
    for (int pk = warp; pk < npk; pk += W) {
      const int r = (pk << 5) + lane;
      bool pass = r < n;
      for (int f = 0; f < d.nfilt; f++) {
        const Filt& F = d.filt[f];
        if (pass) pass = filt_pass(F, ld_stage(d, sb, F.ref, r));
        const unsigned m = __ballot_sync(0xffffffffu, pass);
        if (lane == 0) cnt[f] += __popc(m);
      }
      long long sreg[MAXP] = {0, 0, 0, 0};
#pragma unroll
      for (int p = 0; p < MAXP; p++) {
        if (p < d.nsprobe) {
          const Probe& P = d.probe[p];
          if (__any_sync(0xffffffffu, pass)) {
            if (pass) {
              unsigned long long k = (uint32_t)ld_stage(d, sb, P.k1, r);
              if (P.k2 >= 0) k = (k << 32) | (uint32_t)ld_stage(d, sb, P.k2, r);
              long long v = 0;
              const bool hit = ht_probe(htp[P.ht], k, &v);
              if (P.kind == P_MARK) {
                sreg[p] = hit ? 1 : 0;
              } else {
                pass = hit;
                sreg[p] = v;
              }
            }
          }
          const unsigned m = __ballot_sync(0xffffffffu, pass);
          if (lane == 0) cnt[d.nfilt + p] += __popc(m);
        }
      }
      const unsigned mask = __ballot_sync(0xffffffffu, pass);
      if (mask) {
        if (pass) {
          const int idx = (qhead + qcount + __popc(mask & lanemask_lt())) & (QCAP - 1);
          for (int e = 0; e < d.npush; e++) {
            const Push& E = d.push[e];
            const long long v = E.kind == PUSH_COL ? ld_stage(d, sb, E.src, r) : sel4(sreg, E.src);
            q[e * QCAP + idx] = v;
          }
        }
        qcount += __popc(mask);
        if (qcount >= 32) {
          __syncwarp();
          drain(d, htp, q, (qhead + lane) & (QCAP - 1), true, cnt, acc, stab, lane);
          __syncwarp();
          qhead = (qhead + 32) & (QCAP - 1);
          qcount -= 32;
        }
      }
    }
    __syncwarp();
    if (lane == 0) mbar_arrive(&empty[slot]);
    if (d.flush_each_tile && h.w) flush_reg(d, acc, lane);
    if (++slot == (uint32_t)d.depth) { slot = 0; phase ^= 1u; }
  }
  if (qcount > 0) {
    __syncwarp();
    drain(d, htp, q, (qhead + lane) & (QCAP - 1), lane < qcount, cnt, acc, stab, lane);
  }
  __syncwarp();
  if (d.agg_mode == AGG_REG) flush_reg(d, acc, lane);
  if (lane == 0) {
    const int nops = d.nfilt + d.nprobe + d.nresid;
    for (int o = 0; o < nops; o++)
      if (cnt[o]) atomicAdd(d.op_pass + o, cnt[o]);
  }
  if (d.agg_mode == AGG_SMEM) {
    named_bar_sync(1, (uint32_t)W * 32u);
    for (int i = threadIdx.x; i < d.ngroups_total * d.nagg; i += W * 32) {
      const long long v = (long long)stab[i];
      if (v != 0) atomic_add_i128(d.partials + 2 * i, v);
    }
  }
}

}  // namespace

cudaError_t launch_pipeline(const PipeDesc& d, int grid, cudaStream_t s) {
  static int configured = 0;
  if (d.smem_bytes > configured) {
    cudaError_t e = cudaFuncSetAttribute(pipeline_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, d.smem_bytes);
    if (e != cudaSuccess) return e;
    configured = d.smem_bytes;
  }
  if (d.nwarps + 1 > kMaxWarps || d.depth > kMaxDepth) return cudaErrorInvalidValue;
  pipeline_kernel<<<grid, (d.nwarps + 1) * 32, d.smem_bytes, s>>>(d);
  return cudaGetLastError();
}

int pipeline_fixed_smem() { return kOffCnt + kMaxWarps * MAXOPS * 8; }
int pipeline_max_consumer_warps() { return kMaxWarps - 1; }

}  // namespace gpl
