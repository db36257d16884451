// kernels.h — host launchers of the sm_100a kernels (implemented in *.cu).
#pragma once
#include <cuda_runtime.h>

#include <string>

#include "common.h"

namespace gpl {

// Bytes of a DIRECT table (bitmap when width == 0), 4-byte granular.
inline unsigned long long direct_bytes(int width, unsigned long long nslots) {
  return width == 0 ? (nslots + 31) / 32 * 4
         : width == W_NIBBLE ? (nslots + 7) / 8 * 4
                             : (nslots * (unsigned long long)width + 3) / 4 * 4;
}

// A1 build segment. `trivial` (no filter, no probe): every row is inserted,
// so the host passes the exact header (count, key range, size) and the count
// pass is skipped. Otherwise: count pass (+ on-device sizing) -> clear -> insert.
cudaError_t launch_build(const BuildDesc& d, bool trivial, const HTHeader& known, int num_sms,
                         cudaStream_t s);

// Initialise a freshly allocated header (accumulators in their identity state).
cudaError_t launch_header_init(HTHeader* hdr, cudaStream_t s);

// A2-A8 fused persistent pipeline. d.smem_bytes of dynamic shared memory.
// use_jit: launch the plan-specialised NVRTC build of the kernel (compiled and
// cached on first use of a shape); falls back to the generic build when NVRTC
// is unavailable (reason in *jit_err).
cudaError_t launch_pipeline(const PipeDesc& d, int grid, cudaStream_t s, bool use_jit, std::string* jit_err);

// Resolve once (JIT or generic, dynamic-smem attribute set), then launch many times.
const void* resolve_pipeline_fn(const PipeDesc& d, bool use_jit, std::string* jit_err);
cudaError_t launch_pipeline_fn(const void* fn, const PipeDesc& d, int grid, cudaStream_t s);

// JIT: compile (and, when load is true, load) the specialised kernel for d's
// shape. Returns false with a message when NVRTC is unavailable or fails.
bool jit_prepare(const PipeDesc& d, bool load, std::string* err);
// NVRTC can be loaded (plan-specialised kernels are possible)
bool jit_available();

// Hash group-by result step (hashagg.cu): ORDER BY/LIMIT selection (D.limit
// > 0; D.nblocks = hagg_select_blocks(...) CTAs, D.cand sized nblocks*limit*5 words)
// or compaction of every group. Plain stream order after the fused run.
int hagg_select_blocks(unsigned long long nslots, int num_sms);
// Full device sort of n compacted rows (ORDER BY without LIMIT, else key
// order) into `out`: stable LSD radix passes over the sort words + a gather.
// tmp: sort_hagg_tmp_bytes(n) bytes.
size_t sort_hagg_tmp_bytes(unsigned long long n);
cudaError_t sort_hagg_rows(const HaggResultDesc& D, const unsigned long long* rows, unsigned long long n,
                           unsigned long long* out, void* tmp, int num_sms, cudaStream_t s);
cudaError_t launch_hagg_result(const HaggResultDesc& D, const unsigned long long* hagg_count, int num_sms,
                               cudaStream_t s);

// Zero up to 16 device ranges (8-byte granular sizes) in one kernel launch.
struct ClearList {
  void* ptr[16];
  unsigned long long bytes[16];
  int n;
};
cudaError_t launch_clear(const ClearList& L, int num_sms, cudaStream_t s);

// Copy `words` 8-byte words of device memory to mapped pinned host memory
// (one CTA; programmatic dependent launch after the fused run).
cudaError_t launch_copyout(const unsigned long long* src, unsigned long long* host_dst, int words, cudaStream_t s);

// Column min/max (int32 or int64 column, n rows) -> out[0] = min, out[1] = max.
// out[2] = number of descents (rows i with v[i] > v[i+1]): 0 means sorted.
cudaError_t launch_minmax(const void* col, int width, long long n, long long* out, cudaStream_t s);
// [lower_bound(lo), upper_bound(hi)) of a sorted column (one thread; out[2] device)
cudaError_t launch_sorted_bounds(const void* col, int w, long long n, long long lo, long long hi, long long* out,
                                 cudaStream_t s);
// partition phase (NEXT-4): exclusive scan of the [nparts][grid] counts into offsets + the row count
size_t part_scan_tmp_bytes(size_t n);
cudaError_t launch_part_scan(const unsigned* hist, unsigned* offs, size_t n, unsigned* total, void* tmp, size_t tmp_bytes,
                             cudaStream_t s);
// device scan scratch of a MULTI (fan-out) build over nslots keys
size_t multi_scan_tmp_bytes(unsigned long long nslots);
// per-column {min, max, descents} of one table's columns in two launches (A0 load)
cudaError_t launch_minmax_cols(const char* const* cols, const int* widths, int ncols, long long n, long long* out,
                               cudaStream_t s);

// KBE baseline: kernel-at-a-time with materialisation. Returns the
// bytes of intermediates written to HBM in *inter_bytes (host-side count).
// `pool` must hold kbe_pool_bytes(d) bytes (per-context, reused).
size_t kbe_pool_bytes(const PipeDesc& d, bool device_sized = false);
// device_bytes != nullptr: device-sized buffers, no host round trip (GPL w/o CE tiles); the
// materialised bytes accumulate in *device_bytes (device memory)
cudaError_t run_kbe(const PipeDesc& d, int num_sms, cudaStream_t s, void* pool, size_t pool_bytes, double* inter_bytes,
                    unsigned long long* device_bytes = nullptr);

}  // namespace gpl
