// pipeline.cu — generic (precompiled) instantiation of the fused probe-segment
// kernel (pipeline_body.cuh) and its launcher. The launcher prefers the
// plan-specialised NVRTC build of the same body (jit.cpp) when available.
#include <algorithm>

#include "kernels.h"
#include "pipeline_body.cuh"

namespace gpl {
namespace {

__global__ void __launch_bounds__(pipe::kMaxThreads, 1) pipeline_kernel(const __grid_constant__ PipeDesc d) {
  pipe::pipeline_body(d);
}

// Zero a list of 8-byte-granular ranges in one launch (a query's DIRECT
// tables, their tile counters and the run's counters + partials): one graph
// node instead of one memset per segment.
__global__ void __launch_bounds__(256) clear_ranges_kernel(const __grid_constant__ ClearList L) {
  grid_dep_launch_dependents();  // the first build may be scheduled early (it waits for us)
  for (int r = 0; r < L.n; r++) {
    unsigned long long* p = (unsigned long long*)L.ptr[r];
    const unsigned long long n8 = L.bytes[r] / 8;
    // 16-B stores where the range allows, then the 8-B tail
    const bool a16 = ((unsigned long long)p & 15ull) == 0;
    const unsigned long long n16 = a16 ? n8 / 2 : 0;
    uint4* q = (uint4*)p;
    for (unsigned long long i = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; i < n16;
         i += (unsigned long long)gridDim.x * blockDim.x)
      q[i] = make_uint4(0u, 0u, 0u, 0u);
    for (unsigned long long i = n16 * 2 + (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; i < n8;
         i += (unsigned long long)gridDim.x * blockDim.x)
      p[i] = 0ull;
  }
}

// Result copy-out: device scratch words -> mapped pinned host memory, after
// the fused run (PDL: scheduled during the run's drain, waits for its end).
__global__ void __launch_bounds__(256) copyout_kernel(const unsigned long long* src, unsigned long long* dst, int words) {
  grid_dep_wait();
  for (int i = threadIdx.x; i < words; i += blockDim.x) dst[i] = __ldcg(src + i);
}

}  // namespace

cudaError_t launch_copyout(const unsigned long long* src, unsigned long long* host_dst, int words, cudaStream_t s) {
  const void* args_[] = {(const void*)&src, (const void*)&host_dst, (const void*)&words};
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(1);
  cfg.blockDim = dim3(256);
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  return cudaLaunchKernelExC(&cfg, (const void*)copyout_kernel, (void**)args_);
}

cudaError_t launch_clear(const ClearList& L, int num_sms, cudaStream_t s) {
  if (L.n <= 0) return cudaSuccess;
  unsigned long long total = 0;
  for (int r = 0; r < L.n; r++) total += L.bytes[r];
  long long blocks = (long long)((total / 16 + 255) / 256);
  blocks = std::max<long long>(1, std::min<long long>(blocks, (long long)num_sms * 8));
  clear_ranges_kernel<<<(int)blocks, 256, 0, s>>>(L);
  return cudaGetLastError();
}

// jit.cpp: plan-specialised kernel for this descriptor's shape (nullptr if
// NVRTC is unavailable or disabled).
const void* jit_pipeline_kernel(const PipeDesc& d, std::string* err);

const void* resolve_pipeline_fn(const PipeDesc& d, bool use_jit, std::string* jit_err) {
  if (d.nwarps + 1 > pipe::kMaxWarps || d.depth > pipe::kMaxDepth || d.nsprobe > MAXSP || d.stage_rows % 128)
    return nullptr;
  const void* fn = nullptr;
  if (use_jit) fn = jit_pipeline_kernel(d, jit_err);
  // a register-field layout exists only in the plan-specialised kernel: no generic fallback
  if (!fn && d.reg_fields) return nullptr;
  if (!fn) {
    static int configured = 0;
    fn = (const void*)pipeline_kernel;
    if (d.smem_bytes > configured) {
      if (cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, d.smem_bytes) != cudaSuccess)
        return nullptr;
      configured = d.smem_bytes;
    }
  }
  return fn;
}

cudaError_t launch_pipeline_fn(const void* fn, const PipeDesc& d, int grid, cudaStream_t s) {
  void* args[] = {(void*)&d};
  // programmatic dependent launch: this grid may be scheduled while the
  // previous kernel of the stream drains (the body waits in grid_dep_wait)
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3((d.nwarps + 1) * 32);
  cfg.dynamicSmemBytes = (size_t)d.smem_bytes;
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  return cudaLaunchKernelExC(&cfg, fn, args);
}

cudaError_t launch_pipeline(const PipeDesc& d, int grid, cudaStream_t s, bool use_jit, std::string* jit_err) {
  const void* fn = resolve_pipeline_fn(d, use_jit, jit_err);
  if (!fn) return cudaErrorInvalidValue;
  return launch_pipeline_fn(fn, d, grid, s);
}

int pipeline_fixed_smem() { return 4096; }
int pipeline_max_consumer_warps() { return pipe::kMaxWarps - 1; }

}  // namespace gpl
