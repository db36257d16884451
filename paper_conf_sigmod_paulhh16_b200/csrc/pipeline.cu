// pipeline.cu — generic (precompiled) instantiation of the fused probe-segment
// kernel (pipeline_body.cuh) and its launcher. The launcher prefers the
// plan-specialised NVRTC build of the same body (jit.cpp) when available.
#include "kernels.h"
#include "pipeline_body.cuh"

namespace gpl {
namespace {

__global__ void __launch_bounds__(pipe::kMaxThreads, 1) pipeline_kernel(const __grid_constant__ PipeDesc d) {
  pipe::pipeline_body(d);
}

}  // namespace

// jit.cpp: plan-specialised kernel for this descriptor's shape (nullptr if
// NVRTC is unavailable or disabled).
const void* jit_pipeline_kernel(const PipeDesc& d, std::string* err);

const void* resolve_pipeline_fn(const PipeDesc& d, bool use_jit, std::string* jit_err) {
  if (d.nwarps + 1 > pipe::kMaxWarps || d.depth > pipe::kMaxDepth || d.nsprobe > MAXSP || d.stage_rows % 128)
    return nullptr;
  const void* fn = nullptr;
  if (use_jit) fn = jit_pipeline_kernel(d, jit_err);
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
  return cudaLaunchKernel(fn, dim3(grid), dim3((d.nwarps + 1) * 32), args, (size_t)d.smem_bytes, s);
}

cudaError_t launch_pipeline(const PipeDesc& d, int grid, cudaStream_t s, bool use_jit, std::string* jit_err) {
  const void* fn = resolve_pipeline_fn(d, use_jit, jit_err);
  if (!fn) return cudaErrorInvalidValue;
  return launch_pipeline_fn(fn, d, grid, s);
}

int pipeline_fixed_smem() { return 4096; }
int pipeline_max_consumer_warps() { return pipe::kMaxWarps - 1; }

}  // namespace gpl
