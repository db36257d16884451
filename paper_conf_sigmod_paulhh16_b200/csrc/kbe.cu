// kbe.cu — placeholder until the KBE baseline lands.
#include "kernels.h"
namespace gpl {
cudaError_t run_kbe(const PipeDesc&, int, cudaStream_t, double* inter) {
  *inter = 0;
  return cudaErrorNotSupported;
}
}  // namespace gpl
