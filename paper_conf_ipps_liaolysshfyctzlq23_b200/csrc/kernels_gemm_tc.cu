// tcgen05 / TMEM / TMA GEMM for bf16 mode (sm_100a).  Placeholder until the
// tensor-core path lands: returning false routes to the SIMT GEMM.
#include "kernels.h"
namespace mimose {
bool gemm_tc(Epi, const GemmArgs&, cudaStream_t) { return false; }
bool tc_available() { return false; }
}  // namespace mimose
