// kernel_fused.cu -- placeholder; the fused cycle kernel lands in the next commit.
#include "kernels.h"
namespace hydro {
void launch_cycle_fused(const DomView &, const Phys &, DevState *, cudaStream_t) {}
}  // namespace hydro
