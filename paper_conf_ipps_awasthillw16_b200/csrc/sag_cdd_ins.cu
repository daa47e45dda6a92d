// sag_cdd_ins.cu -- group-kernel SA instantiations: CDD, trace off, insertion move
// (sa_impl.cuh; one translation unit per variant so nvcc compiles them in parallel).
#include "sa_impl.cuh"

namespace cdd {
CDD_SAG_VARIANT(sag_cdd_ins, false, false, 1)
CDD_SAG_SYNC_VARIANT(sag_cdd_ins, false, 1)
}  // namespace cdd
