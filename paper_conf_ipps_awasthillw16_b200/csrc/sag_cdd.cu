// sag_cdd.cu -- group-kernel SA instantiations: CDD, trace off, moves of <= 4 positions
// (sa_impl.cuh; one translation unit per variant so nvcc compiles them in parallel).
#include "sa_impl.cuh"

namespace cdd {
CDD_SAG_VARIANT(sag_cdd, false, false, 0)
CDD_SAG_SYNC_VARIANT(sag_cdd, false, 0)
CDD_SAG_T0_VARIANT(sag_cdd, false)
}  // namespace cdd
