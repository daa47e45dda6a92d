// sag_ucd.cu -- group-kernel SA instantiations: UCDDCP, trace off, moves of <= 4 positions
// (sa_impl.cuh; one translation unit per variant so nvcc compiles them in parallel).
#include "sa_impl.cuh"

namespace cdd {
CDD_SAG_VARIANT(sag_ucd, true, false, 0)
CDD_SAG_SYNC_VARIANT(sag_ucd, true, 0)
CDD_SAG_T0_VARIANT(sag_ucd, true)
}  // namespace cdd
