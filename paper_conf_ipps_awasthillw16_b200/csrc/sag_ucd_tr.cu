// sag_ucd_tr.cu -- group-kernel SA instantiations: UCDDCP, trace on, moves of <= 4 positions
// (sa_impl.cuh; one translation unit per variant so nvcc compiles them in parallel).
#include "sa_impl.cuh"

namespace cdd {
CDD_SAG_VARIANT(sag_ucd_tr, true, true, 0)
}  // namespace cdd
