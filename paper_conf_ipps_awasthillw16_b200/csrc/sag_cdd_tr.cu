// sag_cdd_tr.cu -- group-kernel SA instantiations: CDD, trace on, moves of <= 4 positions
// (sa_impl.cuh; one translation unit per variant so nvcc compiles them in parallel).
#include "sa_impl.cuh"

namespace cdd {
CDD_SAG_VARIANT(sag_cdd_tr, false, true, 0)
}  // namespace cdd
