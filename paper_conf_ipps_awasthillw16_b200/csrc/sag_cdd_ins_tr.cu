// sag_cdd_ins_tr.cu -- group-kernel SA instantiations: CDD, trace on, insertion move
// (sa_impl.cuh; one translation unit per variant so nvcc compiles them in parallel).
#include "sa_impl.cuh"

namespace cdd {
CDD_SAG_VARIANT(sag_cdd_ins_tr, false, true, 1)
}  // namespace cdd
