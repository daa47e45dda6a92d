// sag_cdd_nib.cu -- group-kernel SA instantiation: CDD, trace off, moves of <= 4 positions on the nibble
// layout with sub-block summaries (sa_nib.cuh; G = 8, E = 128), asynchronous and synchronous SA.
#include "sa_impl.cuh"

namespace cdd {
CDD_SAG_NIB_VARIANT(sag_cdd_nib, false)
CDD_SAG_NIB_SYNC_VARIANT(sag_cdd_nib)
}  // namespace cdd
