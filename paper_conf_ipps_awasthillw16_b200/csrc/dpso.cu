// dpso.cu -- discrete PSO (placeholder until the swarm kernel lands).
#include "internal.h"

namespace cdd {
size_t dpso_workspace_bytes(const Instance&, const DpsoLaunch&) { return 256; }
cudaError_t launch_dpso(Instance&, const DpsoLaunch&, void*, cudaStream_t) {
    return cudaErrorNotSupported;
}
}  // namespace cdd
