// K3: level-set updatePartials for the 61-state codon model (placeholder
// until the tensor-core path lands).
#include <cuda_runtime.h>

#include "rrl_internal.h"

namespace rrl {

int launch_update_partials_codon(int, int, const DevOp *, const DevOp *, int, int, int, void *) {
  return (int)cudaErrorNotSupported;
}

}  // namespace rrl
