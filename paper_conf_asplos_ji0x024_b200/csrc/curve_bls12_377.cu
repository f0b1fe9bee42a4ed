// Kernel instantiation for BLS12_377 (one translation unit per curve: parallel builds).
#include "ops_impl.cuh"

namespace msmrt {
CurveOps* make_ops_bls12_377() {
  static Ops<BLS12_377_params> ops;
  return &ops;
}
}  // namespace msmrt
