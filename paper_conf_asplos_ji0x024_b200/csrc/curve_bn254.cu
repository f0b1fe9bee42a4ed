// Kernel instantiation for BN254 (one translation unit per curve: parallel builds).
#include "ops_impl.cuh"

namespace msmrt {
CurveOps* make_ops_bn254() {
  static Ops<BN254_params> ops;
  return &ops;
}
}  // namespace msmrt
