// Kernel instantiation for BLS12_381 (one translation unit per curve: parallel builds).
#include "ops_impl.cuh"

namespace msmrt {
CurveOps* make_ops_bls12_381() {
  static Ops<BLS12_381_params> ops;
  return &ops;
}
}  // namespace msmrt
