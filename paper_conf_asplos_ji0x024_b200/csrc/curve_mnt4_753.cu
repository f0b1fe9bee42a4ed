// Kernel instantiation for MNT4_753 (one translation unit per curve: parallel builds).
#include "ops_impl.cuh"

namespace msmrt {
CurveOps* make_ops_mnt4_753() {
  static Ops<MNT4_753_params> ops;
  return &ops;
}
}  // namespace msmrt
