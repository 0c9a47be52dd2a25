// su3_variant.cu -- one module per runtime-mode variant of SU3 mat_nn
// (see xs_variant.cu and build.py).
#include "su3_impl.cuh"
#include "variant_inst.h"

namespace gtr {
namespace su3 {
template <class K> int run_variant(LaunchArgs &a) { return OpRt<K>::run(a); }
#define GTR_INST(M, P, F, NT, FL) template int run_variant<Cfg<M, P, F, NT, FL>>(LaunchArgs &);
GTR_VARIANT_INSTANCES
}  // namespace su3
}  // namespace gtr
