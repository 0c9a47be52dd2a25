// fj_variant.cu -- one module per runtime-mode variant of the fork/join
// benchmark (see xs_variant.cu and build.py).
#include "fj_impl.cuh"
#include "variant_inst.h"

namespace gtr {
namespace fj {
template <class K> int run_variant(LaunchArgs &a) { return OpRt<K>::run(a); }
#define GTR_INST(M, P, F, NT, FL) template int run_variant<Cfg<M, P, F, NT, FL>>(LaunchArgs &);
GTR_VARIANT_INSTANCES
}  // namespace fj
}  // namespace gtr
