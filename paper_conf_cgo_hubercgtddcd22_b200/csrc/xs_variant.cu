// xs_variant.cu -- one module per runtime-mode variant of the XS lookup.
// Compiled once per (mode, placement, fold, thread_limit) for GENERIC and
// GENERIC_CASCADE (whose indirect calls see every address-taken region of the
// module), and once per thread_limit for the CSM + SPMD variants (no function
// pointers).  The build passes -DGTR_V_MODE=.. -DGTR_V_PL=.. -DGTR_V_FOLD=..
// -DGTR_V_NT=.. or -DGTR_V_GROUP_NT=..
#include "xs_impl.cuh"
#include "variant_inst.h"

namespace gtr {
namespace xs {
template <class K> int run_variant(LaunchArgs &a) { return OpRt<K>::run(a); }
#define GTR_INST(M, P, F, NT, FL) template int run_variant<Cfg<M, P, F, NT, FL>>(LaunchArgs &);
GTR_VARIANT_INSTANCES
}  // namespace xs
}  // namespace gtr
