// sem.cu -- entry points of the runtime semantic programs (sem_impl.cuh).
#include "sem_impl.cuh"

namespace gtr {
namespace sem {

template <class K> int run_variant(LaunchArgs &a);
template <class K> struct VariantOp {
    static int run(LaunchArgs &a) { return run_variant<K>(a); }
};

inline int launch(LaunchArgs &a) {
    const gtr_launch_cfg *c = a.cfg;
    if (!valid_cfg(c)) return GTR_EINVAL;
    if (c->mode == NATIVE) return GTR_EUNSUPPORTED;
    const int fl = c->flags & F_SEPARATE_GUARDS;
#define GTR_SEM_NT(NT)                                                                               \
    if (c->thread_limit == NT) {                                                                     \
        if (fl && c->mode == SPMD) return dispatch_spmd<NT, F_SEPARATE_GUARDS, VariantOp>(c->placement, c->fold, a); \
        return dispatch_mpf<NT, 0, VariantOp>(c->mode, c->placement, c->fold, a);                    \
    }
    GTR_SEM_NT(64)
    GTR_SEM_NT(128)
#undef GTR_SEM_NT
    return GTR_EUNSUPPORTED;
}

}  // namespace sem
}  // namespace gtr

using namespace gtr;

int gtr_internal_query_sem(gtr_ctx *ctx, const gtr_launch_cfg *cfg, gtr_variant_info *info) {
    sem::LaunchArgs a{ctx, cfg, sem::Params{}, nullptr, info};
    return sem::launch(a);
}

extern "C" int gtr_semantics(gtr_ctx *ctx, const gtr_launch_cfg *cfg, int32_t test_id, uint64_t *d_out,
                             int64_t out_len, void *stream) {
    if (!ctx || !cfg || !d_out || test_id < 0 || test_id > 8 || out_len < 0) return GTR_EINVAL;
    sem::Params P;
    P.test = test_id;
    P.T = cfg->thread_limit;
    P.out = reinterpret_cast<unsigned long long *>(d_out);
    P.out_len = out_len;
    sem::LaunchArgs a{ctx, cfg, P, static_cast<cudaStream_t>(stream), nullptr};
    return sem::launch(a);
}
