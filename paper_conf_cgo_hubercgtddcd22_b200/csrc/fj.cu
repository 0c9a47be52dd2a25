// fj.cu -- fork/join microbenchmark entry points (variant dispatch, the
// barrier-floor kernel, extern "C" API).  Runtime-mode variants are built in
// fj_variant.cu modules (one per GENERIC/CASCADE variant).
#include "fj_impl.cuh"

namespace gtr {
namespace fj {

template <class K> int run_variant(LaunchArgs &a);
template <class K> struct VariantOp {
    static int run(LaunchArgs &a) { return run_variant<K>(a); }
};

// Floor for one fork/join: 2 CTA barrier phases per iteration, no runtime.
template <int NT> __global__ void __launch_bounds__(NT) kernel_floor(int64_t iters, unsigned long long *out) {
    __shared__ uint64_t s[NT];
    uint64_t acc = 0;
    s[threadIdx.x] = threadIdx.x;
    for (int64_t r = 0; r < iters; r++) {
        __syncthreads();
        acc += s[(threadIdx.x + r) % NT];
        __syncthreads();
    }
    s[threadIdx.x] = acc;
    __syncthreads();
    if (threadIdx.x == 0) {
        uint64_t t = 0;
        for (int i = 0; i < NT; i++) t += s[i];
        out[blockIdx.x] = t;
    }
}

template <int NT> int run_floor(gtr_ctx *ctx, const gtr_launch_cfg *cfg, int64_t iters, uint64_t *d_out,
                                cudaStream_t s, gtr_variant_info *info) {
    const void *fn = reinterpret_cast<const void *>(&kernel_floor<NT>);
    int per_sm = 0;
    GTR_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, NT, 0));
    Launch L;
    L.block = NT;
    L.dyn_smem = 0;
    L.teams = cfg->num_teams > 0 ? cfg->num_teams : per_sm * ctx->num_sms;
    if (info) return fill_info<Cfg<NATIVE, PL_STACK, true, NT>>(fn, L, per_sm, info);
    kernel_floor<NT><<<L.teams, NT, 0, s>>>(iters, reinterpret_cast<unsigned long long *>(d_out));
    GTR_CUDA_TRY(cudaGetLastError());
    return GTR_OK;
}

inline int launch(LaunchArgs &a) {
    const gtr_launch_cfg *c = a.cfg;
    if (!valid_cfg(c) || c->mode == NATIVE) return valid_cfg(c) ? GTR_EUNSUPPORTED : GTR_EINVAL;
    const int fl = c->flags & F_BCAST_1BAR;
#define GTR_FJ_NT(NT)                                                                          \
    if (c->thread_limit == NT) {                                                               \
        if (fl && c->mode == SPMD) return dispatch_spmd<NT, F_BCAST_1BAR, VariantOp>(c->placement, c->fold, a); \
        return dispatch_mpf<NT, 0, VariantOp>(c->mode, c->placement, c->fold, a);              \
    }
    GTR_FJ_NT(32)
    GTR_FJ_NT(128)
    GTR_FJ_NT(256)
    GTR_FJ_NT(512)
#undef GTR_FJ_NT
    return GTR_EUNSUPPORTED;
}

}  // namespace fj
}  // namespace gtr

using namespace gtr;

int gtr_internal_query_fj(gtr_ctx *ctx, const gtr_launch_cfg *cfg, gtr_variant_info *info, int floor) {
    if (floor) {
        if (!cfg) return GTR_EINVAL;
        switch (cfg->thread_limit) {
        case 32: return fj::run_floor<32>(ctx, cfg, 0, nullptr, nullptr, info);
        case 128: return fj::run_floor<128>(ctx, cfg, 0, nullptr, nullptr, info);
        case 256: return fj::run_floor<256>(ctx, cfg, 0, nullptr, nullptr, info);
        case 512: return fj::run_floor<512>(ctx, cfg, 0, nullptr, nullptr, info);
        case 1024: return fj::run_floor<1024>(ctx, cfg, 0, nullptr, nullptr, info);
        default: return GTR_EUNSUPPORTED;
        }
    }
    fj::LaunchArgs a{ctx, cfg, fj::Params{}, nullptr, info, false};
    return fj::launch(a);
}

extern "C" int gtr_forkjoin(gtr_ctx *ctx, const gtr_launch_cfg *cfg, int64_t regions, int32_t body,
                            int32_t n_distinct, uint64_t *d_out, void *stream) {
    if (!ctx || !cfg || !d_out || regions < 0 || body < 0 || body > 2 || n_distinct < 1 || n_distinct > 16)
        return GTR_EINVAL;
    fj::Params P;
    P.R = regions;
    P.body = body;
    P.K = n_distinct;
    P.out = reinterpret_cast<unsigned long long *>(d_out);
    P.heavy_buf = nullptr;
    fj::LaunchArgs a{ctx, cfg, P, static_cast<cudaStream_t>(stream), nullptr, false};
    return fj::launch(a);
}

extern "C" int gtr_barrier_floor(gtr_ctx *ctx, const gtr_launch_cfg *cfg, int64_t iters, uint64_t *d_out,
                                 void *stream) {
    if (!ctx || !cfg || !d_out || iters < 0) return GTR_EINVAL;
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    switch (cfg->thread_limit) {
    case 32: return fj::run_floor<32>(ctx, cfg, iters, d_out, s, nullptr);
    case 128: return fj::run_floor<128>(ctx, cfg, iters, d_out, s, nullptr);
    case 256: return fj::run_floor<256>(ctx, cfg, iters, d_out, s, nullptr);
    case 512: return fj::run_floor<512>(ctx, cfg, iters, d_out, s, nullptr);
    case 1024: return fj::run_floor<1024>(ctx, cfg, iters, d_out, s, nullptr);
    default: return GTR_EUNSUPPORTED;
    }
}
