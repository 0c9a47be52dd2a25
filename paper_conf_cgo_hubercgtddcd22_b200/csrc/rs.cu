// rs.cu -- RS lookup entry points: variant dispatch, the NATIVE (CUDA
// watermark) kernel and the extern "C" API.
#include "rs_impl.cuh"

namespace gtr {
namespace rs {

template <class K> int run_variant(LaunchArgs &a);
template <class K> struct VariantOp {
    static int run(LaunchArgs &a) { return run_variant<K>(a); }
};

template <int NT> __global__ void __launch_bounds__(NT) kernel_native(Params P) {
    using KN = Cfg<NATIVE, PL_STACK, true, NT>;
    __shared__ uint32_t tally[17];
    if (threadIdx.x < 17) tally[threadIdx.x] = 0;
    __syncthreads();
    const uint64_t stride = (uint64_t)gridDim.x * NT;
    for (uint64_t k = (uint64_t)blockIdx.x * NT + threadIdx.x; k < P.n; k += stride)
        lookup<KN>(P, P.first + k, tally);
    __syncthreads();
    flush(tally, P.out, threadIdx.x, NT);
}

template <int NT> int run_native(LaunchArgs &a) {
    const void *fn = reinterpret_cast<const void *>(&kernel_native<NT>);
    int per_sm = 0;
    GTR_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, NT, 0));
    Launch L;
    L.block = NT;
    L.dyn_smem = 0;
    L.teams = a.cfg->num_teams > 0 ? a.cfg->num_teams : per_sm * a.ctx->num_sms;
    if (a.info) return fill_info<Cfg<NATIVE, PL_STACK, true, NT>>(fn, L, per_sm, a.info);
    kernel_native<NT><<<L.teams, NT, 0, a.stream>>>(a.P);
    GTR_CUDA_TRY(cudaGetLastError());
    return GTR_OK;
}

template <int NT> int run_native_bucketed(LaunchArgs &a) {
    using KN = Cfg<NATIVE, PL_STACK, true, NT>;
    const void *fn = reinterpret_cast<const void *>(&kernel_native_bucketed<KN>);
    const uint32_t smem = (uint32_t)sizeof(ChunkBuf<KN>);
    GTR_CUDA_TRY(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    int per_sm = 0;
    GTR_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, NT, smem));
    if (per_sm < 1) return GTR_EINVAL;
    Launch L;
    L.block = NT;
    L.dyn_smem = smem;
    L.teams = a.cfg->num_teams > 0 ? a.cfg->num_teams : per_sm * a.ctx->num_sms;
    if (a.info) return fill_info<KN>(fn, L, per_sm, a.info);
    a.P.chunk = fit_chunk(a.P.n, kBucketLookupsPerThread * NT, L.teams);
    kernel_native_bucketed<KN><<<L.teams, NT, smem, a.stream>>>(a.P);
    GTR_CUDA_TRY(cudaGetLastError());
    return GTR_OK;
}

inline int launch(LaunchArgs &a) {
    const gtr_launch_cfg *c = a.cfg;
    if (!valid_cfg(c)) return GTR_EINVAL;
    a.P.plain = (c->flags & GTR_F_PLAIN) ? 1 : 0;
    if (c->mode == NATIVE && (c->flags & GTR_F_NATIVE_BUCKETED)) {
        if (a.P.plain) return GTR_EINVAL;
        if (c->thread_limit == 128) return run_native_bucketed<128>(a);
        return GTR_EUNSUPPORTED;
    }
    if (c->mode == NATIVE) {
        if (c->thread_limit == 128) return run_native<128>(a);
        if (c->thread_limit == 256) return run_native<256>(a);
        return GTR_EUNSUPPORTED;
    }
    if (c->thread_limit == 128) return dispatch_mpf<128, 0, VariantOp>(c->mode, c->placement, c->fold, a);
    return GTR_EUNSUPPORTED;
}

}  // namespace rs
}  // namespace gtr

using namespace gtr;

static rs::Params make_params(const gtr_rs_tables *t, uint64_t first, uint64_t n, uint64_t seed,
                              uint64_t *d_out, const gtr_rs_verify *v) {
    rs::Params P{};
    if (t) {
        P.n_windows = t->n_windows;
        P.poles = t->poles;
        P.windows = t->windows;
        P.k0rs = t->k0rs;
        P.num_nucs = t->num_nucs;
        P.mats = t->mats;
        P.concs = t->concs;
        P.poles_wide = t->poles_wide;
        P.wide = ((reinterpret_cast<uintptr_t>(t->windows) | reinterpret_cast<uintptr_t>(t->k0rs)) & 31u) == 0;
        P.n_nuc = t->n_nuc;
        P.max_poles = t->max_poles;
        P.max_windows = t->max_windows;
        P.max_num_nucs = t->max_num_nucs;
    }
    P.first = first;
    P.n = n;
    P.seed = seed;
    P.v_mat = v ? v->mat : nullptr;
    P.v_am = v ? v->am : nullptr;
    P.v_macro = v ? v->macro : nullptr;
    P.out = reinterpret_cast<unsigned long long *>(d_out);
    return P;
}

int gtr_internal_query_rs(gtr_ctx *ctx, const gtr_launch_cfg *cfg, gtr_variant_info *info) {
    rs::LaunchArgs a{ctx, cfg, make_params(nullptr, 0, 0, 0, nullptr, nullptr), nullptr, info};
    return rs::launch(a);
}

namespace gtr {
namespace rs {
// Words 9..11 hold the pole's lookup-invariant factors of exp(12 i Z)
// (Z = (E - EA)/2): |exp| = fast_exp(-12 Z.i) depends on EA.i only -- the
// same operations as the lookup would do, so the same bits -- and the phase
// factor exp(-6 i EA.r), which the lookup rotates by exp(6 i E).
__global__ void k_wide_poles(const double *__restrict__ poles, int64_t n_rec, double *__restrict__ out) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n_rec * 12;
         i += (int64_t)gridDim.x * blockDim.x) {
        const int64_t r = i / 12, w = i - r * 12;
        double v;
        if (w < 9) {
            v = __ldg(poles + r * 9 + w);
        } else if (w == 9) {
            const double zi = (0.0 - __ldg(poles + r * 9 + 1)) * 0.5;     // Z.i, exact
            v = fast_exp(-12.0 * zi);
        } else {
            double sp, cp;
            sincos(6.0 * __ldg(poles + r * 9 + 0), &sp, &cp);
            v = w == 10 ? cp : sp;
        }
        out[i] = v;
    }
}
}  // namespace rs
}  // namespace gtr

extern "C" int gtr_rs_build_wide_poles(gtr_ctx *ctx, const double *d_poles, int64_t n_records,
                                       double *d_poles_wide_out, void *stream) {
    if (!ctx || !d_poles || !d_poles_wide_out || n_records < 1 ||
        (reinterpret_cast<uintptr_t>(d_poles_wide_out) & 31u))
        return GTR_EINVAL;
    const int64_t blocks = (n_records * 12 + 255) / 256, cap = (int64_t)ctx->num_sms * 16;
    rs::k_wide_poles<<<(int)(blocks < cap ? blocks : cap), 256, 0, static_cast<cudaStream_t>(stream)>>>(
        d_poles, n_records, d_poles_wide_out);
    GTR_CUDA_TRY(cudaGetLastError());
    return GTR_OK;
}

extern "C" int gtr_rs_lookup(gtr_ctx *ctx, const gtr_launch_cfg *cfg, const gtr_rs_tables *t, uint64_t first,
                             uint64_t n, uint64_t seed, uint64_t *d_out, const gtr_rs_verify *verify,
                             void *stream) {
    if (!ctx || !cfg || !t || !d_out || !t->n_windows || !t->poles || !t->windows || !t->k0rs ||
        !t->num_nucs || !t->mats || !t->concs || t->n_nuc < 1 || t->max_poles < 1 || t->max_windows < 1 ||
        (reinterpret_cast<uintptr_t>(t->poles_wide) & 31u))
        return GTR_EINVAL;
    if (n == 0) return GTR_OK;
    rs::LaunchArgs a{ctx, cfg, make_params(t, first, n, seed, d_out, verify), static_cast<cudaStream_t>(stream),
                     nullptr};
    return rs::launch(a);
}

// ---------------------------------------------------------------- fp64 probe
// The fp64 ALU ceiling of the RS roofline, measured: every thread runs 8
// independent chains of `iters` DFMA (a = a*b + c, 2 flops each), 8 warps x
// 4 CTAs per SM.  d_out[0] receives a data-dependent sum (keeps the chains).
namespace gtr {
namespace rs {
__global__ void __launch_bounds__(256) kernel_fp64_probe(int64_t iters, double b, double c,
                                                         unsigned long long *out) {
    double a[8];
#pragma unroll
    for (int k = 0; k < 8; k++) a[k] = (double)(threadIdx.x + k) * 1e-3;
    for (int64_t i = 0; i < iters; i++) {
#pragma unroll
        for (int k = 0; k < 8; k++) a[k] = __fma_rn(a[k], b, c);
    }
    double s = 0.0;
#pragma unroll
    for (int k = 0; k < 8; k++) s += a[k];
    if (s == 12345.678) atomicAdd(out, 1ull);             // never true; keeps the work
}
}  // namespace rs
}  // namespace gtr

extern "C" int gtr_fp64_probe(gtr_ctx *ctx, int64_t iters, uint64_t *d_out, double *flops_per_launch,
                              void *stream) {
    if (!ctx || !d_out || iters < 1) return GTR_EINVAL;
    const int blocks = 4 * ctx->num_sms;
    rs::kernel_fp64_probe<<<blocks, 256, 0, static_cast<cudaStream_t>(stream)>>>(
        iters, 0.999999, 1e-7, reinterpret_cast<unsigned long long *>(d_out));
    GTR_CUDA_TRY(cudaGetLastError());
    if (flops_per_launch) *flops_per_launch = 2.0 * 8.0 * (double)iters * 256.0 * (double)blocks;
    return GTR_OK;
}
