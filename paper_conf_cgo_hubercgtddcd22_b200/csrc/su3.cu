// su3.cu -- SU3 mat_nn entry points: variant dispatch, the NATIVE (CUDA
// watermark) kernel and the extern "C" API.
#include "su3_impl.cuh"

namespace gtr {
namespace su3 {

template <class K> int run_variant(LaunchArgs &a);
template <class K> struct VariantOp {
    static int run(LaunchArgs &a) { return run_variant<K>(a); }
};

// NATIVE: one thread per output element (site, j, k, l); consecutive threads
// write consecutive 16-byte complex values (coalesced), the 3 A values of a
// row are shared by 3 neighbouring threads through L1.
template <int NT> __global__ void __launch_bounds__(NT) kernel_native(Params P) {
    const int64_t total = P.sites * 36;
    for (int64_t t = (int64_t)blockIdx.x * NT + threadIdx.x; t < total; t += (int64_t)gridDim.x * NT) {
        const int64_t s = t / 36;
        const int e = (int)(t - s * 36);
        const int j = e / 9, k = (e / 3) % 3, l = e % 3;
        double re = 0.0, im = 0.0;
#pragma unroll
        for (int m = 0; m < 3; m++) {
            const double2 a = __ldg(P.A + ((s * 4 + j) * 3 + k) * 3 + m);
            const double2 b = __ldg(P.B + (j * 3 + m) * 3 + l);
            const double rr = a.x * b.x, ii = a.y * b.y, ri = a.x * b.y, ir = a.y * b.x;
            re = re + (rr - ii);
            im = im + (ri + ir);
        }
        P.C[t] = make_double2(re, im);
    }
}

// NATIVE, tile-streamed (GTR_F_TMA): persistent CTAs; thread 0 streams
// 16-site A tiles into a double buffer with bulk asynchronous copies (TMA) and
// C tiles back; the CTA computes each tile from shared memory.
template <int NT> __global__ void __launch_bounds__(NT) kernel_native_tma(Params P, uint32_t *err, uint64_t spin_limit) {
    extern __shared__ __align__(128) uint8_t dyn[];
    TileBuf &tb = *reinterpret_cast<TileBuf *>(dyn);
    const int64_t ntiles = (P.sites + kTileSites - 1) / kTileSites;
    auto tile_sites = [&](int64_t t) {
        return (uint32_t)((t + 1) * kTileSites <= P.sites ? kTileSites : P.sites - t * kTileSites);
    };
    if (threadIdx.x == 0) {
        tma::mbar_init(&tb.bar[0]);
        tma::mbar_init(&tb.bar[1]);
        tma::fence_mbar_init();
        if ((int64_t)blockIdx.x < ntiles)
            tma::load_async(tb.a[0], P.A + (int64_t)blockIdx.x * kTileSites * 36, tile_sites(blockIdx.x) * kSiteBytes,
                            &tb.bar[0]);
    }
    __syncthreads();
    int i = 0;
    for (int64_t t = blockIdx.x; t < ntiles; t += gridDim.x, i++) {
        if (threadIdx.x == 0) {
            const int64_t tn = t + gridDim.x;
            if (tn < ntiles)
                tma::load_async(tb.a[(i + 1) & 1], P.A + tn * kTileSites * 36, tile_sites(tn) * kSiteBytes,
                                &tb.bar[(i + 1) & 1]);
            tma::store_wait_read();
        }
        __syncthreads();
        tma::mbar_wait(&tb.bar[i & 1], (uint32_t)((i >> 1) & 1), spin_limit, err, ERR_HANG);
        const double2 *At = tb.a[i & 1];
        const int total = (int)tile_sites(t) * 36;
        for (int q = threadIdx.x; q < total; q += NT) {
            const int site = q / 36, e = q - site * 36;
            const int j = e / 9, k = (e / 3) % 3, l = e % 3;
            double re = 0.0, im = 0.0;
#pragma unroll
            for (int m = 0; m < 3; m++) {
                const double2 av = At[site * 36 + (j * 3 + k) * 3 + m];
                const double2 b = __ldg(P.B + (j * 3 + m) * 3 + l);
                const double rr = av.x * b.x, ii = av.y * b.y, ri = av.x * b.y, ir = av.y * b.x;
                re = re + (rr - ii);
                im = im + (ri + ir);
            }
            tb.c[q] = make_double2(re, im);
        }
        tma::fence_async_shared();
        __syncthreads();
        if (threadIdx.x == 0) tma::store_async(P.C + t * kTileSites * 36, tb.c, tile_sites(t) * kSiteBytes);
    }
    if (threadIdx.x == 0) tma::store_wait_all();
}

template <int NT> int run_native_tma(LaunchArgs &a) {
    const void *fn = reinterpret_cast<const void *>(&kernel_native_tma<NT>);
    const uint32_t smem = (uint32_t)sizeof(TileBuf);
    GTR_CUDA_TRY(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    int per_sm = 0;
    GTR_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, NT, smem));
    Launch L;
    L.block = NT;
    L.dyn_smem = smem;
    L.teams = a.cfg->num_teams > 0 ? a.cfg->num_teams : per_sm * a.ctx->num_sms;
    if (a.info) return fill_info<Cfg<NATIVE, PL_STACK, true, NT>>(fn, L, per_sm, a.info);
    for (int32_t it = 0; it < a.iters; it++)
        kernel_native_tma<NT><<<L.teams, NT, smem, a.stream>>>(a.P, a.ctx->d_err, a.ctx->spin_limit);
    GTR_CUDA_TRY(cudaGetLastError());
    return GTR_OK;
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
    for (int32_t it = 0; it < a.iters; it++) kernel_native<NT><<<L.teams, NT, 0, a.stream>>>(a.P);
    GTR_CUDA_TRY(cudaGetLastError());
    return GTR_OK;
}

inline int launch(LaunchArgs &a) {
    const gtr_launch_cfg *c = a.cfg;
    if (!valid_cfg(c)) return GTR_EINVAL;
    a.P.tma = (c->flags & GTR_F_TMA) ? 1 : 0;
    if (c->mode == NATIVE && a.P.tma) {
        if (c->thread_limit == 128) return run_native_tma<128>(a);
        if (c->thread_limit == 256) return run_native_tma<256>(a);
        if (c->thread_limit == 512) return run_native_tma<512>(a);
        return GTR_EUNSUPPORTED;
    }
    if (c->mode == NATIVE) {
        if (c->thread_limit == 128) return run_native<128>(a);
        if (c->thread_limit == 256) return run_native<256>(a);
        if (c->thread_limit == 512) return run_native<512>(a);
        return GTR_EUNSUPPORTED;
    }
    if (c->thread_limit == 64) return dispatch_mpf<64, 0, VariantOp>(c->mode, c->placement, c->fold, a);
    if (c->thread_limit == 128) return dispatch_mpf<128, 0, VariantOp>(c->mode, c->placement, c->fold, a);
    return GTR_EUNSUPPORTED;
}

}  // namespace su3
}  // namespace gtr

using namespace gtr;

int gtr_internal_query_su3(gtr_ctx *ctx, const gtr_launch_cfg *cfg, gtr_variant_info *info) {
    su3::LaunchArgs a{ctx, cfg, su3::Params{}, 0, nullptr, info};
    return su3::launch(a);
}

extern "C" int gtr_su3_mat_nn(gtr_ctx *ctx, const gtr_launch_cfg *cfg, const double *d_A, const double *d_B,
                              double *d_C, int64_t sites, int32_t iters, void *stream) {
    if (!ctx || !cfg || !d_A || !d_B || !d_C || sites < 0 || iters < 0) return GTR_EINVAL;
    if (sites == 0 || iters == 0) return GTR_OK;
    su3::Params P;
    P.A = reinterpret_cast<const double2 *>(d_A);
    P.B = reinterpret_cast<const double2 *>(d_B);
    P.C = reinterpret_cast<double2 *>(d_C);
    P.sites = sites;
    P.tma = 0;
    su3::LaunchArgs a{ctx, cfg, P, iters, static_cast<cudaStream_t>(stream), nullptr};
    return su3::launch(a);
}
