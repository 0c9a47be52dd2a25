// su3_impl.cuh -- SU3Bench mat_nn (BASELINE config 3) on the team runtime.
//
// Paper: SU3Bench version 0, the CPU-style OpenMP implementation, runs in
// generic mode with "a very lightweight parallel region" (P:933-944,
// P:1012-1013); 4 globalized variables (Fig. 9).
// Kernel shape (AMB-9): `teams distribute` over lattice sites; per site the
// main thread forks a `parallel for` over the 36 (link j, row k, column l)
// outputs, each computed as a 3-term complex multiply-accumulate
//   C[s][j][k][l] = sum_m A[s][j][k][m] * B[j][m][l]
// with 4 complex temporaries (accumulator, a, b, product) whose addresses are
// taken by the complex operators -> globalized (AMB-7).  fp64 (AMB-8); every
// product rounded before the add/sub (this TU: -fmad=false).
#pragma once
#include "gtr_internal.h"

namespace gtr {
namespace su3 {

struct Params {
    const double2 *A;   // [sites][4][3][3]
    const double2 *B;   // [4][3][3]
    double2 *C;
    int64_t sites;
};
static __shared__ Params g_p;

struct TagCC {};
struct TagA {};
struct TagB {};
struct TagP {};

// complex operators on globalized temporaries (address-taken, as C++ operator
// overloads taking references are)
__device__ __forceinline__ void cmul(double *p, const double *a, const double *b) {
    const double rr = a[0] * b[0], ii = a[1] * b[1], ri = a[0] * b[1], ir = a[1] * b[0];
    p[0] = rr - ii;
    p[1] = ri + ir;
}
__device__ __forceinline__ void cadd_to(double *acc, const double *p) {
    acc[0] = acc[0] + p[0];
    acc[1] = acc[1] + p[1];
}

// one output element e = (j, k, l) of site s
template <class K> __device__ __forceinline__ void element(const Params &P, int64_t s, int e) {
    const int j = e / 9, k = (e / 3) % 3, l = e % 3;
    Local<K, double, 2, TagCC> cc;
    Local<K, double, 2, TagA> a;
    Local<K, double, 2, TagB> b;
    Local<K, double, 2, TagP> p;
    cc[0] = 0.0;
    cc[1] = 0.0;
#pragma unroll
    for (int m = 0; m < 3; m++) {
        const double2 av = __ldg(P.A + ((s * 4 + j) * 3 + k) * 3 + m);
        const double2 bv = __ldg(P.B + (j * 3 + m) * 3 + l);
        a[0] = av.x; a[1] = av.y;
        b[0] = bv.x; b[1] = bv.y;
        cmul(p.ptr(), a.ptr(), b.ptr());
        cadd_to(cc.ptr(), p.ptr());
    }
    P.C[((s * 4 + j) * 3 + k) * 3 + l] = make_double2(cc[0], cc[1]);
}

struct Site {
    int64_t s;
};
struct TagSite {};

template <class K> struct SiteRegion {
    static constexpr int ID = 1;
    static __device__ void run(void *a) {
        const int64_t s = static_cast<const Site *>(a)->s;
        for_static<K>(0, 36, [&](int64_t e) { element<K>(g_p, s, (int)e); });
    }
};

template <class K> __global__ void __launch_bounds__(K::BLOCK) kernel_rt(Params P, RtParams rp) {
    const Role role = team_init<K>(rp);
    if (role == Role::Exit) return;
    if (role == Role::Worker) {
        worker_loop<K, SiteRegion<K>>();
        return;
    }
    guarded<K>([&] { g_p = P; });
    for (int64_t s = team_num<K>(); s < P.sites; s += num_teams<K>()) {   // teams distribute
        TeamLocal<K, Site, TagSite> site;
        site.set([&](Site &x) { x.s = s; });
        parallel<K, SiteRegion<K>>(site.get());
    }
    team_deinit<K>();
}

struct LaunchArgs {
    gtr_ctx *ctx;
    const gtr_launch_cfg *cfg;
    Params P;
    int32_t iters;
    cudaStream_t stream;
    gtr_variant_info *info;
};

template <class K> struct OpRt {
    static int run(LaunchArgs &a) {
        const void *fn = reinterpret_cast<const void *>(&kernel_rt<K>);
        Launch L;
        int st = resolve<K>(a.ctx, a.cfg, fn, 80, &L);
        if (st) return st;
        if (a.info) {
            int per_sm = 0;
            GTR_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, K::BLOCK, L.dyn_smem));
            return fill_info<K>(fn, L, per_sm, a.info);
        }
        for (int32_t it = 0; it < a.iters; it++)
            kernel_rt<K><<<L.teams, L.block, L.dyn_smem, a.stream>>>(a.P, L.rp);
        GTR_CUDA_TRY(cudaGetLastError());
        return GTR_OK;
    }
};

}  // namespace su3
}  // namespace gtr
