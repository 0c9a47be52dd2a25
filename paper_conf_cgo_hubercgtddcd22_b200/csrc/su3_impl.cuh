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
//
// GTR_F_TMA (B200-native form of the same program): `teams distribute` over
// tiles of 16 sites; the team's sequential code -- main thread (generic) or a
// guard (SPMD) -- issues bulk asynchronous copies (the TMA engine): the next
// tile's A into a second shared buffer while the current tile's parallel
// region runs, and the finished C tile back to HBM.  Regions read A and write C
// in shared memory; HBM traffic is whole-tile streaming.  Same arithmetic.
#pragma once
#include "gtr_internal.h"
#include "tma.cuh"

namespace gtr {
namespace su3 {

struct Params {
    const double2 *A;   // [sites][4][3][3]
    const double2 *B;   // [4][3][3]
    double2 *C;
    int64_t sites;
    int32_t tma;        // GTR_F_TMA: tile-streamed form
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

// one output element e = (j, k, l) of a site whose 36 A values start at
// `As` (global or shared) -> *out
template <class K, bool GLOBAL_A>
__device__ __forceinline__ void element_at(const double2 *As, const double2 *B, int e, double2 *out) {
    const int j = e / 9, k = (e / 3) % 3, l = e % 3;
    Local<K, double, 2, TagCC> cc;
    Local<K, double, 2, TagA> a;
    Local<K, double, 2, TagB> b;
    Local<K, double, 2, TagP> p;
    cc[0] = 0.0;
    cc[1] = 0.0;
#pragma unroll
    for (int m = 0; m < 3; m++) {
        const double2 av = GLOBAL_A ? __ldg(As + (j * 3 + k) * 3 + m) : As[(j * 3 + k) * 3 + m];
        const double2 bv = __ldg(B + (j * 3 + m) * 3 + l);
        a[0] = av.x; a[1] = av.y;
        b[0] = bv.x; b[1] = bv.y;
        cmul(p.ptr(), a.ptr(), b.ptr());
        cadd_to(cc.ptr(), p.ptr());
    }
    *out = make_double2(cc[0], cc[1]);
}
// one output element e = (j, k, l) of site s
template <class K> __device__ __forceinline__ void element(const Params &P, int64_t s, int e) {
    element_at<K, true>(P.A + s * 36, P.B, e, P.C + s * 36 + e);
}

// ---- GTR_F_TMA: tile buffers in dynamic shared memory after the runtime's area
constexpr int kTileSites = 16;
constexpr uint32_t kSiteBytes = 36 * 16;
struct TileBuf {
    double2 a[2][kTileSites * 36];   // double-buffered A tiles (TMA destinations)
    double2 c[kTileSites * 36];      // C tile (TMA store source)
    uint64_t bar[2];                 // completion barriers of the A buffers
};
template <class K> __device__ __forceinline__ TileBuf &tile_buf() {
    const uint32_t off = tstate_bytes<K>() + (uint32_t)K::BLOCK * g_ts.rp.sm_stride_words * 8u;
    return *reinterpret_cast<TileBuf *>(g_dyn + ((off + 127u) & ~127u));
}
struct TileArgs {
    int32_t ns;        // sites in this tile
    int32_t buf;       // A buffer
    uint32_t parity;   // phase parity of that buffer's barrier
};
struct TagTile {};
template <class K> struct TileRegion {
    static constexpr int ID = 2;
    static __device__ void run(void *a) {
        const TileArgs *t = static_cast<const TileArgs *>(a);
        TileBuf &tb = tile_buf<K>();
        tma::mbar_wait(&tb.bar[t->buf], t->parity, g_ts.rp.spin_limit, g_ts.rp.err, ERR_HANG);   // A tile landed
        const double2 *At = tb.a[t->buf];
        for_static<K>(0, (int64_t)t->ns * 36, [&](int64_t q) {
            const int site = (int)(q / 36), e = (int)(q - site * 36);
            element_at<K, false>(At + site * 36, g_p.B, e, &tb.c[q]);
        });
        tma::fence_async_shared();                               // C writes before the bulk store
    }
};
// the team's sequential program of the tiled form
template <class K> __device__ __forceinline__ void team_program_tma() {
    TileBuf &tb = tile_buf<K>();
    const int64_t ntiles = (g_p.sites + kTileSites - 1) / kTileSites;
    const int64_t t0 = team_num<K>(), G = num_teams<K>();
    auto tile_sites = [&](int64_t t) {
        return (int32_t)((t + 1) * kTileSites <= g_p.sites ? kTileSites : g_p.sites - t * kTileSites);
    };
    guarded<K>([&] {
        tma::mbar_init(&tb.bar[0]);
        tma::mbar_init(&tb.bar[1]);
        tma::fence_mbar_init();
        if (t0 < ntiles)
            tma::load_async(tb.a[0], g_p.A + t0 * kTileSites * 36, (uint32_t)tile_sites(t0) * kSiteBytes, &tb.bar[0]);
    });
    int i = 0;
    for (int64_t t = t0; t < ntiles; t += G, i++) {
        guarded<K>([&] {
            const int64_t tn = t + G;                            // prefetch the next tile
            if (tn < ntiles)
                tma::load_async(tb.a[(i + 1) & 1], g_p.A + tn * kTileSites * 36,
                                (uint32_t)tile_sites(tn) * kSiteBytes, &tb.bar[(i + 1) & 1]);
            tma::store_wait_read();                              // C buffer free again
        });
        TeamLocal<K, TileArgs, TagTile> args;
        args.set([&](TileArgs &x) {
            x.ns = tile_sites(t);
            x.buf = i & 1;
            x.parity = (uint32_t)((i >> 1) & 1);
        });
        parallel<K, TileRegion<K>>(args.get());
        guarded<K>([&] { tma::store_async(g_p.C + t * kTileSites * 36, tb.c, (uint32_t)tile_sites(t) * kSiteBytes); });
    }
    guarded<K>([&] { tma::store_wait_all(); });
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
        worker_loop<K, SiteRegion<K>, TileRegion<K>>();
        return;
    }
    guarded<K>([&] { g_p = P; });
    if (P.tma) {
        team_program_tma<K>();
        team_deinit<K>();
        return;
    }
    distribute_static<K>(0, P.sites, [&](int64_t s) {   // teams distribute
        TeamLocal<K, Site, TagSite> site;
        site.set([&](Site &x) { x.s = s; });
        parallel<K, SiteRegion<K>>(site.get());
    });
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
        int st = resolve<K>(a.ctx, a.cfg, fn, 80, &L, false, a.P.tma ? (uint32_t)sizeof(TileBuf) + 128u : 0u);
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
