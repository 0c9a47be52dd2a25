// fj_impl.cuh -- fork/join microbenchmark (BASELINE config 2) on the team
// runtime.  Isolates the costs the paper attributes to generic-mode execution:
// "diverging control flow and synchronization required by the state machine"
// (P:679-680), the function-pointer hand-off and indirect call (P:613-625,
// P:625-678), the register cost of address-taken regions (fn. 4),
// and the guard/broadcast barriers of SPMD-ized code.
//
// Program of team g (oracle/forkjoin.c; SURVEY.md 8(a') "Fork/join bench"):
//   for r < R:  [body 2: v = g*R + ctr; ctr += 1  -- a side effect producing a
//               value, so SPMD needs guard + broadcast]
//               args = {r, v}                     (globalized team variable)
//               parallel region k = r mod K       (K distinct regions, 1..16)
//               [body 0: count += 1]
//   team result = count (body 0) or sum of the workers' accumulators.
// A never-executed HEAVY region (many live fp64 values) is forked by a second
// kernel of the same module: GENERIC/CASCADE kernels, whose indirect call may
// reach any address-taken region, pay its registers; CSM/SPMD do not.
#pragma once
#include "gtr_internal.h"

namespace gtr {
namespace fj {

struct Params {
    int64_t R;
    int32_t body;
    int32_t K;
    unsigned long long *out;   // [num_teams]; out[g] doubles as team g's side-effect counter
    double *heavy_buf;
};
static __shared__ Params g_p;

struct Args {
    int64_t r;
    uint64_t v;
};
struct TagArgs {};

template <class K> __device__ __forceinline__ uint64_t *acc_slots() {
    __shared__ uint64_t acc[K::BLOCK];
    return acc;
}

// BODY is a compile-time property of the program (0 empty, 1 trivial,
// 2 broadcast) so an empty region is really empty after inlining.
template <class K, int BODY, int k> struct Region {
    static constexpr int ID = k + 1;
    static __device__ void run(void *a) {
        const Args *x = static_cast<const Args *>(a);
        if constexpr (BODY == 1) {
            const uint64_t t = (uint64_t)thread_num<K>();
            acc_slots<K>()[threadIdx.x] += (uint64_t)(k + 1) * (uint64_t)(x->r + 1) * (t + 1);
        } else if constexpr (BODY == 2) {
            acc_slots<K>()[threadIdx.x] += x->v;
        } else {
            (void)x;
        }
    }
};

// The heavy region: 48 live fp64 accumulators (never run by the benchmark).
template <class K> struct Heavy {
    static constexpr int ID = 17;
    static __device__ __noinline__ void run(void *a) {
        double *p = static_cast<double *>(a);
        double acc[48];
#pragma unroll
        for (int i = 0; i < 48; i++) acc[i] = p[i * 1024 + threadIdx.x];
        for (int it = 0; it < 64; it++) {
#pragma unroll
            for (int i = 0; i < 48; i++) acc[i] = acc[i] * acc[(i + 7) % 48] + acc[(i + 13) % 48];
        }
#pragma unroll
        for (int i = 0; i < 48; i++) p[i * 1024 + threadIdx.x] = acc[i];
    }
};

#define GTR_FJ_REGIONS(K, B)                                                                       \
    Region<K, B, 0>, Region<K, B, 1>, Region<K, B, 2>, Region<K, B, 3>, Region<K, B, 4>, Region<K, B, 5>, \
        Region<K, B, 6>, Region<K, B, 7>, Region<K, B, 8>, Region<K, B, 9>, Region<K, B, 10>,              \
        Region<K, B, 11>, Region<K, B, 12>, Region<K, B, 13>, Region<K, B, 14>, Region<K, B, 15>

template <class K, int B, int k> __device__ __forceinline__ void fork_k(int kk, void *a) {
    if constexpr (k < 16) {
        if (kk == k) parallel<K, Region<K, B, k>>(a);
        else fork_k<K, B, k + 1>(kk, a);
    }
}

// KMAX = 1: the team loop forks one region; KMAX = 16: region k = r mod K of
// up to 16 distinct regions (a switch in the sequential code).
template <class K, int BODY, int KMAX> __device__ __forceinline__ uint64_t team_program() {
    const int64_t R = g_p.R;
    const int KK = g_p.K;
    const uint64_t g = (uint64_t)team_num<K>();
    uint64_t count = 0;
    int kk = 0;                                   // r mod K, kept as a counter
    for (int64_t r = 0; r < R; r++) {
        uint64_t v = 0;
        if constexpr (BODY == 2)
            v = guarded_bcast<K, uint64_t>(
                [&] {
                    unsigned long long *ctr = &g_p.out[g];
                    uint64_t x = g * (uint64_t)R + *ctr;
                    *ctr += 1;
                    return x;
                });
        TeamLocal<K, Args, TagArgs> args;
        args.set([&](Args &x) {
            x.r = r;
            x.v = v;
        });
        if constexpr (KMAX == 1) {
            parallel<K, Region<K, BODY, 0>>(args.get());
        } else {
            fork_k<K, BODY, 0>(kk, args.get());
            kk = (kk + 1 == KK) ? 0 : kk + 1;
        }
        count += 1;
    }
    return count;
}

template <class K, int BODY, int KMAX>
__global__ void __launch_bounds__(K::BLOCK) kernel_fj(Params P, RtParams rp) {
    const Role role = team_init<K>(rp);
    if (role == Role::Exit) return;
    acc_slots<K>()[threadIdx.x] = 0;
    if (role == Role::Worker) {
        if constexpr (KMAX == 1) worker_loop<K, Region<K, BODY, 0>>();
        else worker_loop<K, GTR_FJ_REGIONS(K, BODY)>();
        return;
    }
    guarded<K>([&] { g_p = P; });
    const uint64_t count = team_program<K, BODY, KMAX>();
    // all regions joined: reduce the workers' accumulators
    guarded<K>([&] {
        uint64_t res = 0;
        if constexpr (BODY == 0) {
            res = count;
        } else {
            for (int t = 0; t < K::NT; t++) res += acc_slots<K>()[t];
        }
        g_p.out[team_num<K>()] = res;
    });
    team_deinit<K>();
}

// Second kernel of the module: forks the heavy region (takes its address in
// GENERIC / CASCADE).  Launched only on request.
template <class K> __global__ void __launch_bounds__(K::BLOCK) kernel_heavy(Params P, RtParams rp) {
    const Role role = team_init<K>(rp);
    if (role == Role::Exit) return;
    if (role == Role::Worker) {
        worker_loop<K, Heavy<K>>();
        return;
    }
    parallel<K, Heavy<K>>(P.heavy_buf);
    team_deinit<K>();
}

struct LaunchArgs {
    gtr_ctx *ctx;
    const gtr_launch_cfg *cfg;
    Params P;
    cudaStream_t stream;
    gtr_variant_info *info;
    bool heavy;
};

template <class K, int BODY, int KMAX> int launch_fj(LaunchArgs &a) {
    const void *fn = reinterpret_cast<const void *>(&kernel_fj<K, BODY, KMAX>);
    Launch L;
    int st = resolve<K>(a.ctx, a.cfg, fn, 64, &L);
    if (st) return st;
    if (a.info) {
        int per_sm = 0;
        GTR_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, K::BLOCK, L.dyn_smem));
        return fill_info<K>(fn, L, per_sm, a.info);
    }
    kernel_fj<K, BODY, KMAX><<<L.teams, L.block, L.dyn_smem, a.stream>>>(a.P, L.rp);
    GTR_CUDA_TRY(cudaGetLastError());
    return GTR_OK;
}

template <class K> struct OpRt {
    static int run(LaunchArgs &a) {
        if (a.heavy) {
            const void *fn = reinterpret_cast<const void *>(&kernel_heavy<K>);
            Launch L;
            int st = resolve<K>(a.ctx, a.cfg, fn, 64, &L);
            if (st) return st;
            kernel_heavy<K><<<L.teams, L.block, L.dyn_smem, a.stream>>>(a.P, L.rp);
            GTR_CUDA_TRY(cudaGetLastError());
            return GTR_OK;
        }
        const bool one = a.P.K == 1;
        switch (a.P.body) {
        case 0: return one ? launch_fj<K, 0, 1>(a) : launch_fj<K, 0, 16>(a);
        case 1: return one ? launch_fj<K, 1, 1>(a) : launch_fj<K, 1, 16>(a);
        default: return one ? launch_fj<K, 2, 1>(a) : launch_fj<K, 2, 16>(a);
        }
    }
};

}  // namespace fj
}  // namespace gtr
