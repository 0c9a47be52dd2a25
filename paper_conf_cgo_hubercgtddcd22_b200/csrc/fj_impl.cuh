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

template <class K, int k> struct Region {
    static constexpr int ID = k + 1;
    static __device__ void run(void *a) {
        const Args *x = static_cast<const Args *>(a);
        const int body = g_p.body;
        if (body == 1) {
            const uint64_t t = (uint64_t)thread_num<K>();
            acc_slots<K>()[threadIdx.x] += (uint64_t)(k + 1) * (uint64_t)(x->r + 1) * (t + 1);
        } else if (body == 2) {
            acc_slots<K>()[threadIdx.x] += x->v;
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

#define GTR_FJ_REGIONS(K)                                                                  \
    Region<K, 0>, Region<K, 1>, Region<K, 2>, Region<K, 3>, Region<K, 4>, Region<K, 5>,     \
        Region<K, 6>, Region<K, 7>, Region<K, 8>, Region<K, 9>, Region<K, 10>, Region<K, 11>, \
        Region<K, 12>, Region<K, 13>, Region<K, 14>, Region<K, 15>

template <class K, int k> __device__ __forceinline__ void fork_k(int kk, void *a) {
    if constexpr (k < 16) {
        if (kk == k) parallel<K, Region<K, k>>(a);
        else fork_k<K, k + 1>(kk, a);
    }
}

template <class K> __device__ __forceinline__ uint64_t team_program() {
    const int64_t R = g_p.R;
    const int body = g_p.body, KK = g_p.K;
    const uint64_t g = (uint64_t)team_num<K>();
    uint64_t count = 0;
    int kk = 0;                                   // r mod K, kept as a counter
    for (int64_t r = 0; r < R; r++) {
        uint64_t v = 0;
        if (body == 2)
            v = guarded_bcast<K, uint64_t>(
                [&] {
                    unsigned long long *ctr = &g_p.out[g];
                    uint64_t x = g * (uint64_t)R + *ctr;
                    *ctr += 1;
                    return x;
                },
                (int)(r & 1));
        TeamLocal<K, Args, TagArgs> args;
        args.set([&](Args &x) {
            x.r = r;
            x.v = v;
        });
        fork_k<K, 0>(kk, args.get());
        kk = (kk + 1 == KK) ? 0 : kk + 1;
        count += 1;
    }
    return count;
}

template <class K> __global__ void __launch_bounds__(K::BLOCK) kernel_fj(Params P, RtParams rp) {
    const Role role = team_init<K>(rp);
    if (role == Role::Exit) return;
    acc_slots<K>()[threadIdx.x] = 0;
    if (role == Role::Worker) {
        worker_loop<K, GTR_FJ_REGIONS(K)>();
        return;
    }
    guarded<K>([&] { g_p = P; });
    const uint64_t count = team_program<K>();
    // all regions joined: reduce the workers' accumulators
    guarded<K>([&] {
        uint64_t res = 0;
        if (g_p.body == 0) {
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

template <class K> struct OpRt {
    static int run(LaunchArgs &a) {
        const void *fn = a.heavy ? reinterpret_cast<const void *>(&kernel_heavy<K>)
                                 : reinterpret_cast<const void *>(&kernel_fj<K>);
        Launch L;
        int st = resolve<K>(a.ctx, a.cfg, fn, 64, &L);
        if (st) return st;
        if (a.info) {
            int per_sm = 0;
            GTR_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, K::BLOCK, L.dyn_smem));
            return fill_info<K>(fn, L, per_sm, a.info);
        }
        if (a.heavy)
            kernel_heavy<K><<<L.teams, L.block, L.dyn_smem, a.stream>>>(a.P, L.rp);
        else
            kernel_fj<K><<<L.teams, L.block, L.dyn_smem, a.stream>>>(a.P, L.rp);
        GTR_CUDA_TRY(cudaGetLastError());
        return GTR_OK;
    }
};

}  // namespace fj
}  // namespace gtr
