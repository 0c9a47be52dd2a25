// gtr_internal.h -- host-side helpers shared by the kernel translation units
// (context, launch-configuration resolution, variant dispatch).
#pragma once
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

#include "../../include/gtr.h"
#include "gtr_rt.cuh"

struct gtr_ctx {
    int device;
    int num_sms;
    uint64_t *pool;
    uint64_t pool_bytes;
    uint32_t *d_err;       // device error word (+8: fallback high-water mark, u64)
    void *d_stage;         // 256 B staging buffer (e2e request / results)
    uint64_t spin_limit;   // watchdog polls per spin-wait (gtr_ctx_set_spin_limit)
};
#define GTR_DEFAULT_SPIN_LIMIT (1ull << 26)

namespace gtr {

#define GTR_CUDA_TRY(x)                                                                    \
    do {                                                                                   \
        cudaError_t e_ = (x);                                                              \
        if (e_ != cudaSuccess) {                                                           \
            if (getenv("GTR_DEBUG")) fprintf(stderr, "gtr: %s:%d %s\n", __FILE__, __LINE__, \
                                             cudaGetErrorString(e_));                      \
            return GTR_ECUDA;                                                              \
        }                                                                                  \
    } while (0)

// Resolved launch geometry for one variant.
struct Launch {
    int block;          // hardware threads per CTA
    int teams;          // grid size
    uint32_t dyn_smem;  // dynamic shared memory bytes
    RtParams rp;
};

inline uint32_t odd_words(uint32_t bytes) {
    uint32_t w = (bytes + 7u) / 8u;
    return (w % 2u == 1u) ? w : w + 1u;
}

// Compute geometry + runtime params for variant K of kernel `fn`.
template <class K>
int resolve(gtr_ctx *ctx, const gtr_launch_cfg *cfg, const void *fn, uint32_t default_stack_bytes,
            Launch *L, bool stack_always = false, uint32_t extra_dyn_bytes = 0) {
    L->block = K::BLOCK;
    uint32_t stack_words = 0, stride = 0;
    if (K::PL == PL_RUNTIME || K::PL == PL_COALESCED || (stack_always && K::PL != PL_GLOBAL)) {
        uint32_t bytes = cfg->smem_stack_bytes ? cfg->smem_stack_bytes : default_stack_bytes;
        stack_words = (bytes + 7u) / 8u;
        if (stack_words > 4095u) return GTR_EINVAL;
        stride = odd_words(bytes);
    }
    L->dyn_smem = tstate_bytes<K>() + (uint32_t)K::BLOCK * stride * 8u;
    if (extra_dyn_bytes) L->dyn_smem = ((L->dyn_smem + 15u) & ~15u) + extra_dyn_bytes;
    // static + dynamic above 48 KB needs the opt-in; set it for every launch
    // with dynamic shared memory (cheap host call)
    if (L->dyn_smem > 0) {
        if (cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)L->dyn_smem) !=
            cudaSuccess)
            return GTR_EINVAL;
    }
    int per_sm = 0;
    GTR_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, K::BLOCK, L->dyn_smem));
    if (per_sm < 1) return GTR_EINVAL;
    L->teams = cfg->num_teams > 0 ? cfg->num_teams : per_sm * ctx->num_sms;
    L->rp.err = ctx->d_err;
    L->rp.hwm = reinterpret_cast<unsigned long long *>(reinterpret_cast<char *>(ctx->d_err) + 8);
    L->rp.pool = ctx->pool;
    uint64_t hw = (uint64_t)L->teams * (uint64_t)K::BLOCK;
    L->rp.pool_wpt = ctx->pool ? (ctx->pool_bytes / 8u) / hw : 0;
    L->rp.sm_stack_words = stack_words;
    L->rp.sm_stride_words = stride;
    L->rp.spin_limit = ctx->spin_limit ? ctx->spin_limit : GTR_DEFAULT_SPIN_LIMIT;
    return GTR_OK;
}

// `teams distribute` chunk for n iterations: the kernel's chunk, or -- when
// that leaves teams idle (n < chunk * teams) -- ceil(n / teams) rounded up to
// a warp multiple, so the league is busy (results do not depend on it).
inline uint32_t fit_chunk(uint64_t n, uint32_t chunk, int teams) {
    if (teams < 1 || n >= (uint64_t)chunk * (uint64_t)teams) return chunk;
    uint64_t c = (n + (uint64_t)teams - 1) / (uint64_t)teams;
    c = (c + 31u) & ~(uint64_t)31u;
    if (c < 32u) c = 32u;
    return c < chunk ? (uint32_t)c : chunk;
}

// Balanced `teams distribute` chunk: the fewest rounds the kernel's chunk
// allows (ceil(n / (chunk * teams))), each as full as possible -- the last
// round of equal chunks otherwise leaves most teams idle (10M RS lookups in
// chunks of 4096 over 592 teams: 4.1 rounds run as 5).
inline uint32_t balanced_chunk(uint64_t n, uint32_t chunk, int teams) {
    if (teams < 1 || n == 0) return chunk;
    const uint64_t per_round = (uint64_t)chunk * (uint64_t)teams;
    const uint64_t rounds = (n + per_round - 1) / per_round;
    uint64_t c = (n + rounds * (uint64_t)teams - 1) / (rounds * (uint64_t)teams);
    c = (c + 31u) & ~(uint64_t)31u;
    if (c < 32u) c = 32u;
    return c < chunk ? (uint32_t)c : chunk;
}

template <class K> int fill_info(const void *fn, const Launch &L, int per_sm, gtr_variant_info *out) {
    cudaFuncAttributes a;
    GTR_CUDA_TRY(cudaFuncGetAttributes(&a, fn));
    out->regs = a.numRegs;
    out->static_smem = (int32_t)a.sharedSizeBytes;
    out->dyn_smem = (int32_t)L.dyn_smem;
    out->local_bytes = (int32_t)a.localSizeBytes;
    out->block_threads = L.block;
    out->teams_per_sm = per_sm;
    out->num_teams = L.teams;
    return GTR_OK;
}

// Variant dispatch: Op<K>::run(args...) for the runtime (mode, placement,
// fold, thread_limit) triple; NATIVE handled by the caller.
template <int NT, int FLAGS, template <class> class Op, class... A>
int dispatch_mpf(int mode, int pl, int fold, A &&...a) {
#define GTR_CASE(M, P)                                                                     \
    if (mode == M && pl == P) {                                                            \
        if (fold) return Op<Cfg<M, P, true, NT, FLAGS>>::run(a...);                        \
        return Op<Cfg<M, P, false, NT, FLAGS>>::run(a...);                                 \
    }
#define GTR_CASES(M)                                                                       \
    GTR_CASE(M, PL_RUNTIME) GTR_CASE(M, PL_GLOBAL) GTR_CASE(M, PL_SHARED_STATIC) GTR_CASE(M, PL_STACK) \
    GTR_CASE(M, PL_COALESCED)
    GTR_CASES(GENERIC)
    GTR_CASES(GENERIC_CASCADE)
    GTR_CASES(CSM)
    GTR_CASES(SPMD)
#undef GTR_CASES
#undef GTR_CASE
    return GTR_EUNSUPPORTED;
}

// SPMD-only dispatch (flags that only change SPMD-ized code).
template <int NT, int FLAGS, template <class> class Op, class... A>
int dispatch_spmd(int pl, int fold, A &&...a) {
#define GTR_CASE(P)                                                                        \
    if (pl == P) {                                                                         \
        if (fold) return Op<Cfg<SPMD, P, true, NT, FLAGS>>::run(a...);                     \
        return Op<Cfg<SPMD, P, false, NT, FLAGS>>::run(a...);                              \
    }
    GTR_CASE(PL_RUNTIME) GTR_CASE(PL_GLOBAL) GTR_CASE(PL_SHARED_STATIC) GTR_CASE(PL_STACK) GTR_CASE(PL_COALESCED)
#undef GTR_CASE
    return GTR_EUNSUPPORTED;
}

inline bool valid_cfg(const gtr_launch_cfg *c) {
    if (!c) return false;
    if (c->mode < 0 || c->mode > 4) return false;
    if (c->placement < 0 || c->placement > 4) return false;
    if (c->thread_limit <= 0 || c->thread_limit % 32 != 0) return false;
    if (c->num_teams < 0) return false;
    return true;
}

}  // namespace gtr
