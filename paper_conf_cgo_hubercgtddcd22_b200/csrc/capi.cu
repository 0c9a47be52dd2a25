// capi.cu -- context management, status strings and variant queries of the
// C ABI declared in include/gtr.h.
#include <cstdlib>

#include "gtr_internal.h"
#include "tma.cuh"

using namespace gtr;

extern "C" int gtr_version(void) { return GTR_VERSION; }

extern "C" const char *gtr_strerror(int status) {
    switch (status) {
    case GTR_OK: return "ok";
    case GTR_EINVAL: return "invalid argument or configuration";
    case GTR_ECUDA: return "CUDA runtime error";
    case GTR_ENOMEM: return "workspace or pool too small";
    case GTR_EHEAP: return "device fallback heap exhausted (globalized variables did not fit)";
    case GTR_EDEVICE: return "device-side error flag set";
    case GTR_EUNSUPPORTED: return "configuration not instantiated";
    default: return "unknown status";
    }
}

extern "C" int gtr_ctx_create(int device, void *fallback_pool, uint64_t fallback_pool_bytes, gtr_ctx **out) {
    if (!out) return GTR_EINVAL;
    *out = nullptr;
    int n = 0;
    GTR_CUDA_TRY(cudaGetDeviceCount(&n));
    if (device < 0 || device >= n) return GTR_EINVAL;
    GTR_CUDA_TRY(cudaSetDevice(device));
    gtr_ctx *c = static_cast<gtr_ctx *>(calloc(1, sizeof(gtr_ctx)));
    if (!c) return GTR_ENOMEM;
    c->device = device;
    if (cudaDeviceGetAttribute(&c->num_sms, cudaDevAttrMultiProcessorCount, device) != cudaSuccess ||
        cudaMalloc(&c->d_err, 256) != cudaSuccess || cudaMalloc(&c->d_stage, 256) != cudaSuccess ||
        cudaMemset(c->d_err, 0, 256) != cudaSuccess) {
        if (c->d_err) cudaFree(c->d_err);
        if (c->d_stage) cudaFree(c->d_stage);
        free(c);
        return GTR_ECUDA;
    }
    c->pool = static_cast<uint64_t *>(fallback_pool);
    c->pool_bytes = fallback_pool ? fallback_pool_bytes : 0;
    c->spin_limit = GTR_DEFAULT_SPIN_LIMIT;
    *out = c;
    return GTR_OK;
}

extern "C" int gtr_ctx_destroy(gtr_ctx *c) {
    if (!c) return GTR_EINVAL;
    cudaFree(c->d_err);
    cudaFree(c->d_stage);
    free(c);
    return GTR_OK;
}

extern "C" int gtr_ctx_check(gtr_ctx *c, void *stream) {
    if (!c) return GTR_EINVAL;
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    uint32_t err = 0;
    GTR_CUDA_TRY(cudaMemcpyAsync(&err, c->d_err, sizeof(err), cudaMemcpyDeviceToHost, s));
    GTR_CUDA_TRY(cudaStreamSynchronize(s));
    GTR_CUDA_TRY(cudaGetLastError());
    if (err == 0) return GTR_OK;
    GTR_CUDA_TRY(cudaMemsetAsync(c->d_err, 0, sizeof(err), s));
    GTR_CUDA_TRY(cudaStreamSynchronize(s));
    if (err & ERR_HEAP) return GTR_EHEAP;
    return GTR_EDEVICE;     // ERR_HANG (watchdog), ERR_LIFO, ERR_DUP_ENERGY, ERR_BUILD
}

extern "C" int gtr_ctx_set_spin_limit(gtr_ctx *c, uint64_t polls) {
    if (!c) return GTR_EINVAL;
    c->spin_limit = polls ? polls : GTR_DEFAULT_SPIN_LIMIT;
    return GTR_OK;
}

// Watchdog self-test: a kernel whose waits never complete (kind 0: a team's
// software barrier expecting one more arrival than the team has; kind 1: an
// mbarrier phase no one completes).  With the watchdog each wait gives up
// after the context's spin limit, sets ERR_HANG and the kernel exits.
namespace gtr {
__global__ void k_watchdog_selftest(int32_t kind, RtParams rp) {
    using K = Cfg<SPMD, PL_STACK, false, 64>;
    team_init<K>(rp);
    if (kind == 0) {
        soft_barrier(K::NT + 1);                  // one arrival short: never completes
    } else {
        __shared__ uint64_t bar;
        if (threadIdx.x == 0) tma::mbar_init(&bar);
        __syncthreads();
        tma::mbar_wait(&bar, 0, rp.spin_limit, rp.err, ERR_HANG);   // phase 0 never completes
    }
}
}  // namespace gtr

extern "C" int gtr_watchdog_selftest(gtr_ctx *c, int32_t kind, void *stream) {
    if (!c || kind < 0 || kind > 1) return GTR_EINVAL;
    using K = gtr::Cfg<gtr::SPMD, gtr::PL_STACK, false, 64>;
    gtr::Launch L;
    gtr_launch_cfg cfg = {2, 64, gtr::SPMD, gtr::PL_STACK, 0, 0, 0};
    int st = gtr::resolve<K>(c, &cfg, reinterpret_cast<const void *>(&gtr::k_watchdog_selftest), 0, &L);
    if (st) return st;
    gtr::k_watchdog_selftest<<<L.teams, L.block, L.dyn_smem, static_cast<cudaStream_t>(stream)>>>(kind, L.rp);
    GTR_CUDA_TRY(cudaGetLastError());
    return GTR_OK;
}

extern "C" int gtr_ctx_fallback_high_water(gtr_ctx *c, uint64_t *bytes_out, int32_t reset, void *stream) {
    if (!c || !bytes_out) return GTR_EINVAL;
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    unsigned long long *d = reinterpret_cast<unsigned long long *>(reinterpret_cast<char *>(c->d_err) + 8);
    unsigned long long v = 0;
    GTR_CUDA_TRY(cudaMemcpyAsync(&v, d, sizeof(v), cudaMemcpyDeviceToHost, s));
    if (reset) GTR_CUDA_TRY(cudaMemsetAsync(d, 0, sizeof(v), s));
    GTR_CUDA_TRY(cudaStreamSynchronize(s));
    *bytes_out = v;
    return GTR_OK;
}

// family query hooks (each family's TU)
int gtr_internal_query_xs(gtr_ctx *, const gtr_launch_cfg *, gtr_variant_info *);
int gtr_internal_query_su3(gtr_ctx *, const gtr_launch_cfg *, gtr_variant_info *);
int gtr_internal_query_rs(gtr_ctx *, const gtr_launch_cfg *, gtr_variant_info *);
int gtr_internal_query_fj(gtr_ctx *, const gtr_launch_cfg *, gtr_variant_info *, int floor);
int gtr_internal_query_sem(gtr_ctx *, const gtr_launch_cfg *, gtr_variant_info *);

extern "C" int gtr_query_variant(int kernel, const gtr_launch_cfg *cfg, gtr_variant_info *out) {
    if (!cfg || !out) return GTR_EINVAL;
    gtr_ctx tmp = {};
    int dev = 0;
    GTR_CUDA_TRY(cudaGetDevice(&dev));
    tmp.device = dev;
    GTR_CUDA_TRY(cudaDeviceGetAttribute(&tmp.num_sms, cudaDevAttrMultiProcessorCount, dev));
    switch (kernel) {
    case GTR_K_XS: return gtr_internal_query_xs(&tmp, cfg, out);
    case GTR_K_SU3: return gtr_internal_query_su3(&tmp, cfg, out);
    case GTR_K_RS: return gtr_internal_query_rs(&tmp, cfg, out);
    case GTR_K_FORKJOIN: return gtr_internal_query_fj(&tmp, cfg, out, 0);
    case GTR_K_BARRIER_FLOOR: return gtr_internal_query_fj(&tmp, cfg, out, 1);
    case GTR_K_SEMANTICS: return gtr_internal_query_sem(&tmp, cfg, out);
    default: return GTR_EINVAL;
    }
}

extern "C" int gtr_l2_persist(gtr_ctx *c, const void *base, uint64_t bytes, uint64_t persist_bytes, float hit_ratio,
                              void *stream) {
    if (!c || hit_ratio < 0.f || hit_ratio > 1.f || (bytes && !base)) return GTR_EINVAL;
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    cudaStreamAttrValue v = {};
    if (bytes) {
        int max_persist = 0, max_window = 0;
        GTR_CUDA_TRY(cudaDeviceGetAttribute(&max_persist, cudaDevAttrMaxPersistingL2CacheSize, c->device));
        GTR_CUDA_TRY(cudaDeviceGetAttribute(&max_window, cudaDevAttrMaxAccessPolicyWindowSize, c->device));
        uint64_t lim = persist_bytes < (uint64_t)max_persist ? persist_bytes : (uint64_t)max_persist;
        GTR_CUDA_TRY(cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, lim));
        v.accessPolicyWindow.base_ptr = const_cast<void *>(base);
        v.accessPolicyWindow.num_bytes = bytes < (uint64_t)max_window ? bytes : (uint64_t)max_window;
        v.accessPolicyWindow.hitRatio = hit_ratio;
        v.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
        v.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
    } else {
        v.accessPolicyWindow.num_bytes = 0;
        GTR_CUDA_TRY(cudaCtxResetPersistingL2Cache());
    }
    GTR_CUDA_TRY(cudaStreamSetAttribute(s, cudaStreamAttributeAccessPolicyWindow, &v));
    return GTR_OK;
}
