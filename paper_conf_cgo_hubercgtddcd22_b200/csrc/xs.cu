// xs.cu -- XS entry points: variant dispatch, the NATIVE (CUDA watermark)
// kernel, the unionized-grid builders and the extern "C" API (include/gtr.h).
// The runtime-mode variants live in separate modules (xs_variant.cu compiled
// once per variant): a GENERIC kernel's indirect
// call may reach every address-taken region of its module, so sharing a
// module across variants would inflate each one's registers and shared
// memory (the spurious call edges of P:593-597, fn. 4).
#include "xs_impl.cuh"

namespace gtr {
namespace xs {

// ---------------------------------------------------------------- native form
template <int NT> __global__ void __launch_bounds__(NT) kernel_native(Params P) {
    using KN = Cfg<NATIVE, PL_STACK, true, NT>;
    __shared__ uint32_t tally[17];
    if (threadIdx.x < 17) tally[threadIdx.x] = 0;
    if (P.req) { P.first = P.req->first; P.n = P.req->n; P.seed = P.req->seed; }
    __syncthreads();
    const uint64_t stride = (uint64_t)gridDim.x * NT;
    if (P.s_rec) {                                    // sorted mode: thread per sorted position
        for (uint64_t q = (uint64_t)blockIdx.x * NT + threadIdx.x; q < P.n; q += stride)
            lookup_sorted<KN>(P, q, tally);
    } else if (P.history) {                           // history mode: thread per particle
        const uint64_t np = (P.n + kHistoryLookups - 1) / kHistoryLookups;
        for (uint64_t p = (uint64_t)blockIdx.x * NT + threadIdx.x; p < np; p += stride)
            for (uint64_t k = p * kHistoryLookups; k < P.n && k < (p + 1) * kHistoryLookups; k++)
                lookup<KN>(P, P.first + k, tally);
    } else {
        for (uint64_t k = (uint64_t)blockIdx.x * NT + threadIdx.x; k < P.n; k += stride)
            lookup<KN>(P, P.first + k, tally);
    }
    __syncthreads();
    flush_out(P, tally, threadIdx.x, NT);
}

// ---------------------------------------------------------------- builders
// energies e[n][k] = grid[n][k][0]
__global__ void k_extract_energies(const double *__restrict__ grid, int64_t total, double *__restrict__ e) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < total;
         i += (int64_t)gridDim.x * blockDim.x)
        e[i] = __ldg(grid + i * 6);
}
// number of entries of sorted a[0..n) that are < x (strict) or <= x
__device__ __forceinline__ int64_t count_below(const double *__restrict__ a, int64_t n, double x, bool inclusive) {
    int64_t lo = 0, hi = n;   // answer in [lo, hi]
    while (lo < hi) {
        int64_t mid = (lo + hi) >> 1;
        double v = __ldg(a + mid);
        if (inclusive ? (v <= x) : (v < x)) lo = mid + 1;
        else hi = mid;
    }
    return lo;
}
// position of energy (n,k) in the union: the number of energies before it in
// (energy, nuclide, gridpoint) order -- smaller energies, equal energies of
// lower nuclides, and equal energies earlier in its own (sorted) nuclide, of
// which there are k - #{smaller}: so its own nuclide contributes exactly k.
// Distinct ranks even with duplicate energies (equal values in any order
// make the same ascending egrid).
__global__ void k_union_scatter(const double *__restrict__ e, int64_t n_iso, int64_t n_gp,
                                double *__restrict__ egrid) {
    const int64_t total = n_iso * n_gp;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < total;
         i += (int64_t)gridDim.x * blockDim.x) {
        const double x = e[i];
        const int64_t n = i / n_gp, k = i - n * n_gp;
        int64_t rank = k;
        for (int64_t m = 0; m < n_iso; m++)
            if (m != n) rank += count_below(e + m * n_gp, n_gp, x, m < n);
        egrid[rank] = x;
    }
}
__global__ void k_fill_nan(double *p, int64_t n) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        p[i] = __longlong_as_double(0x7FF8000000000000LL);
}
// ascending (also catches unwritten NaN slots: unsorted nuclides or NaN input)
__global__ void k_check_increasing(const double *__restrict__ eg, int64_t n, uint32_t *err) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
         i += (int64_t)gridDim.x * blockDim.x) {
        const double a = eg[i];
        bool ok = (a == a);
        if (i + 1 < n) ok = ok && (eg[i + 1] >= a);
        if (!ok) atomicOr(err, (uint32_t)ERR_BUILD);
    }
}
// closed form cf(u) = clamp(#{k: e_n[k] <= egrid[u]} - 1, 0, n_gp - 2)
__global__ void k_index_grid(const double *__restrict__ e, int64_t n_iso, int64_t n_gp,
                             const double *__restrict__ egrid, int64_t n_union, int32_t *__restrict__ idx) {
    const int64_t total = n_union * n_iso;
    for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < total;
         t += (int64_t)gridDim.x * blockDim.x) {
        const int64_t u = t / n_iso, n = t - u * n_iso;
        int64_t c = count_below(e + n * n_gp, n_gp, __ldg(egrid + u), true) - 1;
        c = c < 0 ? 0 : (c > n_gp - 2 ? n_gp - 2 : c);
        idx[t] = (int32_t)c;
    }
}
// XSBench's sequential rule (idx_low advances by at most one per
// union point, idx(-1) = 0) from the closed form: the step is taken exactly
// when cf(u) > idx(u-1) (e_n[idx+1] <= egrid[u] <=> cf(u) >= idx+1 for
// idx < n_gp - 2), and idx(u) <= cf(u) throughout, so
// idx(u) = min(idx(u-1) + 1, cf(u)) = u + min(1, min_{v<=u} (cf(v) - v)):
// a prefix minimum down each column.  Without duplicate energies cf grows by
// at most one per union point and idx = cf (the pass changes nothing).
// Blocked scan: (1) per block of kIdxRows rows the column minimum of cf - u,
// (2) per column the exclusive prefix minimum over blocks, (3) the rewrite.
constexpr int64_t kIdxRows = 4096;
__global__ void k_index_colmin(const int32_t *__restrict__ idx, int64_t n_union, int64_t n_iso,
                               int32_t *__restrict__ bmin) {
    const int64_t nblk = (n_union + kIdxRows - 1) / kIdxRows;
    for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < nblk * n_iso;
         t += (int64_t)gridDim.x * blockDim.x) {
        const int64_t blk = t / n_iso, n = t - blk * n_iso;
        const int64_t u1 = min(n_union, (blk + 1) * kIdxRows);
        int32_t m = INT32_MAX;
        for (int64_t u = blk * kIdxRows; u < u1; u++) m = min(m, (int32_t)(idx[u * n_iso + n] - u));
        bmin[t] = m;
    }
}
__global__ void k_index_colscan(int32_t *__restrict__ bmin, int64_t nblk, int64_t n_iso) {
    for (int64_t n = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; n < n_iso; n += (int64_t)gridDim.x * blockDim.x) {
        int32_t run = INT32_MAX;                      // exclusive: the minimum over earlier blocks
        for (int64_t b = 0; b < nblk; b++) {
            const int32_t v = bmin[b * n_iso + n];
            bmin[b * n_iso + n] = run;
            run = min(run, v);
        }
    }
}
__global__ void k_index_sequential(int32_t *__restrict__ idx, int64_t n_union, int64_t n_iso,
                                   const int32_t *__restrict__ carry) {
    const int64_t nblk = (n_union + kIdxRows - 1) / kIdxRows;
    for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < nblk * n_iso;
         t += (int64_t)gridDim.x * blockDim.x) {
        const int64_t blk = t / n_iso, n = t - blk * n_iso;
        const int64_t u1 = min(n_union, (blk + 1) * kIdxRows);
        int32_t run = carry[t];
        for (int64_t u = blk * kIdxRows; u < u1; u++) {
            run = min(run, (int32_t)(idx[u * n_iso + n] - u));
            idx[u * n_iso + n] = (int32_t)(u + min(1, run));
        }
    }
}

// Self-test of the branch-free interpolation-factor division (ddiv_fast,
// DESIGN.md R-XS-div): operand pairs from a counter-based hash -- raw 64-bit
// patterns (every exponent, subnormals, Inf, NaN), pairs of unit-interval
// energies as the lookups form them, and near-equal / near-overflow pairs --
// each compared bit for bit with the IEEE division wherever ddiv_fast's
// guard accepts.  counts[0] += mismatches, counts[1] += accepted pairs.
__device__ __forceinline__ uint64_t mix64(uint64_t z) {
    z += 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}
__global__ void k_ddiv_selftest(uint64_t n, uint64_t seed, unsigned long long *counts) {
    unsigned long long bad = 0, acc = 0;
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
        const uint64_t a = mix64(seed ^ (2 * i)), b = mix64(seed ^ (2 * i + 1));
        double x, y;
        switch (i & 3) {
        case 0:                                        // raw bit patterns
            x = __longlong_as_double((long long)a);
            y = __longlong_as_double((long long)b);
            break;
        case 1: {                                      // (hi.e - E) / (hi.e - lo.e), energies in [0, 1)
            const double e0 = (double)(a >> 11) * 0x1p-53, e1 = (double)(b >> 11) * 0x1p-53;
            const double lo = fmin(e0, e1), hi = fmax(e0, e1);
            const double E = lo + (hi - lo) * ((double)(mix64(a ^ b) >> 11) * 0x1p-53);
            x = hi - E;
            y = hi - lo;
            break;
        }
        case 2: {                                      // neighbouring doubles: tiny denominators
            const double e = (double)(a >> 11) * 0x1p-53;
            const double h = __longlong_as_double(__double_as_longlong(e) + (long long)(1 + (b & 7)));
            x = h - (double)((b >> 8) >> 11) * 0x1p-53 * (h - e);
            y = h - e;
            break;
        }
        default: {                                     // random exponents across the whole range
            x = ldexp(1.0 + (double)(a >> 12) * 0x1p-52, (int)(a & 2047) - 1075);
            y = ldexp(1.0 + (double)(b >> 12) * 0x1p-52, (int)(b & 2047) - 1075);
            if (b & 0x800) y = -y;
        }
        }
        bool ok;
        const double q = xs::ddiv_fast(x, y, ok);
        if (ok) {
            acc++;
            const double r = x / y;
            const bool same = (__double_as_longlong(q) == __double_as_longlong(r)) || (q != q && r != r);
            if (!same) bad++;
        }
    }
    if (bad) atomicAdd(counts, bad);
    atomicAdd(counts + 1, acc);
}

// Runtime-mode variants: defined (explicitly instantiated) in xs_variant.cu.
template <class K> int run_variant(LaunchArgs &a);
template <class K> struct VariantOp {
    static int run(LaunchArgs &a) { return run_variant<K>(a); }
};

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
    const uint32_t smem = (uint32_t)(sizeof(ChunkBuf<KN>) > sizeof(CoBuf<KN>) ? sizeof(ChunkBuf<KN>) : sizeof(CoBuf<KN>));
    GTR_CUDA_TRY(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    int per_sm = 0;
    GTR_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, NT, smem));
    if (per_sm < 1) return GTR_EINVAL;
    Launch L;
    L.block = NT;
    L.dyn_smem = smem;
    L.teams = a.cfg->num_teams > 0 ? a.cfg->num_teams : per_sm * a.ctx->num_sms;
    if (a.info) return fill_info<KN>(fn, L, per_sm, a.info);
    if (a.P.req || a.P.history) return GTR_EUNSUPPORTED;
    a.P.chunk = fit_chunk(a.P.n, kBucketLookupsPerThread * NT, L.teams);
    kernel_native_bucketed<KN><<<L.teams, NT, smem, a.stream>>>(a.P);
    GTR_CUDA_TRY(cudaGetLastError());
    return GTR_OK;
}

inline int launch(LaunchArgs &a) {
    const gtr_launch_cfg *c = a.cfg;
    if (!valid_cfg(c)) return GTR_EINVAL;
    a.P.plain = (c->flags & GTR_F_PLAIN) ? 1 : 0;
    a.P.history = (c->flags & GTR_F_HISTORY) ? 1 : 0;
    if (c->mode == NATIVE && (c->flags & GTR_F_NATIVE_BUCKETED)) {
        if (a.P.plain) return GTR_EINVAL;
        if (c->thread_limit == 128) return run_native_bucketed<128>(a);
        if (c->thread_limit == 256) return run_native_bucketed<256>(a);
        return GTR_EUNSUPPORTED;
    }
    if (c->mode == NATIVE) {
        if (c->thread_limit == 128) return run_native<128>(a);
        if (c->thread_limit == 256) return run_native<256>(a);
        if (c->thread_limit == 512) return run_native<512>(a);
        return GTR_EUNSUPPORTED;
    }
    if (c->thread_limit == 128) return dispatch_mpf<128, 0, VariantOp>(c->mode, c->placement, c->fold, a);
    if (c->thread_limit == 256) return dispatch_mpf<256, 0, VariantOp>(c->mode, c->placement, c->fold, a);
    return GTR_EUNSUPPORTED;
}

}  // namespace xs
}  // namespace gtr

using namespace gtr;

int gtr_internal_query_xs(gtr_ctx *ctx, const gtr_launch_cfg *cfg, gtr_variant_info *info) {
    gtr_xs_tables t = {};
    xs::LaunchArgs a{ctx, cfg, xs::make_params(&t, 0, 0, 0, nullptr, nullptr, nullptr), nullptr, info};
    return xs::launch(a);
}

extern "C" int gtr_ddiv_selftest(gtr_ctx *ctx, uint64_t n, uint64_t seed, uint64_t *d_counts, void *stream) {
    if (!ctx || !d_counts) return GTR_EINVAL;
    if (n == 0) return GTR_OK;
    xs::k_ddiv_selftest<<<ctx->num_sms * 8, 256, 0, static_cast<cudaStream_t>(stream)>>>(
        n, seed, reinterpret_cast<unsigned long long *>(d_counts));
    GTR_CUDA_TRY(cudaGetLastError());
    return GTR_OK;
}

extern "C" uint64_t gtr_xs_build_workspace_bytes(int64_t n_iso, int64_t n_gp) {
    // energies (8 B each) + the index builder's per-block column minima
    const uint64_t total = (uint64_t)n_iso * (uint64_t)n_gp;
    const uint64_t nblk = (total + (uint64_t)xs::kIdxRows - 1) / (uint64_t)xs::kIdxRows;
    return total * 8u + nblk * (uint64_t)n_iso * 4u;
}

static int grid_blocks(gtr_ctx *ctx, int64_t work, int threads) {
    int64_t b = (work + threads - 1) / threads;
    int64_t cap = (int64_t)ctx->num_sms * 16;
    return (int)(b < 1 ? 1 : (b > cap ? cap : b));
}

extern "C" int gtr_xs_build_egrid(gtr_ctx *ctx, const double *d_grid, int64_t n_iso, int64_t n_gp,
                                  double *d_egrid_out, void *d_workspace, void *stream) {
    if (!ctx || !d_grid || !d_egrid_out || !d_workspace || n_iso < 1 || n_gp < 2) return GTR_EINVAL;
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    const int64_t total = n_iso * n_gp;
    double *e = static_cast<double *>(d_workspace);
    xs::k_extract_energies<<<grid_blocks(ctx, total, 256), 256, 0, s>>>(d_grid, total, e);
    xs::k_fill_nan<<<grid_blocks(ctx, total, 256), 256, 0, s>>>(d_egrid_out, total);
    xs::k_union_scatter<<<grid_blocks(ctx, total, 128), 128, 0, s>>>(e, n_iso, n_gp, d_egrid_out);
    xs::k_check_increasing<<<grid_blocks(ctx, total, 256), 256, 0, s>>>(d_egrid_out, total, ctx->d_err);
    GTR_CUDA_TRY(cudaGetLastError());
    return GTR_OK;
}

extern "C" int gtr_xs_build_index_grid(gtr_ctx *ctx, const double *d_grid, int64_t n_iso, int64_t n_gp,
                                       const double *d_egrid, int32_t *d_index_out, void *d_workspace,
                                       void *stream) {
    if (!ctx || !d_grid || !d_egrid || !d_index_out || !d_workspace || n_iso < 1 || n_gp < 2)
        return GTR_EINVAL;
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    const int64_t total = n_iso * n_gp;
    double *e = static_cast<double *>(d_workspace);
    xs::k_extract_energies<<<grid_blocks(ctx, total, 256), 256, 0, s>>>(d_grid, total, e);
    xs::k_index_grid<<<grid_blocks(ctx, total * n_iso, 256), 256, 0, s>>>(e, n_iso, n_gp, d_egrid, total,
                                                                          d_index_out);
    // the sequential rule (differs from the closed form only where energies
    // repeat); block minima live in the workspace after the energies
    const int64_t nblk = (total + xs::kIdxRows - 1) / xs::kIdxRows;
    int32_t *bmin = reinterpret_cast<int32_t *>(e + total);
    xs::k_index_colmin<<<grid_blocks(ctx, nblk * n_iso, 256), 256, 0, s>>>(d_index_out, total, n_iso, bmin);
    xs::k_index_colscan<<<grid_blocks(ctx, n_iso, 128), 128, 0, s>>>(bmin, nblk, n_iso);
    xs::k_index_sequential<<<grid_blocks(ctx, nblk * n_iso, 256), 256, 0, s>>>(d_index_out, total, n_iso, bmin);
    GTR_CUDA_TRY(cudaGetLastError());
    return GTR_OK;
}

namespace gtr {
namespace xs {
// hash[b][n] = clamp(#{k: e_n[k] <= b * (1/bins)} - 1, 0, n_gp - 2)
__global__ void k_hash_grid(const double *__restrict__ e, int64_t n_iso, int64_t n_gp, int32_t bins,
                            int32_t *__restrict__ out) {
    const int64_t total = (int64_t)bins * n_iso;
    const double du = 1.0 / bins;
    for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < total;
         t += (int64_t)gridDim.x * blockDim.x) {
        const int64_t b = t / n_iso, n = t - b * n_iso;
        int64_t c = count_below(e + n * n_gp, n_gp, (double)b * du, true) - 1;
        c = c < 0 ? 0 : (c > n_gp - 2 ? n_gp - 2 : c);
        out[t] = (int32_t)c;
    }
}
}  // namespace xs
}  // namespace gtr

extern "C" int gtr_xs_build_energies(gtr_ctx *ctx, const double *d_grid, int64_t n_iso, int64_t n_gp,
                                     double *d_energies_out, void *stream) {
    if (!ctx || !d_grid || !d_energies_out || n_iso < 1 || n_gp < 2) return GTR_EINVAL;
    const int64_t total = n_iso * n_gp;
    xs::k_extract_energies<<<grid_blocks(ctx, total, 256), 256, 0, static_cast<cudaStream_t>(stream)>>>(
        d_grid, total, d_energies_out);
    GTR_CUDA_TRY(cudaGetLastError());
    return GTR_OK;
}

extern "C" int gtr_xs_build_hash_grid(gtr_ctx *ctx, const double *d_energies, int64_t n_iso, int64_t n_gp,
                                      int32_t hash_bins, int32_t *d_hash_out, void *stream) {
    if (!ctx || !d_energies || !d_hash_out || n_iso < 1 || n_gp < 2 || hash_bins < 1) return GTR_EINVAL;
    xs::k_hash_grid<<<grid_blocks(ctx, (int64_t)hash_bins * n_iso, 256), 256, 0, static_cast<cudaStream_t>(stream)>>>(
        d_energies, n_iso, n_gp, hash_bins, d_hash_out);
    GTR_CUDA_TRY(cudaGetLastError());
    return GTR_OK;
}

namespace gtr {
namespace xs {
// B[b] = #{m : egrid[m] < b / 2^L}, b in [0, 2^L] (b / 2^L exact in fp64)
__global__ void k_union_bins(const double *__restrict__ egrid, int64_t n, int32_t log2b, uint32_t *__restrict__ out) {
    const int64_t nb = (1ll << log2b) + 1;
    for (int64_t b = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; b < nb; b += (int64_t)gridDim.x * blockDim.x)
        out[b] = (uint32_t)count_below(egrid, n, (double)b / (double)(1ll << log2b), false);
}
}  // namespace xs
}  // namespace gtr

extern "C" int gtr_xs_build_union_bins(gtr_ctx *ctx, const double *d_egrid, int64_t n_union, int32_t log2_bins,
                                       uint32_t *d_bins_out, void *stream) {
    if (!ctx || !d_egrid || !d_bins_out || n_union < 2 || n_union >= ((int64_t)1 << 32) || log2_bins < 0 ||
        log2_bins > 26)
        return GTR_EINVAL;
    const int64_t nb = ((int64_t)1 << log2_bins) + 1;
    xs::k_union_bins<<<grid_blocks(ctx, nb, 256), 256, 0, static_cast<cudaStream_t>(stream)>>>(
        d_egrid, n_union, log2_bins, d_bins_out);
    GTR_CUDA_TRY(cudaGetLastError());
    return GTR_OK;
}

static bool tables_ok(const gtr_xs_tables *t) {
    if (!(t && t->grid && t->num_nucs && t->mats && t->concs && t->n_iso > 0 && t->n_gp >= 2 &&
          t->max_num_nucs > 0 && t->n_iso * t->n_gp < ((int64_t)1 << 28)))   // u packs in 28 bits
        return false;
    if (t->union_bins && (t->union_bins_log2 < 0 || t->union_bins_log2 > 26)) return false;
    switch (t->grid_type) {
    case GTR_XS_UNIONIZED: return t->egrid && t->index_grid && t->n_union >= 2;
    case GTR_XS_NUCLIDE: return t->energies != nullptr;
    case GTR_XS_HASH: return t->energies && t->hash_index && t->hash_bins >= 1 && t->hash_bins < (1 << 28);
    default: return false;
    }
}

extern "C" int gtr_xs_lookup(gtr_ctx *ctx, const gtr_launch_cfg *cfg, const gtr_xs_tables *tables,
                             uint64_t first, uint64_t n, uint64_t seed, uint64_t *d_out,
                             const gtr_xs_verify *verify, void *stream) {
    if (!ctx || !cfg || !tables_ok(tables) || !d_out) return GTR_EINVAL;
    if (n == 0) return GTR_OK;
    xs::LaunchArgs a{ctx, cfg, xs::make_params(tables, first, n, seed, d_out, verify, nullptr),
                     static_cast<cudaStream_t>(stream), nullptr};
    return xs::launch(a);
}

extern "C" int gtr_xs_lookup_host(gtr_ctx *ctx, const gtr_launch_cfg *cfg, const gtr_xs_tables *tables,
                                  const gtr_xs_request *h_req, uint64_t *h_out, void *stream) {
    if (!ctx || !cfg || !tables_ok(tables) || !h_req || !h_out) return GTR_EINVAL;
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    gtr_xs_request *d_req = static_cast<gtr_xs_request *>(ctx->d_stage);
    uint64_t *d_out = reinterpret_cast<uint64_t *>(static_cast<char *>(ctx->d_stage) + 64);
    GTR_CUDA_TRY(cudaMemcpyAsync(d_req, h_req, sizeof(gtr_xs_request), cudaMemcpyHostToDevice, s));
    GTR_CUDA_TRY(cudaMemsetAsync(d_out, 0, 18 * sizeof(uint64_t), s));
    // the kernel reads (first, n, seed) from d_req; n bounds the launch only
    xs::LaunchArgs a{ctx, cfg, xs::make_params(tables, h_req->first, h_req->n, h_req->seed, d_out, nullptr, d_req),
                     s, nullptr};
    int st = xs::launch(a);
    if (st) return st;
    GTR_CUDA_TRY(cudaMemcpyAsync(h_out, d_out, 18 * sizeof(uint64_t), cudaMemcpyDeviceToHost, s));
    GTR_CUDA_TRY(cudaStreamSynchronize(s));
    return GTR_OK;
}

// ---------------------------------------------------------------- sorted mode
// XSBench's sorted event-based variant: sample every lookup,
// sort the lookups by (material, unionized-grid index), then run them in
// that order -- neighbouring threads share a material (equal-length nuclide
// loops) and nearly equal energies (the same gridpoints, adjacent index-grid
// rows), which the warp-coherent nuclide loops (CoherentRegion) exploit.
// Results are identical: each lookup's arithmetic is its own, the tallies
// are sums.  The sort: counting sort by (material, u bucket) with 2^17
// buckets per material (fuel: ~18 lookups, ~30 union points per bucket), so
// a warp's 32 lookups span ~2-3 buckets.  GTR_XS_SORT_RANK=1 additionally
// orders each bucket by (u, lookup) with a rank count (a deterministic order;
// measured: the lookups gain 2%, the rank pass costs 6% of the step).  Workspace (caller-owned,
// gtr_xs_sorted_workspace_bytes), 16-byte aligned:
//   rec0[n] SortRec | rec1[n] SortRec | key[n] u32 | hist[12*NB] u32 | totals u32
// rec0 holds the samples in lookup order, then the final (ranked) order.
namespace gtr {
namespace xs {
#ifndef GTR_XS_SORT_RANK
#define GTR_XS_SORT_RANK 0
#endif
#ifndef GTR_XS_SORT_LOG2
#define GTR_XS_SORT_LOG2 17
#endif
// u buckets per material: 2^lg with lg = ceil(log2(n / 128)) clamped to
// [8, GTR_XS_SORT_LOG2] -- ~128 lookups per bucket row of 12 materials, so a
// small request does not pay for a 1.57M-bin histogram (17M lookups: 2^17)
inline uint32_t sort_log2(uint64_t n) {
    uint32_t lg = 8;
    while (lg < GTR_XS_SORT_LOG2 && (128ull << lg) < n) lg++;
    return lg;
}
inline uint64_t sort_bins(uint64_t n) { return 12ull << sort_log2(n); }   // a multiple of 1024 (lg >= 8)
constexpr uint32_t kRankMax = 256;                    // larger buckets keep the scatter's order

__device__ __forceinline__ uint32_t sort_key(uint32_t mat, uint32_t u, int64_t n_union, uint32_t lg) {
    const uint32_t nb = 1u << lg;
    uint32_t b = (uint32_t)(((uint64_t)u << lg) / (uint64_t)n_union);
    b = b < nb ? b : nb - 1;
    return mat * nb + b;
}
__device__ __forceinline__ void store_rec(SortRec *d, const SortRec &r) {
    *reinterpret_cast<uint4 *>(d) =
        make_uint4(r.k, r.mu, (uint32_t)__double2loint(r.E), (uint32_t)__double2hiint(r.E));
}
// grid-stride over the lookups; a thread's next lookup is `stride` further,
// so its state advances by the precomputed map of 2*stride steps (exact)
__global__ void k_sort_sample(Params P, SortRec *__restrict__ rec, uint32_t *__restrict__ key,
                              uint32_t *__restrict__ hist, uint64_t A2s, uint64_t C2s, uint32_t lg) {
    using KN = Cfg<NATIVE, PL_STACK, true, 128>;
    if (P.req) { P.first = P.req->first; P.seed = P.req->seed; }
    const int64_t nu = P.grid_type == 0 ? P.n_union : (P.grid_type == 2 ? P.hash_bins : 1);
    const uint64_t k0 = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    uint64_t st = smp::lcg_jump(P.seed, 2ULL * (P.first + k0));
    for (uint64_t k = k0; k < P.n; k += (uint64_t)gridDim.x * blockDim.x, st = smp::lcg_apply(A2s, C2s, st)) {
        double E;
        int mat;
        int64_t u;
        sample_state<KN>(P, st, E, mat, u);
        // the nuclide grid has no u: bucket by energy (the same monotone role)
        const uint32_t kk = P.grid_type == 1
                                ? sort_key((uint32_t)mat, (uint32_t)(E * (double)(1u << lg)), (int64_t)(1u << lg), lg)
                                : sort_key((uint32_t)mat, (uint32_t)u, nu, lg);
        key[k] = kk;
        SortRec r;
        r.k = (uint32_t)k;
        r.mu = ((uint32_t)mat << 28) | (uint32_t)u;
        r.E = E;
        store_rec(rec + k, r);
        atomicAdd(hist + kk, 1u);
    }
}
// exclusive scan of hist[bins] in place: per 1024-bin block a shared-
// memory scan + the block total, then every block adds the totals before it
__global__ void __launch_bounds__(1024) k_sort_scan_local(uint32_t *hist, uint32_t *totals) {
    __shared__ uint32_t part[1024];
    uint32_t *h = hist + (size_t)blockIdx.x * 1024;
    const uint32_t x = h[threadIdx.x];
    part[threadIdx.x] = x;
    __syncthreads();
    for (uint32_t off = 1; off < 1024; off <<= 1) {       // Hillis-Steele inclusive scan
        const uint32_t v = threadIdx.x >= off ? part[threadIdx.x - off] : 0u;
        __syncthreads();
        part[threadIdx.x] += v;
        __syncthreads();
    }
    h[threadIdx.x] = part[threadIdx.x] - x;
    if (threadIdx.x == 1023) totals[blockIdx.x] = part[1023];
}
__global__ void __launch_bounds__(1024) k_sort_scan_add(uint32_t *hist, const uint32_t *totals) {
    __shared__ uint32_t off;
    if (threadIdx.x < 32) {
        uint32_t s = 0;
        for (uint32_t b = threadIdx.x; b < blockIdx.x; b += 32) s += totals[b];
        for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
        if (threadIdx.x == 0) off = s;
    }
    __syncthreads();
    hist[(size_t)blockIdx.x * 1024 + threadIdx.x] += off;
}
__global__ void k_sort_scatter(uint64_t n, const uint32_t *__restrict__ key, const SortRec *__restrict__ in,
                               uint32_t *__restrict__ cursor, SortRec *__restrict__ out) {
    for (uint64_t k = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; k < n; k += (uint64_t)gridDim.x * blockDim.x) {
        const uint32_t pos = atomicAdd(cursor + key[k], 1u);
        *reinterpret_cast<uint4 *>(out + pos) = __ldg(reinterpret_cast<const uint4 *>(in + k));
    }
}
// order each bucket by (u, lookup): after the scatter cursor[b] is the end of
// bucket b (= the start of b+1); position p moves to start + its rank
__global__ void k_sort_rank(uint64_t n, const uint32_t *__restrict__ key, const uint32_t *__restrict__ end,
                            const SortRec *__restrict__ in, SortRec *__restrict__ out) {
    for (uint64_t p = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; p < n; p += (uint64_t)gridDim.x * blockDim.x) {
        const uint4 v = __ldg(reinterpret_cast<const uint4 *>(in + p));
        const uint32_t k = v.x, u = v.y & 0x0FFFFFFFu;
        const uint32_t b = key[k];
        const uint32_t s = b ? __ldg(end + b - 1) : 0u, e = __ldg(end + b);
        uint32_t dest = (uint32_t)p;
        if (e - s <= kRankMax) {
            uint32_t r = 0;
            for (uint32_t q = s; q < e; q++) {
                const uint2 w = __ldg(reinterpret_cast<const uint2 *>(in + q));
                const uint32_t uq = w.y & 0x0FFFFFFFu;
                r += (uq < u || (uq == u && w.x < k)) ? 1u : 0u;
            }
            dest = s + r;
        }
        *reinterpret_cast<uint4 *>(out + dest) = v;
    }
}
}  // namespace xs
}  // namespace gtr

extern "C" uint64_t gtr_xs_sorted_workspace_bytes(uint64_t n) {
    return 36u * n + 4u * (xs::sort_bins(n) + xs::sort_bins(n) / 1024u);
}

// the sampling pass and the sort into the workspace (rec0 = the sorted records)
static int sort_pass(gtr_ctx *ctx, const gtr_launch_cfg *cfg, const xs::Params &P, uint64_t n, void *d_workspace,
                     uint64_t workspace_bytes, cudaStream_t s) {
    if (n > 0xFFFFFFFFull || workspace_bytes < gtr_xs_sorted_workspace_bytes(n) ||
        (reinterpret_cast<uintptr_t>(d_workspace) & 15u) || (uint64_t)P.n_union >= (1ull << 28) ||
        (cfg && (cfg->flags & GTR_F_HISTORY)))
        return GTR_EINVAL;
    if (cfg && !valid_cfg(cfg)) return GTR_EINVAL;
    xs::SortRec *rec0 = static_cast<xs::SortRec *>(d_workspace), *rec1 = rec0 + n;
    uint32_t *key = reinterpret_cast<uint32_t *>(rec1 + n), *hist = key + n;
    const uint32_t lg = xs::sort_log2(n);
    const uint32_t bins = (uint32_t)xs::sort_bins(n), blocks = bins / 1024u;
    GTR_CUDA_TRY(cudaMemsetAsync(hist, 0, 4u * bins, s));
    const int sb = grid_blocks(ctx, (int64_t)n, 256);
    uint64_t A2s, C2s;
    smp::lcg_map(2ULL * (uint64_t)sb * 256u, A2s, C2s);
#if GTR_XS_SORT_RANK
    xs::k_sort_sample<<<sb, 256, 0, s>>>(P, rec0, key, hist, A2s, C2s, lg);
    xs::k_sort_scan_local<<<blocks, 1024, 0, s>>>(hist, hist + bins);
    xs::k_sort_scan_add<<<blocks, 1024, 0, s>>>(hist, hist + bins);
    xs::k_sort_scatter<<<grid_blocks(ctx, (int64_t)n, 256), 256, 0, s>>>(n, key, rec0, hist, rec1);
    xs::k_sort_rank<<<grid_blocks(ctx, (int64_t)n, 256), 256, 0, s>>>(n, key, hist, rec1, rec0);
#else   // bucket order only (no in-bucket ranking): samples in rec1, the scatter into rec0
    xs::k_sort_sample<<<sb, 256, 0, s>>>(P, rec1, key, hist, A2s, C2s, lg);
    xs::k_sort_scan_local<<<blocks, 1024, 0, s>>>(hist, hist + bins);
    xs::k_sort_scan_add<<<blocks, 1024, 0, s>>>(hist, hist + bins);
    xs::k_sort_scatter<<<grid_blocks(ctx, (int64_t)n, 256), 256, 0, s>>>(n, key, rec1, hist, rec0);
#endif
    GTR_CUDA_TRY(cudaGetLastError());
    return GTR_OK;
}
// the lookups in sorted order from a sorted workspace
static int presorted_pass(gtr_ctx *ctx, const gtr_launch_cfg *cfg, xs::Params P, uint64_t n, void *d_workspace,
                          uint64_t workspace_bytes, cudaStream_t s) {
    if (n > 0xFFFFFFFFull || workspace_bytes < gtr_xs_sorted_workspace_bytes(n) ||
        (reinterpret_cast<uintptr_t>(d_workspace) & 15u) || (cfg->flags & GTR_F_HISTORY))
        return GTR_EINVAL;
    P.s_rec = static_cast<const xs::SortRec *>(d_workspace);
    xs::LaunchArgs a{ctx, cfg, P, s, nullptr};
    return xs::launch(a);
}
// the sampling pass, the sort and the lookups in sorted order; P carries the
// outputs (d_out / verify / peer buffers) and, for the host-request form, req
static int sorted_launch(gtr_ctx *ctx, const gtr_launch_cfg *cfg, xs::Params P, uint64_t n, void *d_workspace,
                         uint64_t workspace_bytes, cudaStream_t s) {
    const int st = sort_pass(ctx, cfg, P, n, d_workspace, workspace_bytes, s);
    if (st) return st;
    return presorted_pass(ctx, cfg, P, n, d_workspace, workspace_bytes, s);
}

extern "C" int gtr_xs_sort_lookups(gtr_ctx *ctx, const gtr_xs_tables *tables, uint64_t first, uint64_t n,
                                   uint64_t seed, void *d_workspace, uint64_t workspace_bytes, void *stream) {
    if (!ctx || !tables_ok(tables) || !d_workspace) return GTR_EINVAL;
    if (n == 0) return GTR_OK;
    return sort_pass(ctx, nullptr, xs::make_params(tables, first, n, seed, nullptr, nullptr, nullptr), n,
                     d_workspace, workspace_bytes, static_cast<cudaStream_t>(stream));
}

extern "C" int gtr_xs_lookup_presorted(gtr_ctx *ctx, const gtr_launch_cfg *cfg, const gtr_xs_tables *tables,
                                       uint64_t first, uint64_t n, uint64_t *d_out, const gtr_xs_verify *verify,
                                       const void *d_workspace, uint64_t workspace_bytes, void *stream) {
    if (!ctx || !cfg || !tables_ok(tables) || !d_out || !d_workspace) return GTR_EINVAL;
    if (n == 0) return GTR_OK;
    return presorted_pass(ctx, cfg, xs::make_params(tables, first, n, 0, d_out, verify, nullptr), n,
                          const_cast<void *>(d_workspace), workspace_bytes, static_cast<cudaStream_t>(stream));
}

extern "C" int gtr_xs_lookup_sorted(gtr_ctx *ctx, const gtr_launch_cfg *cfg, const gtr_xs_tables *tables,
                                    uint64_t first, uint64_t n, uint64_t seed, uint64_t *d_out,
                                    const gtr_xs_verify *verify, void *d_workspace, uint64_t workspace_bytes,
                                    void *stream) {
    if (!ctx || !cfg || !tables_ok(tables) || !d_out || !d_workspace) return GTR_EINVAL;
    if (n == 0) return GTR_OK;
    return sorted_launch(ctx, cfg, xs::make_params(tables, first, n, seed, d_out, verify, nullptr), n, d_workspace,
                         workspace_bytes, static_cast<cudaStream_t>(stream));
}

extern "C" int gtr_xs_lookup_presorted_peers(gtr_ctx *ctx, const gtr_launch_cfg *cfg, const gtr_xs_tables *tables,
                                             uint64_t first, uint64_t n, uint64_t *const *h_peer_outs, int32_t n_peers,
                                             const void *d_workspace, uint64_t workspace_bytes, void *stream) {
    if (!ctx || !cfg || !tables_ok(tables) || !h_peer_outs || n_peers < 1 || n_peers > 8 || !d_workspace)
        return GTR_EINVAL;
    for (int p = 0; p < n_peers; p++)
        if (!h_peer_outs[p]) return GTR_EINVAL;
    if (n == 0) return GTR_OK;
    xs::Params P = xs::make_params(tables, first, n, 0, h_peer_outs[0], nullptr, nullptr);
    P.n_peers = n_peers;
    for (int p = 0; p < n_peers; p++) P.peer_out[p] = reinterpret_cast<unsigned long long *>(h_peer_outs[p]);
    return presorted_pass(ctx, cfg, P, n, const_cast<void *>(d_workspace), workspace_bytes,
                          static_cast<cudaStream_t>(stream));
}

extern "C" int gtr_xs_lookup_sorted_host(gtr_ctx *ctx, const gtr_launch_cfg *cfg, const gtr_xs_tables *tables,
                                         const gtr_xs_request *h_req, uint64_t *h_out, void *d_workspace,
                                         uint64_t workspace_bytes, void *stream) {
    if (!ctx || !cfg || !tables_ok(tables) || !h_req || !h_out || !d_workspace) return GTR_EINVAL;
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    gtr_xs_request *d_req = static_cast<gtr_xs_request *>(ctx->d_stage);
    uint64_t *d_out = reinterpret_cast<uint64_t *>(static_cast<char *>(ctx->d_stage) + 64);
    GTR_CUDA_TRY(cudaMemcpyAsync(d_req, h_req, sizeof(gtr_xs_request), cudaMemcpyHostToDevice, s));
    GTR_CUDA_TRY(cudaMemsetAsync(d_out, 0, 18 * sizeof(uint64_t), s));
    if (h_req->n) {
        // the kernels read (first, seed) from d_req; n sizes the launches and the workspace
        const int st = sorted_launch(ctx, cfg,
                                     xs::make_params(tables, h_req->first, h_req->n, h_req->seed, d_out, nullptr,
                                                     d_req),
                                     h_req->n, d_workspace, workspace_bytes, s);
        if (st) return st;
    }
    GTR_CUDA_TRY(cudaMemcpyAsync(h_out, d_out, 18 * sizeof(uint64_t), cudaMemcpyDeviceToHost, s));
    GTR_CUDA_TRY(cudaStreamSynchronize(s));
    return GTR_OK;
}

extern "C" int gtr_xs_lookup_peers(gtr_ctx *ctx, const gtr_launch_cfg *cfg, const gtr_xs_tables *tables,
                                   uint64_t first, uint64_t n, uint64_t seed, uint64_t *const *h_peer_outs,
                                   int32_t n_peers, void *stream) {
    if (!ctx || !cfg || !tables_ok(tables) || !h_peer_outs || n_peers < 1 || n_peers > 8) return GTR_EINVAL;
    for (int p = 0; p < n_peers; p++)
        if (!h_peer_outs[p]) return GTR_EINVAL;
    if (n == 0) return GTR_OK;
    xs::Params P = xs::make_params(tables, first, n, seed, h_peer_outs[0], nullptr, nullptr);
    P.n_peers = n_peers;
    for (int p = 0; p < n_peers; p++) P.peer_out[p] = reinterpret_cast<unsigned long long *>(h_peer_outs[p]);
    xs::LaunchArgs a{ctx, cfg, P, static_cast<cudaStream_t>(stream), nullptr};
    return xs::launch(a);
}
