// rs_impl.cuh -- RSBench-style windowed multipole cross-section lookup
// (BASELINE config 4) on the team runtime.
//
// Paper: RSBench is the compute-bound alternative to XSBench,
// timed as `rsbench -s large -m event`; already SPMD, 7 globalized
// variables (Fig. 9) whose runtime globalization caused OOM or
// "tremendous slowdowns" until heap-to-stack applied.
// Algorithm step by step as in oracle/rs.c (R1-R6),
// written independently here.  Globalized per-lookup variables (AMB-7):
// seed, macro[4], micro[4], sigTfactors[4] (complex), Z, W, sig[3].
// Shapes as XS: GENERIC/CASCADE/CSM `teams distribute` over lookup chunks with
// a forked `parallel for`; SPMD-ized; NATIVE thread per lookup.
#pragma once
#include <cfloat>

#include "gtr_internal.h"
#include "sampling.cuh"

namespace gtr {
namespace rs {

struct Params {
    const int32_t *n_windows;
    const double *poles;      // 9 words per record
    const double *windows;    // 4 words per record
    const double *k0rs;
    const int32_t *num_nucs;
    const int32_t *mats;
    const double *concs;
    const double *poles_wide; // 12 words per record, 32-byte aligned, or null
    int32_t wide;             // windows and k0rs 32-byte aligned: 256-bit loads
    int64_t n_nuc, max_poles, max_windows;
    int32_t max_num_nucs;
    uint32_t chunk;
    int32_t plain;            // 1: the paper's schedule (GTR_F_PLAIN)
    uint64_t first, n, seed;
    uint8_t *v_mat;
    uint8_t *v_am;
    double *v_macro;
    unsigned long long *out;
};

// ---- complex arithmetic in RSBench's operation order ----------------------
struct cx {
    double r, i;
};
__device__ __forceinline__ cx cadd(cx a, cx b) { return {a.r + b.r, a.i + b.i}; }
__device__ __forceinline__ cx csub(cx a, cx b) { return {a.r - b.r, a.i - b.i}; }
__device__ __forceinline__ cx cmul(cx a, cx b) { return {a.r * b.r - a.i * b.i, a.r * b.i + a.i * b.r}; }
__device__ __forceinline__ cx cdiv(cx a, cx b) {
    const double d = b.r * b.r + b.i * b.i;
    return {((a.r * b.r) + (a.i * b.i)) / d, ((a.i * b.r) - (a.r * b.i)) / d};
}
__device__ __forceinline__ double cabs_(cx a) { return sqrt(a.r * a.r + a.i * a.i); }

#ifndef GTR_RS_PREFETCH
#define GTR_RS_PREFETCH 1
#endif
#ifndef GTR_RS_PRESUF
#define GTR_RS_PRESUF 0
#endif
#ifndef GTR_RS_SF_SELECT
#define GTR_RS_SF_SELECT 0
#endif
#ifndef GTR_RS_PCOPY
#define GTR_RS_PCOPY 0   // measured: the copy spills at 128 registers, 104.1 -> 99.8 M lookups/s
#endif
__device__ __forceinline__ void ld256(const double *a, double &x0, double &x1, double &x2, double &x3) {
    asm("ld.global.nc.v4.f64 {%0, %1, %2, %3}, [%4];" : "=d"(x0), "=d"(x1), "=d"(x2), "=d"(x3) : "l"(a));
}

__device__ __forceinline__ double fast_exp(double x) {
    x = 1.0 + x * 0.000244140625;
#pragma unroll
    for (int k = 0; k < 12; k++) x *= x;
    return x;
}
__device__ __forceinline__ cx fast_cexp(cx z) {
    const double t1 = fast_exp(z.r);
    double s, c;
    sincos(z.i, &s, &c);
    return {t1 * c, t1 * s};
}

// Faddeeva W(z): Abrarov series (N = 10, Tm = 12) inside |z| < 6, two-pole
// asymptotic expansion outside; RSBench's tabulated constants.
//
// Evaluated for sm_100a's fp64 units rather than in RSBench's operation
// order (parity is within R-RS-tol): the 11 complex divisions of
// the inner branch share ONE reciprocal (batched inversion of the real
// denominators |12 Z|^2 and |dl_n - 144 Z^2|^2, prefix products), the
// loop-invariant exp(12 i Z) and 144 Z^2 are computed once, and the ten terms
// collapse into two sums because the numerators alternate between
// -e - 1 (n even) and e - 1 (n odd).  RSBench's form needs 22 fp64 divisions
// per pole, each an XU-pipe reciprocal plus a Newton sequence; the XU pipe
// was the busiest unit (ncu: 75% of peak).
//
// The branch must be the oracle's: |Z| = sqrt(Z.r*Z.r + Z.i*Z.i) < 6 with
// every operation rounded separately (no FMA -- this TU contracts, so the
// squares and the sum are explicit round-to-nearest intrinsics).  Then
// sqrt(x) < 6 <=> x < 36 for every double x: sqrt is monotonic, correctly
// rounded, and sqrt(pred(36)) = 6 - 0.667 ulp(6^-) rounds below 6 (pinned
// by tests/test_oracle_rs.py::test_branch_predicate_sqrt_equivalence).
__device__ __forceinline__ bool faddeeva_inner_branch(cx Z) {
    return __dadd_rn(__dmul_rn(Z.r, Z.r), __dmul_rn(Z.i, Z.i)) < 36.0;
}
// e = exp(12 i Z) (fast_cexp); the wide-pole path passes it precomputed
__device__ __forceinline__ cx faddeeva_series(cx Z, cx e) {
    {
        constexpr double an[10] = {2.758402e-01, 2.245740e-01, 1.594149e-01, 9.866577e-02, 5.324414e-02,
                                   2.505215e-02, 1.027747e-02, 3.676164e-03, 1.146494e-03, 3.117570e-04};
        constexpr double dl[10] = {9.869604e+00, 3.947842e+01, 8.882644e+01, 1.579137e+02, 2.467401e+02,
                                   3.553058e+02, 4.836106e+02, 6.316547e+02, 7.994379e+02, 9.869604e+02};
        const cx den = {12.0 * Z.r, 12.0 * Z.i};                        // 12 Z
        const double b_r = 144.0 * (Z.r * Z.r - Z.i * Z.i), b_i = 144.0 * (2.0 * Z.r * Z.i);   // 144 Z^2
        // batched inversion of q_0 = |12 Z|^2, q_{n+1} = |dl_n - 144 Z^2|^2
#if GTR_RS_PRESUF
        // prefix and suffix products side by side (two independent chains of
        // 10 instead of prefix -> reciprocal -> backward sweep): 1/q_n =
        // pre[n] * suf[n+1] / P, a shorter dependent path per pole
        double q[11], pre[11], suf[12];
        q[0] = den.r * den.r + den.i * den.i;
#pragma unroll
        for (int n = 0; n < 10; n++) {
            const double br = dl[n] - b_r;
            q[n + 1] = br * br + b_i * b_i;
        }
        pre[0] = 1.0;
        suf[11] = 1.0;
#pragma unroll
        for (int n = 0; n < 10; n++) {
            pre[n + 1] = pre[n] * q[n];
            suf[10 - n] = suf[11 - n] * q[10 - n];
        }
        const double invP = 1.0 / (pre[10] * q[10]);
        cx Se = {0.0, 0.0}, So = {0.0, 0.0};
#pragma unroll
        for (int n = 9; n >= 0; n--) {
            const double br = dl[n] - b_r;
            const double w = an[n] * ((pre[n + 1] * suf[n + 2]) * invP);  // an / q_{n+1}
            if (n & 1) { So.r += w * br; So.i += w * b_i; }
            else       { Se.r += w * br; Se.i += w * b_i; }
        }
        const double inv = (pre[0] * suf[1]) * invP;                      // 1 / q_0
#else
        double pre[11];
        pre[0] = den.r * den.r + den.i * den.i;
#pragma unroll
        for (int n = 0; n < 10; n++) {
            const double br = dl[n] - b_r;
            pre[n + 1] = pre[n] * (br * br + b_i * b_i);
        }
        double inv = 1.0 / pre[10];
        cx Se = {0.0, 0.0}, So = {0.0, 0.0};
#pragma unroll
        for (int n = 9; n >= 0; n--) {
            const double br = dl[n] - b_r;
            const double w = an[n] * (inv * pre[n]);                     // an / |bot_n|^2
            inv *= br * br + b_i * b_i;
            if (n & 1) { So.r += w * br; So.i += w * b_i; }             // an conj(bot_n) / |bot_n|^2
            else       { Se.r += w * br; Se.i += w * b_i; }
        }
#endif
        // W0 = i (1 - e) / (12 Z) = {e.i, 1 - e.r} conj(den) / |den|^2
        const double nr = e.i, ni = 1.0 - e.r;
        const cx W0 = {(nr * den.r + ni * den.i) * inv, (ni * den.r - nr * den.i) * inv};
        const cx te = {-e.r - 1.0, -e.i}, to = {e.r - 1.0, e.i};
        const cx sum = cadd(cmul(te, Se), cmul(to, So));
        const cx zs = cmul(Z, sum);
        return {W0.r - 8.124330e+01 * zs.i, W0.i + 8.124330e+01 * zs.r};   // W0 + i 81.2433 Z sum
    }
}
__device__ __forceinline__ cx faddeeva_asymptotic(cx Z);
__device__ __forceinline__ cx faddeeva(cx Z) {
    if (faddeeva_inner_branch(Z)) return faddeeva_series(Z, fast_cexp(cx{-12.0 * Z.i, 12.0 * Z.r}));   // exp(i 12 Z)
    return faddeeva_asymptotic(Z);
}
// the wide-pole form: exp(12 i Z) = t1 * exp(6 i E) * exp(-6 i EA.r), the
// pole's factors t1 = fast_exp(-12 Z.i) (bit-identical to computing it here)
// and (cos, sin)(6 EA.r) precomputed in its record, (cE, sE) = (cos, sin)(6 E)
// once per lookup: one complex rotation instead of fast_exp + sincos per pole
// (6 E - 6 EA.r = 12 Z.r in exact arithmetic; the phase differs from the
// oracle's 12 Z.r by rounding only, ~1e-15 rad, within R-RS-tol)
__device__ __forceinline__ cx faddeeva_pre(cx Z, double t1, double cp, double sp, double cE, double sE) {
    if (faddeeva_inner_branch(Z)) {
        const double c = cE * cp + sE * sp, sn = sE * cp - cE * sp;
        return faddeeva_series(Z, cx{t1 * c, t1 * sn});
    }
    return faddeeva_asymptotic(Z);
}
__device__ __forceinline__ cx faddeeva_asymptotic(cx Z) {
    const cx a = {0.512424224754768462984202823134979415014943561548661637413182, 0.0};
    const cx b = {0.275255128608410950901357962647054304017026259671664935783653, 0.0};
    const cx c = {0.051765358792987823963876628425793170829107067780337219430904, 0.0};
    const cx d = {2.724744871391589049098642037352945695982973740328335064216346, 0.0};
    const cx I = {0.0, 1.0};
    const cx Z2 = cmul(Z, Z);
    return cmul(cmul(Z, I), cadd(cdiv(a, csub(Z2, b)), cdiv(c, csub(Z2, d))));
}

struct TagSeed {};
struct TagMacro {};
struct TagMicro {};
struct TagSigTF {};
struct TagZ {};
struct TagW {};
struct TagSig {};

// microscopic XS of nuclide nuc at energy E (4 channels) into micro
template <class K, class LM>
__device__ __forceinline__ void micro_xs(const Params &P, int64_t nuc, double E, double cE, double sE, LM &micro) {
    Local<K, double, 8, TagSigTF> sf;     // sigTfactors[4] complex
    Local<K, double, 2, TagZ> Zv;
    Local<K, double, 2, TagW> Wv;
    Local<K, double, 3, TagSig> sig;
    const int32_t nw = __ldg(P.n_windows + nuc);
    const double spacing = 1.0 / nw;
    int32_t window = (int32_t)(E / spacing);
    if (window == nw) window--;
    const double sqE = sqrt(E);
    double k0[4];
    if (P.wide) {
        ld256(P.k0rs + nuc * 4, k0[0], k0[1], k0[2], k0[3]);
    } else {
#pragma unroll
        for (int l = 0; l < 4; l++) k0[l] = __ldg(P.k0rs + nuc * 4 + l);
    }
#pragma unroll
    for (int l = 0; l < 4; l++) {
        double phi = k0[l] * sqE;
        if (l == 1) phi -= -atan(phi);
        else if (l == 2) phi -= atan(3.0 * phi / (3.0 - phi * phi));
        else if (l == 3) phi -= atan(phi * (15.0 - phi * phi) / (15.0 - 6.0 * phi * phi));
        phi *= 2.0;
        double s, c;
        sincos(phi, &s, &c);
        sf[2 * l] = c;
        sf[2 * l + 1] = -s;
    }
    const double *w = P.windows + (nuc * P.max_windows + window) * 4;
    double wT, wA, wF, wse;
    if (P.wide) {                                    // one 32-byte record, one sector
        ld256(w, wT, wA, wF, wse);
    } else {
        wT = __ldg(w + 0);
        wA = __ldg(w + 1);
        wF = __ldg(w + 2);
        wse = __ldg(w + 3);
    }
    const int2 se = make_int2(__double2loint(wse), __double2hiint(wse));
    sig[0] = E * wT;
    sig[1] = E * wA;
    sig[2] = E * wF;
    // one pole (c4 step 4), in pole order
    // pre: a wide record's {t1, cos 6EA.r, sin 6EA.r}
    auto pole = [&](double2 EA, double2 RT, double2 RA, double2 RF, int lv, bool pre, double t1, double cp,
                    double sp) {
        const cx Z = cmul(csub(cx{E, 0.0}, cx{EA.x, EA.y}), cx{0.5, 0.0});
        Zv[0] = Z.r;
        Zv[1] = Z.i;
        const cx W = pre ? faddeeva_pre(cx{Zv[0], Zv[1]}, t1, cp, sp, cE, sE) : faddeeva(cx{Zv[0], Zv[1]});
        Wv[0] = W.r;
        Wv[1] = W.i;
        const cx Wl = {Wv[0], Wv[1]};
#if GTR_RS_SF_SELECT
        // constant indices only: in the heap-to-stack placement the factors
        // stay in registers (a runtime index puts the array in local memory,
        // one 16-byte LDL per pole)
        cx f = {sf[0], sf[1]};
        if (lv == 1) f = cx{sf[2], sf[3]};
        if (lv == 2) f = cx{sf[4], sf[5]};
        if (lv == 3) f = cx{sf[6], sf[7]};
#else
        const cx f = {sf[2 * lv], sf[2 * lv + 1]};
#endif
        sig[0] = sig[0] + cmul(cx{RT.x, RT.y}, cmul(Wl, f)).r;
        sig[1] = sig[1] + cmul(cx{RA.x, RA.y}, Wl).r;
        sig[2] = sig[2] + cmul(cx{RF.x, RF.y}, Wl).r;
    };
    if (P.poles_wide) {
        // 96-byte records: 2 x 256 bit + the l word
        const double *base = P.poles_wide + nuc * P.max_poles * 12;
#if GTR_RS_PREFETCH
        // the next pole's first 32 bytes (EA, RT) are loaded before this
        // pole's Faddeeva evaluation: the load that starts each pole is
        // already in flight
        double2 nEA = {0.0, 0.0}, nRT = {0.0, 0.0};
        if (se.x < se.y) ld256(base + (int64_t)se.x * 12, nEA.x, nEA.y, nRT.x, nRT.y);
        for (int32_t p = se.x; p < se.y; p++) {
            const double *pr = base + (int64_t)p * 12;
            const double2 EA = nEA, RT = nRT;
            double2 RA, RF;
            double w8, t1, cp, sp;
            ld256(pr + 4, RA.x, RA.y, RF.x, RF.y);
            ld256(pr + 8, w8, t1, cp, sp);                       // l_value + the pole's exp factors
            if (p + 1 < se.y) ld256(pr + 12, nEA.x, nEA.y, nRT.x, nRT.y);
            pole(EA, RT, RA, RF, __double2loint(w8), true, t1, cp, sp);
        }
#else
        for (int32_t p = se.x; p < se.y; p++) {
            const double *pr = base + (int64_t)p * 12;
            double2 EA, RT, RA, RF;
            double w8, t1, cp, sp;
            ld256(pr + 0, EA.x, EA.y, RT.x, RT.y);
            ld256(pr + 4, RA.x, RA.y, RF.x, RF.y);
            ld256(pr + 8, w8, t1, cp, sp);
            pole(EA, RT, RA, RF, __double2loint(w8), true, t1, cp, sp);
        }
#endif
    } else {
        for (int32_t p = se.x; p < se.y; p++) {      // 72-byte records: 8-byte aligned only, scalar loads
            const double *pr = P.poles + (nuc * P.max_poles + p) * 9;
            pole(make_double2(__ldg(pr + 0), __ldg(pr + 1)), make_double2(__ldg(pr + 2), __ldg(pr + 3)),
                 make_double2(__ldg(pr + 4), __ldg(pr + 5)), make_double2(__ldg(pr + 6), __ldg(pr + 7)),
                 __ldg(reinterpret_cast<const int *>(pr + 8)), false, 0.0, 0.0, 0.0);
        }
    }
    micro[0] = sig[0];
    micro[1] = sig[1];
    micro[2] = sig[2];
    micro[3] = sig[0] - sig[1];
}

template <class K>
__device__ __forceinline__ void lookup(const Params &P, uint64_t i, uint32_t *tally) {
    Local<K, uint64_t, 1, TagSeed> seed;
    Local<K, double, 4, TagMacro> macro;
    Local<K, double, 4, TagMicro> micro;
    seed[0] = smp::lcg_jump(P.seed, 2ULL * i);
    const double E = smp::lcg_uniform(seed[0]);
    const int mat = smp::sample_material(seed[0]);
#pragma unroll
    for (int c = 0; c < 4; c++) macro[c] = 0.0;
    // the lookup's rotation exp(6 i E) for the wide records' precomputed pole factors
    double sE = 0.0, cE = 1.0;
    if (P.poles_wide) sincos(6.0 * E, &sE, &cE);
    const int nn = __ldg(P.num_nucs + mat);
    for (int j = 0; j < nn; j++) {
        const int64_t nuc = __ldg(P.mats + (int64_t)mat * P.max_num_nucs + j);
        const double conc = __ldg(P.concs + (int64_t)mat * P.max_num_nucs + j);
        micro_xs<K>(P, nuc, E, cE, sE, micro);
#pragma unroll
        for (int c = 0; c < 4; c++) macro[c] += micro[c] * conc;
    }
    double mx = -DBL_MAX;
    int am = 0;
#pragma unroll
    for (int c = 0; c < 4; c++)
        if (macro[c] > mx) { mx = macro[c]; am = c; }
    atomicAdd(&tally[mat], 1u);
    atomicAdd(&tally[12 + am], 1u);
    const uint64_t o = i - P.first;
    if (P.v_mat) P.v_mat[o] = (uint8_t)mat;
    if (P.v_am) P.v_am[o] = (uint8_t)am;
    if (P.v_macro) {
#pragma unroll
        for (int c = 0; c < 4; c++) P.v_macro[o * 4 + c] = macro[c];
    }
}

__device__ __forceinline__ void flush(const uint32_t *tally, unsigned long long *out, int tid, int nthr) {
    if (tid == 0) {
        unsigned long long h = 0;
        for (int a = 0; a < 4; a++) h += (unsigned long long)(a + 1) * tally[12 + a];
        if (h) atomicAdd(&out[0], h);
    }
    for (int k = tid; k < 17; k += nthr)
        if (tally[k]) atomicAdd(&out[1 + k], (unsigned long long)tally[k]);
}

static __shared__ Params g_p;
static __shared__ uint32_t g_tally[17];

struct Chunk {
    uint64_t base, count;
};
struct TagChunk {};

template <class K> struct LookupRegion {
    static constexpr int ID = 1;
    static __device__ void run(void *a) {
        const Chunk *c = static_cast<const Chunk *>(a);
        const uint64_t base = c->base, cnt = c->count;
        for_static<K>(0, (int64_t)cnt, [&](int64_t k) { lookup<K>(g_p, base + (uint64_t)k, g_tally); });
    }
};

// Material-bucketed schedule (as XS): fuel lookups evaluate 321
// nuclides' windows, the others 4-27, so a warp of mixed lookups idles most
// lanes.  Region 1 samples each lookup's material, the main thread forms
// buckets, region 2 scatters, region 3 runs whole lookups bucket by bucket
// with schedule(dynamic, 32).  Per-lookup arithmetic unchanged.
#ifndef GTR_RS_LPT
#define GTR_RS_LPT 32   // measured (10M, SPMD / CSM): 8: 93.7 / 84.2, 16: 104.1 / 98.4, 32: 105.8 / 99.1 M lookups/s
#endif
constexpr uint32_t kBucketLookupsPerThread = GTR_RS_LPT;
// Buckets are (material, energy bin): inside a material bucket the lookups
// are also grouped by energy (GTR_RS_EBINS bins of [0,1)), so the 32 lanes
// of a warp claim lookups of nearly equal energy -- they read the same
// windows and pole records (one L1 request per warp instead of one per lane)
// and run pole loops of equal length.  Results unchanged.
#ifndef GTR_RS_BALANCED
#define GTR_RS_BALANCED 0
#endif
#ifndef GTR_RS_EBINS
#define GTR_RS_EBINS 64
#endif
constexpr int kEBins = GTR_RS_EBINS;
constexpr int kBuckets = 12 * kEBins;
__device__ __forceinline__ int bucket_of(int mat, double E) {
    int eb = (int)(E * (double)kEBins);
    eb = eb < kEBins - 1 ? eb : kEBins - 1;
    return mat * kEBins + eb;
}
template <class K> struct ChunkBuf {
    static constexpr int CH = kBucketLookupsPerThread * K::NT;
    uint16_t perm[CH];
    uint16_t key[CH];                // bucket of lookup k
    uint32_t cnt[kBuckets], cur[kBuckets];
    unsigned int next;
};
// sequential code of a chunk: zero the counters / turn them into bucket offsets
template <class K> __device__ __forceinline__ void buckets_reset(ChunkBuf<K> &b) {
    for (int m = 0; m < kBuckets; m++) b.cnt[m] = 0;
    b.next = 0;
}
template <class K> __device__ __forceinline__ void buckets_offsets(ChunkBuf<K> &b) {
    uint32_t off = 0;
    for (int m = 0; m < kBuckets; m++) {
        b.cur[m] = off;
        off += b.cnt[m];
    }
}
template <class K> __device__ __forceinline__ ChunkBuf<K> &chunk_buf() {
    if constexpr (K::MODE == NATIVE) return *reinterpret_cast<ChunkBuf<K> *>(g_dyn);   // no runtime state
    const uint32_t off = tstate_bytes<K>() + (uint32_t)K::BLOCK * g_ts.rp.sm_stride_words * 8u;
    return *reinterpret_cast<ChunkBuf<K> *>(g_dyn + ((off + 15u) & ~15u));
}
template <class K> struct SampleRegion {
    static constexpr int ID = 2;
    static __device__ void run(void *a) {
        const Chunk *c = static_cast<const Chunk *>(a);
        const uint64_t base = c->base, cnt = c->count;
        ChunkBuf<K> &b = chunk_buf<K>();
        for_static<K>(0, (int64_t)cnt, [&](int64_t k) {
            uint64_t s = smp::lcg_jump(g_p.seed, 2ULL * (base + (uint64_t)k));
            const double E = smp::lcg_uniform(s);       // the energy draw
            const int m = smp::sample_material(s);
            const int key = bucket_of(m, E);
            b.key[k] = (uint16_t)key;
            atomicAdd(&b.cnt[key], 1u);
        });
    }
};
template <class K> struct ScatterRegion {
    static constexpr int ID = 3;
    static __device__ void run(void *a) {
        const uint64_t cnt = static_cast<const Chunk *>(a)->count;
        ChunkBuf<K> &b = chunk_buf<K>();
        for_static<K>(0, (int64_t)cnt, [&](int64_t k) {
            const uint32_t pos = atomicAdd(&b.cur[b.key[k]], 1u);
            b.perm[pos] = (uint16_t)k;
        });
    }
};
template <class K> struct BucketRegion {
    static constexpr int ID = 4;
    static __device__ void run(void *a) {
        const Chunk *c = static_cast<const Chunk *>(a);
        const uint64_t base = c->base, cnt = c->count;
        ChunkBuf<K> &b = chunk_buf<K>();
#if GTR_RS_PCOPY
        const Params P = g_p;      // register copy (g_p is shared memory; see xs_impl.cuh)
#else
        const Params &P = g_p;
#endif
        for_dynamic_warp<K>(0, (int64_t)cnt, &b.next,
                            [&](int64_t q) { lookup<K>(P, base + b.perm[q], g_tally); });
    }
};

// 4 teams of 128 per SM: caps registers at 128 (measured +2% over the
// unconstrained 146-register build, which fits 3)
#ifndef GTR_RS_MINB
#define GTR_RS_MINB 4
#endif
// generic modes (thread_limit + 32 threads per team): 3 teams of 160 per SM
// (<= 128 registers; 4 teams forced 96 and ~500 B of spills).  Measured on
// B200, RS 10M lookups: CSM 76.5 -> 83.4 M lookups/s.
#ifndef GTR_RS_MINB_GEN
#define GTR_RS_MINB_GEN 3
#endif
template <class K> __global__ void __launch_bounds__(K::BLOCK, K::NT == 128 ? (K::BLOCK > K::NT ? GTR_RS_MINB_GEN : GTR_RS_MINB) : 1) kernel_rt(Params P, RtParams rp) {
    const Role role = team_init<K>(rp);
    if (role == Role::Exit) return;
    if (role == Role::Worker) {
        worker_loop<K, LookupRegion<K>, SampleRegion<K>, ScatterRegion<K>, BucketRegion<K>>();
        return;
    }
    guarded<K>([&] {
        g_p = P;
        for (int k = 0; k < 17; k++) g_tally[k] = 0;
    });
    const uint64_t n = P.n, ch = P.chunk;
    const uint64_t nchunks = (n + ch - 1) / ch;
    distribute_static<K>(0, (int64_t)nchunks, [&](int64_t ci) {   // teams distribute
        const uint64_t c = (uint64_t)ci;
        TeamLocal<K, Chunk, TagChunk> chunk;
        chunk.set([&](Chunk &x) {
            x.base = P.first + c * ch;
            x.count = (c * ch + ch <= n) ? ch : n - c * ch;
        });
        if (P.plain) {
            parallel<K, LookupRegion<K>>(chunk.get());
            return;
        }
        ChunkBuf<K> &b = chunk_buf<K>();
        guarded<K>([&] { buckets_reset(b); });
        parallel<K, SampleRegion<K>>(chunk.get());
        guarded<K>([&] { buckets_offsets(b); });
        parallel<K, ScatterRegion<K>>(chunk.get());
        parallel<K, BucketRegion<K>>(chunk.get());
    });
    if constexpr (K::MODE == SPMD) flush(g_tally, g_p.out, threadIdx.x, K::NT);
    else flush(g_tally, g_p.out, 0, 1);
    team_deinit<K>();
}

// The CUDA watermark of the bucketed schedule (GTR_F_NATIVE_BUCKETED), as in
// xs_impl.cuh: the team program as a plain CUDA kernel, no runtime.
template <class K>
__global__ void __launch_bounds__(K::NT, K::NT == 128 ? GTR_RS_MINB : 1) kernel_native_bucketed(Params P) {
    static_assert(K::MODE == NATIVE, "plain CUDA");
    if (threadIdx.x == 0) {
        g_p = P;
        for (int k = 0; k < 17; k++) g_tally[k] = 0;
    }
    __syncthreads();
    const uint64_t n = g_p.n, ch = g_p.chunk;
    const uint64_t nchunks = (n + ch - 1) / ch;
    ChunkBuf<K> &b = chunk_buf<K>();
    __shared__ Chunk chunk;
    for (uint64_t c = blockIdx.x; c < nchunks; c += gridDim.x) {
        if (threadIdx.x == 0) {
            chunk.base = g_p.first + c * ch;
            chunk.count = (c * ch + ch <= n) ? ch : n - c * ch;
            buckets_reset(b);
        }
        __syncthreads();
        SampleRegion<K>::run(&chunk);
        __syncthreads();
        if (threadIdx.x == 0) buckets_offsets(b);
        __syncthreads();
        ScatterRegion<K>::run(&chunk);
        __syncthreads();
        BucketRegion<K>::run(&chunk);
        __syncthreads();
    }
    flush(g_tally, g_p.out, threadIdx.x, K::NT);
}

struct LaunchArgs {
    gtr_ctx *ctx;
    const gtr_launch_cfg *cfg;
    Params P;
    cudaStream_t stream;
    gtr_variant_info *info;
};

constexpr uint32_t kDefaultStackBytes = 256;   // 192 B per-lookup locals + chunk
constexpr uint32_t kLookupsPerThreadPerChunk = 2;

template <class K> struct OpRt {
    static int run(LaunchArgs &a) {
        const void *fn = reinterpret_cast<const void *>(&kernel_rt<K>);
        Launch L;
        int st = resolve<K>(a.ctx, a.cfg, fn, kDefaultStackBytes, &L, false,
                            a.P.plain ? 0u : (uint32_t)sizeof(ChunkBuf<K>) + 16u);
        if (st) return st;
        if (a.info) {
            int per_sm = 0;
            GTR_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, K::BLOCK, L.dyn_smem));
            return fill_info<K>(fn, L, per_sm, a.info);
        }
#if GTR_RS_BALANCED
        a.P.chunk = balanced_chunk(a.P.n, (a.P.plain ? kLookupsPerThreadPerChunk : kBucketLookupsPerThread) * K::NT,
                                   L.teams);
#else
        a.P.chunk = fit_chunk(a.P.n, (a.P.plain ? kLookupsPerThreadPerChunk : kBucketLookupsPerThread) * K::NT,
                              L.teams);
#endif
        kernel_rt<K><<<L.teams, L.block, L.dyn_smem, a.stream>>>(a.P, L.rp);
        GTR_CUDA_TRY(cudaGetLastError());
        return GTR_OK;
    }
};

}  // namespace rs
}  // namespace gtr
