// sampling.cuh -- the lookup sampling shared by the XS and RS kernels:
// lookup i draws its energy E and material from the 63-bit LCG jumped ahead
// 2i steps from the lookup seed (the paper is silent, the
// apps' convention [ext]).  Independent of the oracle's implementation.
#pragma once
#include <cstdint>

namespace gtr {
namespace smp {

// 63-bit LCG s <- (a s + c) mod 2^63, implemented here
// independently of the oracle.
__device__ __forceinline__ uint64_t lcg_step(uint64_t s) {
    return (2806196910506780709ULL * s + 1ULL) & 0x7FFFFFFFFFFFFFFFULL;
}
__device__ __forceinline__ double lcg_uniform(uint64_t &s) {
    s = lcg_step(s);
    return __ull2double_rn(s) * 0x1p-63;     // exact scaling by 2^-63
}
// The affine map of n steps, x -> A x + C (mod 2^63), by squaring.
__host__ __device__ __forceinline__ void lcg_map(uint64_t n, uint64_t &A, uint64_t &C) {
    uint64_t mul = 2806196910506780709ULL, add = 1ULL;       // current power of the map
    uint64_t acc_mul = 1ULL, acc_add = 0ULL;                  // accumulated map
    n &= 0x7FFFFFFFFFFFFFFFULL;
    while (n) {
        if (n & 1ULL) {
            acc_mul = acc_mul * mul;
            acc_add = acc_add * mul + add;
        }
        add = add * (mul + 1ULL);
        mul = mul * mul;
        n >>= 1;
    }
    A = acc_mul;
    C = acc_add;
}
// Jump ahead n steps (arithmetic mod 2^64 then masked: 2^63 divides 2^64, so
// composing maps this way is exact mod 2^63).
__device__ __forceinline__ uint64_t lcg_jump(uint64_t seed, uint64_t n) {
    uint64_t A, C;
    lcg_map(n, A, C);
    return (A * seed + C) & 0x7FFFFFFFFFFFFFFFULL;
}
__device__ __forceinline__ uint64_t lcg_apply(uint64_t A, uint64_t C, uint64_t s) {
    return (A * s + C) & 0x7FFFFFFFFFFFFFFFULL;
}
// Material draw: cumulative thresholds built in XSBench's order
// (dist[i] + dist[i-1] + ... + dist[1]); P(material 0) is the remainder.
__device__ __forceinline__ int sample_material(uint64_t &s) {
    const double d1 = 0.052, d2 = 0.275, d3 = 0.134, d4 = 0.154, d5 = 0.064, d6 = 0.066,
                 d7 = 0.055, d8 = 0.008, d9 = 0.015, d10 = 0.025, d11 = 0.013;
    const double c[12] = {0.0,
                          d1,
                          (d2 + d1),
                          ((d3 + d2) + d1),
                          (((d4 + d3) + d2) + d1),
                          ((((d5 + d4) + d3) + d2) + d1),
                          (((((d6 + d5) + d4) + d3) + d2) + d1),
                          ((((((d7 + d6) + d5) + d4) + d3) + d2) + d1),
                          (((((((d8 + d7) + d6) + d5) + d4) + d3) + d2) + d1),
                          ((((((((d9 + d8) + d7) + d6) + d5) + d4) + d3) + d2) + d1),
                          (((((((((d10 + d9) + d8) + d7) + d6) + d5) + d4) + d3) + d2) + d1),
                          ((((((((((d11 + d10) + d9) + d8) + d7) + d6) + d5) + d4) + d3) + d2) + d1)};
    const double r = lcg_uniform(s);
#pragma unroll
    for (int m = 1; m < 12; m++)
        if (r < c[m]) return m;
    return 0;
}

}  // namespace smp
}  // namespace gtr
