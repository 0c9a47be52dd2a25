// gather_bench.cu -- microbenchmark of the XS gather pattern (tools only, not
// part of libgtr): every lane needs one random 96-byte record (two 48-byte
// gridpoints, 16-byte aligned) per step.  Variants:
//   0  per-lane exact-size loads (3 x 256 bit, or 128+256+256+128)  [current kernel]
//   1  cooperative cp.async: 6 lanes copy one record's 16-byte chunks into a
//      per-warp shared ring (2 stages), each lane then reads its own record
//      with 6 x LDS.128 (112-byte stride: conflict-free)
//   2  cooperative LDG.128 into registers -> STS.128 -> LDS.128 (same layout)
// Reports time and a checksum; run under ncu for l1tex wavefronts.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t hash32(uint32_t x) {
    x ^= x >> 16; x *= 0x7feb352dU; x ^= x >> 15; x *= 0x846ca68bU; x ^= x >> 16; return x;
}
__device__ __forceinline__ void ld256(const double *a, double &x0, double &x1, double &x2, double &x3) {
    asm("ld.global.nc.v4.f64 {%0, %1, %2, %3}, [%4];" : "=d"(x0), "=d"(x1), "=d"(x2), "=d"(x3) : "l"(a));
}
__device__ __forceinline__ double2 ld128(const double *a) {
    double2 v;
    asm("ld.global.nc.v2.f64 {%0, %1}, [%2];" : "=d"(v.x), "=d"(v.y) : "l"(a));
    return v;
}

constexpr int NT = 256;
constexpr int STR = 14;   // doubles per record slot (112 B)

template <int V, int D = 2, int MINB = 2>
__global__ void __launch_bounds__(NT, MINB) kern(const double *__restrict__ grid, uint32_t nrec, int steps, double *out) {
    extern __shared__ __align__(16) double dring[];
    double (*ring)[D][32 * STR] = reinterpret_cast<double (*)[D][32 * STR]>(dring);
    const unsigned lane = threadIdx.x & 31u, w = threadIdx.x >> 5;
    const uint32_t gw = blockIdx.x * (NT / 32) + w;
    double acc = 0.0;
    auto rec_of = [&](int j, unsigned l) { return hash32(gw * 0x9E3779B9u + (uint32_t)j * 32u + l) % (nrec - 1); };
    if constexpr (V == 0) {
        for (int j = 0; j < steps; j++) {
            const uint64_t off = (uint64_t)rec_of(j, lane) * 6;
            const double *r = grid + off;
            double v[12];
            if ((off & 3) == 0) {
                ld256(r, v[0], v[1], v[2], v[3]); ld256(r + 4, v[4], v[5], v[6], v[7]); ld256(r + 8, v[8], v[9], v[10], v[11]);
            } else {
                double2 a = ld128(r); ld256(r + 2, v[2], v[3], v[4], v[5]); ld256(r + 6, v[6], v[7], v[8], v[9]);
                double2 b = ld128(r + 10); v[0] = a.x; v[1] = a.y; v[10] = b.x; v[11] = b.y;
            }
            double s = 0;
#pragma unroll
            for (int q = 0; q < 12; q++) s += v[q];
            acc += s;
        }
    } else {
        auto issue = [&](int j, double *slot) {
            const uint32_t myrec = rec_of(j, lane);
#pragma unroll
            for (int s = 0; s < 6; s++) {
                const unsigned q = s * 32 + lane, L = q / 6, c = q % 6;
                const uint32_t r = __shfl_sync(0xffffffffu, myrec, L);
                const double *src = grid + (uint64_t)r * 6 + 2 * c;
                double *dst = slot + L * STR + 2 * c;
                if constexpr (V == 1) {
                    const uint32_t d = (uint32_t)__cvta_generic_to_shared(dst);
                    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(d), "l"(src) : "memory");
                } else {
                    *reinterpret_cast<double2 *>(dst) = ld128(src);
                }
            }
            if constexpr (V == 1) asm volatile("cp.async.commit_group;" ::: "memory");
        };
#pragma unroll
        for (int p = 0; p < D - 1; p++) issue(p, ring[w][p]);
        for (int j = 0; j < steps; j++) {
            if (j + D - 1 < steps) issue(j + D - 1, ring[w][(j + D - 1) % D]);
            else if constexpr (V == 1) asm volatile("cp.async.commit_group;" ::: "memory");
            if constexpr (V == 1) asm volatile("cp.async.wait_group %0;" ::"n"(D - 1) : "memory");
            __syncwarp();
            const double2 *p = reinterpret_cast<const double2 *>(ring[w][j % D] + lane * STR);
            double s = 0;
#pragma unroll
            for (int q = 0; q < 6; q++) { double2 x = p[q]; s += x.x; s += x.y; }
            acc += s;
            __syncwarp();
        }
    }
    out[blockIdx.x * NT + threadIdx.x] = acc;
}

int main(int argc, char **argv) {
    const uint32_t nrec = argc > 2 ? (uint32_t)atol(argv[2]) : 355u * 11303u;
    const int steps = argc > 1 ? atoi(argv[1]) : 400;
    double *grid, *out;
    cudaMalloc(&grid, (size_t)nrec * 48 + 256);
    cudaMemset(grid, 0, (size_t)nrec * 48);
    cudaMalloc(&out, 296 * NT * 8);
    // fill with something
    double *h = (double *)malloc((size_t)nrec * 48);
    for (size_t i = 0; i < (size_t)nrec * 6; i++) h[i] = (double)(i % 1000) * 0.001;
    cudaMemcpy(grid, h, (size_t)nrec * 48, cudaMemcpyHostToDevice);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0); cudaEventCreate(&e1);
    auto run = [&](const char *name, auto kfn, int dd, int blocks_) {
        const int smem = (NT / 32) * dd * 32 * STR * 8;
        cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
        float ms = 0;
        for (int rep = 0; rep < 3; rep++) {
            cudaEventRecord(e0);
            kfn<<<blocks_, NT, smem>>>(grid, nrec, steps * 296 / blocks_, out);
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            cudaEventElapsedTime(&ms, e0, e1);
        }
        const double recs = (double)296 * NT * steps;
        printf("%-28s smem %6d B: %.3f ms, %.1f G records/s, %.2f TB/s (96 B)\n", name, smem, ms, recs / ms / 1e6, recs * 96 / ms / 1e9);
    };
    run("perlane", kern<0, 2, 2>, 2, 296);
    run("cpasync D2 2cta", kern<1, 2, 2>, 2, 296);
    run("cpasync D3 2cta", kern<1, 3, 2>, 3, 296);
    run("cpasync D4 1cta", kern<1, 4, 1>, 4, 148);
    run("cpasync D6 1cta", kern<1, 6, 1>, 6, 148);
    printf("err %s\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
