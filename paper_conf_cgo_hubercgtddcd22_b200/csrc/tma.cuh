// tma.cuh -- sm_100a bulk asynchronous copies (the TMA engine's 1-D form) and
// mbarrier completion, as inline PTX.  Used to stream HBM-bound tiles
// (SU3 lattice sites) through shared memory without registers: one thread
// issues a bulk copy of a whole tile, the copy engine signals an mbarrier with
// the byte count, consumers wait on the barrier's phase parity.
#pragma once
#include <cstdint>

namespace gtr {
namespace tma {

__device__ __forceinline__ uint32_t smem_addr(const void *p) {
    return (uint32_t)__cvta_generic_to_shared(p);
}
// one arrival expected per phase (the producer's arrive.expect_tx)
__device__ __forceinline__ void mbar_init(uint64_t *bar) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_addr(bar)) : "memory");
}
// make the initialised barrier visible to the async proxy (the copy engine)
__device__ __forceinline__ void fence_mbar_init() {
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
// producer: arrive and announce `bytes` of transactions, then start a global
// -> shared bulk copy that completes them (dst, src, bytes: 16-byte multiples)
__device__ __forceinline__ void load_async(void *dst, const void *src, uint32_t bytes, uint64_t *bar) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_addr(bar)), "r"(bytes)
                 : "memory");
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     smem_addr(dst)),
                 "l"(src), "r"(bytes), "r"(smem_addr(bar))
                 : "memory");
}
// consumer: wait until the barrier completed the phase with parity `parity`.
// Watchdog: after `limit` unsuccessful try_waits (each suspends for a
// hardware-chosen time) set `hang_bit` in *err and return -- the data is then
// invalid and the host sees the error (gtr_ctx_check).
__device__ __forceinline__ bool mbar_try_wait(uint64_t *bar, uint32_t parity) {
    uint32_t ok;
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, p;\n}"
        : "=r"(ok)
        : "r"(smem_addr(bar)), "r"(parity)
        : "memory");
    return ok != 0;
}
__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t parity, uint64_t limit, uint32_t *err,
                                          uint32_t hang_bit) {
    for (uint64_t polls = 0; !mbar_try_wait(bar, parity);) {
        if (++polls >= limit) {
            atomicOr(err, hang_bit);
            return;
        }
    }
}
// order this thread's generic-proxy shared-memory writes before later async-
// proxy reads (a bulk store issued after a barrier)
__device__ __forceinline__ void fence_async_shared() {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
// shared -> global bulk store, tracked in the issuing thread's bulk group
__device__ __forceinline__ void store_async(void *dst, const void *src, uint32_t bytes) {
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst), "r"(smem_addr(src)),
                 "r"(bytes)
                 : "memory");
    asm volatile("cp.async.bulk.commit_group;" ::: "memory");
}
// the issuing thread: wait until the source of every committed bulk store was
// read (the shared buffer may be overwritten)
__device__ __forceinline__ void store_wait_read() { asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory"); }
// ... and until the stores completed (before the CTA exits)
__device__ __forceinline__ void store_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }

}  // namespace tma
}  // namespace gtr
