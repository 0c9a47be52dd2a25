// gtr_rt.cuh -- the GPU team runtime: CPU-style OpenMP execution on a CTA.
//
// Device-side counterpart of the paper's "device runtime, roughly the GPU
// equivalent of the host OpenMP runtime" and of the kernel
// shapes its LLVM optimizations produce (Section IV).  Written for
// sm_100a; header-only, included by every kernel translation unit.
//
//   team = CTA, OpenMP thread = hardware thread        (Fig. 2)
//   GENERIC          main thread + worker state machine, regions passed as
//                    function pointers, workers call indirectly
//   GENERIC_CASCADE  workers compare the pointer against the known regions
//                    and call them directly, indirect fallback
//   CSM              custom state machine: region IDs, direct calls only, no
//                    address-taken region functions (fn. 4)
//   SPMD             SPMD-ized: all threads run the team code; side effects
//                    guarded by thread 0 + barrier, values broadcast through
//                    shared memory (Fig. 7)
//   NATIVE           plain CUDA (the paper's CUDA watermark);
//                    kernels written without this runtime.
//
// Globalization: Local<> / TeamLocal<> realise each globalized
// variable in one of four placements --
//   PL_RUNTIME        __runtime_alloc: per-thread LIFO stack in dynamic shared
//                     memory, global-memory fallback pool
//   PL_GLOBAL         the fallback only (shared stack of size 0; the paper's
//                     "LIBOMPTARGET_HEAP_SIZE" configuration)
//   PL_SHARED_STATIC  heap-to-shared: static __shared__ storage;
//                     per-thread variables scaled by the thread count (Fig. 6b)
//   PL_STACK          heap-to-stack: registers / local memory
//   PL_COALESCED      LLVM 12's globalization (Fig. 4b): one
//                     __runtime_coalesced_alloc per warp, every lane's copy at
//                     lane stride inside active parallel regions, runtime
//                     is_spmd / in_active_parallel checks, and the unsound
//                     SPMD shortcut to thread-private memory
//
// Runtime-call folding: with FOLD the execution-mode, parallel-
// level, thread-count and launch-parameter queries are compile-time constants;
// without it they read the team/thread state in shared memory.
#pragma once
#include <cstdint>
#include <cstring>
#include <cuda_runtime.h>

namespace gtr {

enum : int { GENERIC = 0, GENERIC_CASCADE = 1, CSM = 2, SPMD = 3, NATIVE = 4 };
enum : int { PL_RUNTIME = 0, PL_GLOBAL = 1, PL_SHARED_STATIC = 2, PL_STACK = 3, PL_COALESCED = 4 };
enum : uint32_t { ERR_HEAP = 1u, ERR_LIFO = 2u, ERR_DUP_ENERGY = 4u, ERR_BUILD = 8u, ERR_HANG = 16u };
enum : int { F_BCAST_1BAR = 1, F_SEPARATE_GUARDS = 2 };

// Compile-time kernel configuration.
template <int MODE_, int PL_, bool FOLD_, int NT_, int FLAGS_ = 0>
struct Cfg {
    static constexpr int MODE = MODE_, PL = PL_, NT = NT_, FLAGS = FLAGS_;
    static constexpr bool FOLD = FOLD_;
    static constexpr bool GENERIC_LIKE = (MODE_ <= CSM);
    // generic mode: NT workers + one extra warp whose lane 0 is the main thread
    static constexpr int BLOCK = GENERIC_LIKE ? NT_ + 32 : NT_;
    static constexpr int MAIN_HW = GENERIC_LIKE ? NT_ : 0;
    // per-thread runtime state (stack tops, nesting) lives in dynamic shared
    // memory for every variant: a STACK/SHARED_STATIC kernel may still make
    // runtime allocations for variables heap-to-stack could not move (Fig. 6b)
    static constexpr bool TSTATE = true;
    static_assert(NT_ % 32 == 0 && NT_ >= 32 && NT_ <= 1024 - (GENERIC_LIKE ? 32 : 0), "bad NT");
};

// Team-wide synchronisation of SPMD-mode code.  A team of one warp
// (thread_limit 32: BLOCK == 32) is synchronised by __syncwarp -- the warp's
// lanes are the whole team, and bar.warp.sync orders their shared-memory
// accesses ("Team = warp" guards) -- instead of a CTA barrier.
#ifndef GTR_WARP_TEAM
#define GTR_WARP_TEAM 1   // 0: one-warp teams use CTA barriers and the shared broadcast slot (A/B)
#endif
template <class K> __device__ __forceinline__ void cta_sync() {
    if constexpr (K::BLOCK == 32 && GTR_WARP_TEAM) __syncwarp();
    else __syncthreads();
}

// Launch-time runtime parameters (host-filled, by value).
struct RtParams {
    uint32_t *err;              // device error word (ctx-owned)
    unsigned long long *hwm;    // fallback high-water mark, bytes per thread (ctx-owned)
    uint64_t *pool;             // global fallback pool (caller-owned), may be null
    uint64_t pool_wpt;          // fallback capacity per hardware thread, 8-byte words
    uint32_t sm_stack_words;    // shared-memory stack capacity per thread (words)
    uint32_t sm_stride_words;   // per-thread stride of the stack (odd => no bank conflicts)
    uint64_t spin_limit;        // watchdog: polls of a spin-wait before it gives up with ERR_HANG
};

// Watchdog of the runtime's spin-waits (software barrier, mbarrier waits,
// the coalesced-free CAS loop): after `limit` polls the wait sets ERR_HANG in
// the context's error word and returns -- the kernel finishes with results
// declared invalid (gtr_ctx_check -> GTR_EDEVICE) instead of hanging the GPU.
__device__ __forceinline__ bool spin_expired(uint64_t &polls, uint64_t limit, uint32_t *err) {
    if (++polls < limit) return false;
    atomicOr(err, (uint32_t)ERR_HANG);
    return true;
}

typedef void (*RegionFn)(void *);

// Team state, one per CTA (static shared memory).
struct TeamState {
    RegionFn volatile fn;       // work descriptor (GENERIC / CASCADE)
    void *volatile args;
    volatile int32_t region_id; // work descriptor (CSM); 0 = terminate
    volatile int32_t level;     // team parallel level seen by workers (generic)
    volatile int32_t nthreads;  // threads of the active parallel region
    int32_t exec_mode;          // ICV read by non-folded is_spmd()
    volatile int32_t nvar;      // nthreads-var ICV (omp_set_num_threads)
    uint32_t sb_count;          // software barrier of a partial-warp team:
    volatile uint32_t sb_gen;   //   arrivals and generation
    volatile uint32_t hwm_seen; // largest fallback bytes/thread this team already reported
    RtParams rp;
    uint64_t bcast[2];          // guarded-value broadcast slots
};
static __shared__ TeamState g_ts;

// Per-thread state (dynamic shared memory, offset 0) -- only when TSTATE.
struct ThreadState {
    uint16_t sp;      // shared stack top (words)
    uint8_t nested;   // serialized nested parallel depth
    uint8_t level;    // SPMD: this thread's parallel level
    uint32_t gsp;     // global fallback stack top (words)
};                    // 8 bytes: a warp's accesses to .sp are 2-way bank conflicted at most
// PL_COALESCED only: per-lane + per-warp allocation state (after ThreadState)
struct CoalState {
    uint32_t igsp;    // this lane's own global stack top (divergent calls)
    uint32_t frame;   // frame slot k lives in lane k: live lanes << 16 | global << 15 | words
    uint32_t wtop;    // lane 0: warp stack top in shared memory (words)
    uint32_t wgtop;   // lane 0: warp slab top in the fallback pool (words)
    uint32_t nframes; // lane 0: frames on the warp stack
    uint32_t pad;
};
extern __shared__ __align__(16) uint8_t g_dyn[];

template <class K> __host__ __device__ constexpr uint32_t coal_offset() {
    return (uint32_t)((K::BLOCK * sizeof(ThreadState) + 15) / 16 * 16);
}
template <class K> __host__ __device__ constexpr uint32_t bphase_offset() {
    return coal_offset<K>() + (K::PL == 4 /*PL_COALESCED*/ ? (uint32_t)((K::BLOCK * sizeof(CoalState) + 15) / 16 * 16)
                                                           : 0u);
}
// F_BCAST_1BAR only: one u32 per thread, the slot of its next guarded_bcast
template <class K> __host__ __device__ constexpr uint32_t tstate_bytes() {
    return bphase_offset<K>() + ((K::FLAGS & 1 /*F_BCAST_1BAR*/) ? (uint32_t)((K::BLOCK * 4 + 15) / 16 * 16) : 0u);
}
template <class K> __device__ __forceinline__ uint32_t &bphase() {
    return reinterpret_cast<uint32_t *>(g_dyn + bphase_offset<K>())[threadIdx.x];
}
template <class K> __device__ __forceinline__ CoalState &cstate() {
    return reinterpret_cast<CoalState *>(g_dyn + coal_offset<K>())[threadIdx.x];
}
template <class K> __device__ __forceinline__ ThreadState &tstate() {
    return reinterpret_cast<ThreadState *>(g_dyn)[threadIdx.x];
}
template <class K> __device__ __forceinline__ uint64_t *sm_stack_base() {
    return reinterpret_cast<uint64_t *>(g_dyn + tstate_bytes<K>());
}

// ---------------------------------------------------------------- barriers
// Generic mode: the main thread arrives from divergent code while lanes
// 1..31 of its warp have exited; the non-aligned barrier.sync counts the
// team (NT workers + 1 warp).  SPMD: plain CTA barrier.
template <class K> __device__ __forceinline__ void team_barrier() {
    if constexpr (K::GENERIC_LIKE)
        asm volatile("barrier.sync 1, %0;" ::"n"(K::BLOCK) : "memory");
    else
        cta_sync<K>();
}

// `#pragma omp barrier` inside a parallel region: the region's threads only
// (generic: the NT workers on named barrier 2; the main thread waits at the
// join).  SPMD: the whole CTA.
// A team smaller than NT (num_threads clause / ICV, non-folded variants):
// named barrier 2 over its warps when it is whole warps, else a software
// barrier in shared memory.  Serialized nested regions: a team of one.
// Every access to the barrier's count and generation is atomic (the waiting
// threads poll the generation the last arrival advances).
__device__ __forceinline__ uint32_t atomic_load_shared(uint32_t *a) { return atomicOr(a, 0u); }
static __device__ __noinline__ void soft_barrier(int n) {
    __threadfence_block();
    const uint32_t gen = atomic_load_shared(const_cast<uint32_t *>(&g_ts.sb_gen));
    if (atomicAdd(&g_ts.sb_count, 1u) == (uint32_t)n - 1u) {
        atomicExch(&g_ts.sb_count, 0u);
        __threadfence_block();
        atomicAdd(const_cast<uint32_t *>(&g_ts.sb_gen), 1u);
    } else {
        uint64_t polls = 0;
        while (atomic_load_shared(const_cast<uint32_t *>(&g_ts.sb_gen)) == gen) {
            if (spin_expired(polls, g_ts.rp.spin_limit, g_ts.rp.err)) break;
            __nanosleep(32);
        }
    }
    __threadfence_block();
}
template <class K> __device__ __forceinline__ void omp_barrier_full() {
    if constexpr (K::GENERIC_LIKE)
        asm volatile("barrier.sync 2, %0;" ::"n"(K::NT) : "memory");
    else
        cta_sync<K>();
}
template <class K> __device__ __forceinline__ void omp_barrier() {
    if constexpr (K::FOLD) {
        omp_barrier_full<K>();
    } else {
        if (tstate<K>().nested) return;
        const int n = g_ts.nthreads;
        if (n == K::NT) omp_barrier_full<K>();
        else if ((n & 31) == 0) asm volatile("barrier.sync 2, %0;" ::"r"(n) : "memory");
        else soft_barrier(n);
    }
}

// Team-wide sync of SPMD-ized sequential code (e.g. before a shared team
// variable read by all threads is overwritten); generic: no-op (only the main
// thread runs sequential code).
template <class K> __device__ __forceinline__ void spmd_sync() {
    if constexpr (K::MODE == SPMD) cta_sync<K>();
}

// ---------------------------------------------------------------- queries
template <class K> __device__ __forceinline__ int team_num() { return blockIdx.x; }
template <class K> __device__ __forceinline__ int num_teams() { return gridDim.x; }
template <class K> __device__ __forceinline__ int warp_size() { return 32; }
template <class K> __device__ __forceinline__ int warp_id() { return threadIdx.x >> 5; }

template <class K> __device__ __forceinline__ bool is_spmd() {
    if constexpr (K::FOLD) return K::MODE == SPMD;
    else return g_ts.exec_mode == SPMD;
}
// Folded queries assume the region context the analysis proved:
// thread/team-count queries are only folded inside parallel regions.
template <class K> __device__ __forceinline__ int parallel_level() {
    if constexpr (K::FOLD) return 1;
    else if constexpr (K::MODE == SPMD) return tstate<K>().level + tstate<K>().nested;
    else return (threadIdx.x == K::MAIN_HW ? 0 : g_ts.level) + tstate<K>().nested;
}
template <class K> __device__ __forceinline__ bool in_active_parallel() {
    return parallel_level<K>() == 1 && (K::FOLD || tstate<K>().nested == 0);
}
template <class K> __device__ __forceinline__ int thread_num() {
    if constexpr (K::FOLD) return threadIdx.x;
    else return (parallel_level<K>() == 0 || tstate<K>().nested) ? 0 : (int)threadIdx.x;
}
template <class K> __device__ __forceinline__ int num_threads() {
    if constexpr (K::FOLD) return K::NT;
    else return (parallel_level<K>() == 0 || tstate<K>().nested) ? 1 : g_ts.nthreads;
}

// Thread-management ICVs and queries of nested parallelism (OpenMP 5.1
// sec. 3.2).  Only the outermost region of a team is active:
// nested regions are serialized, so levels >= 2 have team size 1
// and thread number 0.  Folded variants assume what the analysis proved for
// them: inside a parallel region of NT threads, no nesting, no
// num_threads clause or omp_set_num_threads reaching the kernel.
template <class K> __device__ __forceinline__ int outer_level() {          // 0 or 1
    if constexpr (K::FOLD) return 1;
    else if constexpr (K::MODE == SPMD) return tstate<K>().level;
    else return threadIdx.x == K::MAIN_HW ? 0 : g_ts.level;
}
template <class K> __device__ __forceinline__ int active_level() {
    if constexpr (K::FOLD) return 1;
    else return (outer_level<K>() == 1 && g_ts.nthreads > 1) ? 1 : 0;
}
template <class K> __device__ __forceinline__ int max_threads() {          // omp_get_max_threads
    if constexpr (K::FOLD) return K::NT;
    else return min((int)g_ts.nvar, K::NT);
}
template <class K> __device__ __forceinline__ int ancestor_thread_num(int l) {
    const int lev = parallel_level<K>();
    if (l < 0 || l > lev) return -1;
    if (l == 0) return 0;
    if (l == 1) return (int)threadIdx.x;          // the outer (active) region
    return 0;                                     // serialized levels
}
template <class K> __device__ __forceinline__ int team_size(int l) {
    const int lev = parallel_level<K>();
    if (l < 0 || l > lev) return -1;
    if (l == 1) {
        if constexpr (K::FOLD) return K::NT;
        else return g_ts.nthreads;
    }
    return 1;                                     // initial team, serialized levels
}
// threads of the next region: the num_threads clause if given, else the
// nthreads-var ICV; at most the team's hardware threads
template <class K> __device__ __forceinline__ int region_threads(int clause) {
    const int n = clause > 0 ? clause : (int)g_ts.nvar;
    return n < K::NT ? n : K::NT;
}

// ---------------------------------------------------------------- roles
enum class Role { Main, Worker, Exit };

// team_init: every hardware thread calls it first.  Generic: lanes 1..31 of
// the main warp exit, workers must then call worker_loop, the main thread
// runs the team's sequential code.  SPMD: everybody is Main (runs the team
// code, guarded).
template <class K> __device__ __forceinline__ Role team_init(const RtParams &rp) {
    if constexpr (K::TSTATE) {
        ThreadState z = {0, 0, 0, 0};
        tstate<K>() = z;
    }
    if constexpr (K::PL == 4 /*PL_COALESCED*/) {
        CoalState c = {0, 0, 0, 0, 0, 0};
        cstate<K>() = c;
    }
    if constexpr ((K::FLAGS & F_BCAST_1BAR) != 0) bphase<K>() = 0;
    if constexpr (K::GENERIC_LIKE) {
        if ((int)threadIdx.x >= K::NT) {
            if ((int)threadIdx.x != K::MAIN_HW) return Role::Exit;
            g_ts.fn = nullptr;
            g_ts.args = nullptr;
            g_ts.region_id = 0;
            g_ts.level = 0;
            g_ts.nthreads = K::NT;
            g_ts.exec_mode = K::MODE;
            g_ts.nvar = K::NT;
            g_ts.sb_count = 0;
            g_ts.sb_gen = 0;
            g_ts.hwm_seen = 0;
            g_ts.rp = rp;
            return Role::Main;
        }
        return Role::Worker;
    } else {
        if (threadIdx.x == 0) {
            g_ts.level = 0;
            g_ts.nthreads = K::NT;
            g_ts.exec_mode = K::MODE;
            g_ts.nvar = K::NT;
            g_ts.sb_count = 0;
            g_ts.sb_gen = 0;
            g_ts.hwm_seen = 0;
            g_ts.rp = rp;
        }
        cta_sync<K>();
        return Role::Main;
    }
}

// ---------------------------------------------------------------- fork/join
// Region types: struct R { static constexpr int ID = ...; static __device__ void run(void*); }
// `num_threads_clause` > 0 is the region's num_threads clause (non-folded
// variants; threads beyond the region's team skip its body).
template <class K, class R> __device__ __forceinline__ void parallel(void *args, int num_threads_clause = 0) {
    if constexpr (!K::FOLD) {
        if (parallel_level<K>() > 0) {          // nested: serialize
            tstate<K>().nested++;
            R::run(args);
            tstate<K>().nested--;
            return;
        }
    }
    if constexpr (K::MODE == SPMD) {
        if constexpr (!K::FOLD) {
            // every thread computes the same team size; publishing a changed
            // one is a guarded side effect (its barriers only when it changes)
            const int n = region_threads<K>(num_threads_clause);
            if (n != g_ts.nthreads) {
                cta_sync<K>();
                if (threadIdx.x == 0) g_ts.nthreads = n;
                cta_sync<K>();
            }
            tstate<K>().level = 1;
            if ((int)threadIdx.x < n) R::run(args);   // in place
            tstate<K>().level = 0;
        } else {
            R::run(args);                        // in place, all threads
        }
        cta_sync<K>();                           // join
    } else {
        static_assert(K::GENERIC_LIKE, "parallel() needs a runtime mode");
        if constexpr (K::MODE == CSM)
            g_ts.region_id = R::ID;
        else
            g_ts.fn = &R::run;                   // address taken: GEN / CAS
        g_ts.args = args;
        g_ts.level = 1;
        if constexpr (!K::FOLD) g_ts.nthreads = region_threads<K>(num_threads_clause);
        team_barrier<K>();                       // fork
        team_barrier<K>();                       // join
        g_ts.level = 0;
    }
}

template <class K, class... Rs> struct Dispatch;
template <class K> struct Dispatch<K> {
    static __device__ __forceinline__ bool csm(int, void *) { return false; }
    static __device__ __forceinline__ bool cascade(RegionFn, void *) { return false; }
};
template <class K, class R, class... Rs> struct Dispatch<K, R, Rs...> {
    static __device__ __forceinline__ bool csm(int id, void *a) {
        if (id == R::ID) { R::run(a); return true; }
        return Dispatch<K, Rs...>::csm(id, a);
    }
    static __device__ __forceinline__ bool cascade(RegionFn fn, void *a) {
        if (fn == &R::run) { R::run(a); return true; }
        return Dispatch<K, Rs...>::cascade(fn, a);
    }
};

// The worker state machine.  Regions... are the parallel regions
// known to reach this kernel (used by CASCADE and CSM; GENERIC ignores them).
template <class K, class... Rs> __device__ void worker_loop() {
    for (;;) {
        team_barrier<K>();                       // wait for work
        void *a = g_ts.args;
        int id = 0;
        RegionFn fn = nullptr;
        if constexpr (K::MODE == CSM) {
            id = g_ts.region_id;
            if (id == 0) return;
        } else {
            fn = g_ts.fn;
            if (fn == nullptr) return;
        }
        // not in this region's team (num_threads clause / ICV): straight to the join
        const bool in_team = K::FOLD || (int)threadIdx.x < g_ts.nthreads;
        if (in_team) {
            if constexpr (K::MODE == CSM) {
                Dispatch<K, Rs...>::csm(id, a);  // direct calls, no fallback
            } else if constexpr (K::MODE == GENERIC_CASCADE) {
                if (!Dispatch<K, Rs...>::cascade(fn, a)) fn(a);   // indirect fallback
            } else {
                fn(a);                           // indirect call
            }
        }
        team_barrier<K>();                       // join
    }
}

template <class K> __device__ __forceinline__ void team_deinit() {
    if constexpr (K::GENERIC_LIKE) {             // main thread: release workers
        g_ts.fn = nullptr;
        g_ts.region_id = 0;
        team_barrier<K>();
    }
}

// ---------------------------------------------------------------- guards
// SPMD-ized sequential side effects.  Generic modes: only the
// main thread executes sequential code, so the guard is the identity.
template <class K, class F> __device__ __forceinline__ void guarded(F &&f) {
    if constexpr (K::MODE == SPMD) {
        if (threadIdx.x == 0) f();
        cta_sync<K>();
    } else {
        f();
    }
}
// A value produced in a guarded region, broadcast to all threads.  Default:
// slot write -> barrier -> read -> barrier (the paper's 2 barriers,
// P:687-688).  F_BCAST_1BAR: double-buffered slot, one barrier -- every
// call of the team alternates the slot (a per-thread phase; all threads make
// the same calls), so thread 0's write of slot b in call k+2 follows call
// k+1's barrier, which every reader of call k's slot b passed after reading
// (a caller-chosen phase let the runtime's own broadcasts, e.g. a TeamLocal
// pointer, reuse the slot a value was still being read from).  A one-warp
// team (thread_limit 32): lane 0 computes, __shfl_sync broadcasts from its
// registers -- no shared slot, no barrier.
template <class K, class T, class F> __device__ __forceinline__ T guarded_bcast(F &&f) {
    static_assert(sizeof(T) <= 8, "broadcast slot is 8 bytes");
    if constexpr (K::MODE == SPMD && K::BLOCK == 32 && GTR_WARP_TEAM) {
        uint64_t w = 0;
        if (threadIdx.x == 0) {
            const T v = f();
            memcpy(&w, &v, sizeof(T));
        }
        w = __shfl_sync(0xffffffffu, w, 0);
        T v;
        memcpy(&v, &w, sizeof(T));
        return v;
    } else if constexpr (K::MODE == SPMD) {
        int b = 0;
        if constexpr ((K::FLAGS & F_BCAST_1BAR) != 0) {
            b = (int)(bphase<K>() & 1u);
            bphase<K>() ^= 1u;
        }
        if (threadIdx.x == 0) *reinterpret_cast<T *>(&g_ts.bcast[b]) = f();
        cta_sync<K>();
        T v = *reinterpret_cast<volatile T *>(&g_ts.bcast[b]);
        if constexpr (!(K::FLAGS & F_BCAST_1BAR)) cta_sync<K>();
        return v;
    } else {
        return f();
    }
}

// omp_set_num_threads in the team's sequential code: a write of the team's
// nthreads-var ICV (a guarded side effect in SPMD mode).
template <class K> __device__ __forceinline__ void set_num_threads(int n) {
    guarded<K>([&] { g_ts.nvar = n > 0 ? n : 1; });
}

// ---------------------------------------------------------------- globalization
// __runtime_alloc / __runtime_free (Fig. 4c): per-thread LIFO stack in dynamic
// shared memory; when full, the thread's slab of the global fallback pool; when
// that is exhausted, ERR_HEAP and a per-CTA sink (results declared invalid).
__device__ __align__(16) static uint64_t g_sink_dummy;
// Fallback high-water mark: the global atomic only when this team has not
// yet reported that many bytes (a per-team shared-memory atomicMax filters:
// a few global atomics per team instead of one per allocation).
__device__ __forceinline__ void note_fallback(const RtParams &rp, uint32_t bytes) {
    if (atomicMax(const_cast<uint32_t *>(&g_ts.hwm_seen), bytes) < bytes)   // shared atomic: the team's filter
        atomicMax(rp.hwm, (unsigned long long)bytes);
}
template <class K> __device__ __noinline__ void *alloc_shared(uint32_t bytes) {
    const uint32_t words = (bytes + 7u) >> 3;
    ThreadState &ts = tstate<K>();
    const RtParams &rp = g_ts.rp;
    if constexpr (K::PL == PL_RUNTIME) {
        if ((uint32_t)ts.sp + words <= rp.sm_stack_words) {
            uint64_t *p = sm_stack_base<K>() + (size_t)threadIdx.x * rp.sm_stride_words + ts.sp;
            ts.sp = (uint16_t)(ts.sp + words);
            return p;
        }
    }
    if (rp.pool != nullptr && (uint64_t)ts.gsp + words <= rp.pool_wpt) {
        uint64_t *p = rp.pool + ((uint64_t)blockIdx.x * K::BLOCK + threadIdx.x) * rp.pool_wpt + ts.gsp;
        ts.gsp += words;
        note_fallback(rp, ts.gsp * 8u);          // fallback bytes in use
        return p;
    }
    atomicOr(rp.err, (uint32_t)ERR_HEAP);
    return &g_sink_dummy;
}
template <class K> __device__ __noinline__ void free_shared(void *p, uint32_t bytes) {
    const uint32_t words = (bytes + 7u) >> 3;
    ThreadState &ts = tstate<K>();
    if (p == &g_sink_dummy) return;
    if (__isShared(p)) {
        ts.sp = (uint16_t)(ts.sp - words);
        if ((uint64_t *)p != sm_stack_base<K>() + (size_t)threadIdx.x * g_ts.rp.sm_stride_words + ts.sp)
            atomicOr(g_ts.rp.err, (uint32_t)ERR_LIFO);
    } else {
        ts.gsp -= words;
    }
}

// __runtime_coalesced_alloc / _free (LLVM 12, Fig. 4b).  A converged warp
// (all 32 lanes in `mask`) allocates once on a warp stack: its 32 per-thread
// stack slices (overflow: the warp's slab of the first half of the fallback
// pool).  Each allocation is a frame with a count of live lanes; a lane's free
// decrements it, and the lane that releases a frame last pops every fully
// released frame from the top -- lanes that diverge after the allocation can
// release it at different times.  Calls from a partial warp (divergent lanes)
// allocate a per-lane copy from the second half of the pool (LIFO per lane).
// `words` is the whole allocation (already x32 for a converged parallel warp);
// `fk` returns the frame index (-1 for a per-lane copy).
template <class K> __device__ __forceinline__ CoalState *warp_states() {
    return reinterpret_cast<CoalState *>(g_dyn + coal_offset<K>()) + (threadIdx.x & ~31u);
}
template <class K> __device__ __noinline__ void *alloc_coalesced(uint32_t words, unsigned mask, int &fk) {
    const RtParams &rp = g_ts.rp;
    const uint64_t half = rp.pool_wpt / 2;
    if (mask != 0xffffffffu) {                            // divergent: per-lane copy
        CoalState &ts = cstate<K>();
        fk = -1;
        if (rp.pool != nullptr && (uint64_t)ts.igsp + words <= half) {
            uint64_t *p = rp.pool + (uint64_t)gridDim.x * K::BLOCK * half +
                          ((uint64_t)blockIdx.x * K::BLOCK + threadIdx.x) * half + ts.igsp;
            ts.igsp += words;
            note_fallback(rp, ts.igsp * 8u);
            return p;
        }
        atomicOr(rp.err, (uint32_t)ERR_HEAP);
        return &g_sink_dummy;
    }
    uint64_t *p = nullptr;
    int k = -1;
    // the converged warp meets here: each lane's accesses to frames it
    // released earlier are ordered before the frame is handed out again
    // (bar.warp.sync; the frame atomics alone do not order plain accesses)
    __syncwarp();
    if ((threadIdx.x & 31u) == 0) {
        CoalState *W = warp_states<K>();
        const uint32_t cap = min(32u * rp.sm_stride_words, 32767u);
        const uint32_t wbase = threadIdx.x & ~31u;
        // the warp stack is also popped by lanes releasing frames (possibly
        // diverged, interleaved with this allocation): atomics throughout
        k = (int)atomic_load_shared(&W[0].nframes);
        uint32_t glob = 0;
        const uint32_t wtop = atomic_load_shared(&W[0].wtop), wgtop = atomic_load_shared(&W[0].wgtop);
        if (k >= 32 || words > 32767u) {
            k = -1;
        } else if (wtop + words <= cap) {
            p = sm_stack_base<K>() + (size_t)wbase * rp.sm_stride_words + wtop;
            atomicAdd(&W[0].wtop, words);
        } else if (rp.pool != nullptr && (uint64_t)wgtop + words <= 32u * half) {
            p = rp.pool + ((uint64_t)blockIdx.x * K::BLOCK + wbase) * half + wgtop;
            atomicAdd(&W[0].wgtop, words);
            note_fallback(rp, (wgtop + words) * 8u / 32u);   // warp SoA: per lane
            glob = 0x8000u;
        } else {
            k = -1;
        }
        if (k < 0) {
            atomicOr(rp.err, (uint32_t)ERR_HEAP);
            p = &g_sink_dummy;
        } else {
            atomicExch(&W[k].frame, (32u << 16) | glob | words);
            __threadfence_block();
            atomicExch(&W[0].nframes, (uint32_t)k + 1u);
        }
    }
    fk = __shfl_sync(0xffffffffu, k, 0);
    return reinterpret_cast<void *>(__shfl_sync(0xffffffffu, reinterpret_cast<uintptr_t>(p), 0));
}
template <class K> __device__ __noinline__ void free_coalesced(void *p, uint32_t words, int fk) {
    if (p == &g_sink_dummy) return;
    if (fk < 0) {
        cstate<K>().igsp -= words;
        return;
    }
    CoalState *W = warp_states<K>();
    __threadfence_block();                                // this lane's uses happen before release
    const uint32_t old = atomicSub(&W[fk].frame, 1u << 16);
    if ((old >> 16) != 1u) return;                        // other lanes still use frame fk
    uint64_t polls = 0;
    for (;;) {                                            // pop fully released frames
        if (spin_expired(polls, g_ts.rp.spin_limit, g_ts.rp.err)) break;
        const uint32_t n = atomic_load_shared(&W[0].nframes);
        if (n == 0) break;
        const uint32_t f = atomic_load_shared(&W[n - 1].frame);
        if ((f >> 16) != 0u) break;
        if (atomicCAS(&W[0].nframes, n, n - 1) != n) continue;
        if (f & 0x8000u) atomicSub(&W[0].wgtop, f & 0x7fffu);
        else atomicSub(&W[0].wtop, f & 0x7fffu);
    }
    __threadfence_block();
}
// the runtime (never folded) queries LLVM 12's lowering evaluates
template <class K> __device__ __forceinline__ bool rt_is_spmd() { return g_ts.exec_mode == SPMD; }
template <class K> __device__ __forceinline__ bool rt_in_active_parallel() {
    const int lvl = (K::MODE == SPMD) ? tstate<K>().level
                                      : ((int)threadIdx.x == K::MAIN_HW ? 0 : g_ts.level);
    return lvl == 1 && tstate<K>().nested == 0;
}

template <int N_WORDS> struct OddStride {
    static constexpr int value = (N_WORDS % 2 == 1) ? N_WORDS : N_WORDS + 1;
};

// A per-thread globalized local of N elements of T (8-byte T for the
// interleaving arithmetic; other sizes round up to whole words).
template <class K, class T, int N, class Tag, int PL = K::PL> struct Local;

template <class K, class T, int N, class Tag> struct Local<K, T, N, Tag, PL_STACK> {
    T v[N];
    __device__ __forceinline__ T &operator[](int i) { return v[i]; }
    __device__ __forceinline__ T *ptr() { return v; }
};
template <class K, class T, int N, class Tag> struct Local<K, T, N, Tag, PL_RUNTIME> {
    T *p;
    __device__ __forceinline__ Local() { p = static_cast<T *>(alloc_shared<K>(N * sizeof(T))); }
    __device__ __forceinline__ ~Local() { free_shared<K>(p, N * sizeof(T)); }
    __device__ __forceinline__ T &operator[](int i) { return p[i]; }
    __device__ __forceinline__ T *ptr() { return p; }
};
template <class K, class T, int N, class Tag> struct Local<K, T, N, Tag, PL_GLOBAL>
    : Local<K, T, N, Tag, PL_RUNTIME> {};
template <class K, class T, int N, class Tag> struct Local<K, T, N, Tag, PL_COALESCED> {
    static constexpr uint32_t WORDS = (uint32_t)((N * sizeof(T) + 7) / 8);
    T v[N];
    T *p;
    uint32_t words;
    int fk;
    __device__ __forceinline__ Local() {
        if (rt_is_spmd<K>()) {                            // LLVM 12: no globalization in SPMD
            p = v;
            words = 0;
        } else {
            const unsigned mask = __activemask();
            const bool par = rt_in_active_parallel<K>() && mask == 0xffffffffu;   // SoA over the warp
            words = par ? 32u * WORDS : WORDS;
            uint64_t *base = static_cast<uint64_t *>(alloc_coalesced<K>(words, mask, fk));
            p = reinterpret_cast<T *>(par ? base + (threadIdx.x & 31u) * WORDS : base);
        }
    }
    __device__ __forceinline__ ~Local() {
        if (words) free_coalesced<K>(p, words, fk);
    }
    __device__ __forceinline__ T &operator[](int i) { return p[i]; }
    __device__ __forceinline__ T *ptr() { return p; }
};
template <class K, class T, int N, class Tag> struct Local<K, T, N, Tag, PL_SHARED_STATIC> {
    static constexpr int WORDS = (int)((N * sizeof(T) + 7) / 8);
    static constexpr int STRIDE = OddStride<WORDS>::value;
    T *p;
    __device__ __forceinline__ Local() {
        __shared__ uint64_t slots[K::BLOCK * STRIDE];     // one instance per Tag
        p = reinterpret_cast<T *>(&slots[threadIdx.x * STRIDE]);
    }
    __device__ __forceinline__ T &operator[](int i) { return p[i]; }
    __device__ __forceinline__ T *ptr() { return p; }
};

// A team-level globalized variable allocated by the main thread only and read
// by the team's threads inside parallel regions.
//   generic, RUNTIME/GLOBAL : main allocates on its stack; pointer passed
//   generic, SHARED_STATIC  : static __shared__ (heap-to-shared)
//   generic, STACK          : heap-to-stack is illegal (the pointer escapes to
//                             the workers) -> heap-to-shared, as h2s2 does
//   SPMD,    STACK          : every thread owns a copy (no escape once the
//                             region runs in place); writes need no guard
//   SPMD,    SHARED_STATIC  : one shared copy; writes guarded by thread 0
//   SPMD,    RUNTIME/GLOBAL : thread 0 allocates, pointer broadcast; writes
//                             guarded
//
// RO = the parallel regions only read it.  If they write it (the variable is
// shared between the team's threads, e.g. Fig. 1's team_val), SPMD + STACK
// cannot privatize it and uses static shared memory instead.
template <class K, class T, class Tag, bool RO = true> struct TeamLocal {
    static constexpr bool PRIVATE = (K::MODE == SPMD && K::PL == PL_STACK && RO);
    static constexpr bool RUNTIME_ALLOC = (K::PL == PL_RUNTIME || K::PL == PL_GLOBAL || K::PL == PL_COALESCED);
    // one copy, allocated in sequential context (coalesced: a single-lane
    // warp allocation, as LLVM 12 does outside parallel regions)
    // (coalesced: sequential context -> a single-lane call -> per-lane copy)
    __device__ __forceinline__ static T *alloc_one() {
        if constexpr (K::PL == PL_COALESCED) {
            int fk;
            return static_cast<T *>(alloc_coalesced<K>((uint32_t)((sizeof(T) + 7) / 8), 1u, fk));
        } else {
            return static_cast<T *>(alloc_shared<K>(sizeof(T)));
        }
    }
    __device__ __forceinline__ static void free_one(T *q) {
        if constexpr (K::PL == PL_COALESCED)
            free_coalesced<K>(q, (uint32_t)((sizeof(T) + 7) / 8), -1);
        else
            free_shared<K>(q, sizeof(T));
    }
    // PRIVATE: the copy itself, never a stored pointer to it -- a member
    // pointing into its own object keeps the whole object in local memory
    // (SROA cannot split it), and every store to that stack slot then has to
    // complete before the region's join barrier (measured: the SPMD
    // heap-to-stack fork/join loop ran 151 ns per empty region at
    // thread_limit 256, 3.5x the shared-memory form, all of it STL + BAR).
    T priv;
    T *p;
    __device__ __forceinline__ static T *static_slot() {
        __shared__ T s;
        return &s;
    }
    __device__ __forceinline__ TeamLocal() {
        if constexpr (PRIVATE) {
        } else if constexpr (RUNTIME_ALLOC) {
            if constexpr (K::MODE == SPMD)
                p = guarded_bcast<K, T *>([] { return alloc_one(); });
            else
                p = alloc_one();
        } else {
            p = static_slot();
        }
    }
    __device__ __forceinline__ ~TeamLocal() {
        if constexpr (RUNTIME_ALLOC) {
            if constexpr (K::MODE == SPMD) {
                cta_sync<K>();
                if (threadIdx.x == 0) free_one(p);
            } else {
                free_one(p);
            }
        }
    }
    // write by "the main thread": guarded in SPMD unless private
    template <class F> __device__ __forceinline__ void set(F &&f) {
        if constexpr (PRIVATE) f(priv);
        else if constexpr (K::MODE != SPMD) f(*p);
        else guarded<K>([&] { f(*p); });
    }
    __device__ __forceinline__ T *get() {
        if constexpr (PRIVATE) return &priv;
        else return p;
    }
};

// ---------------------------------------------------------------- worksharing
// `teams distribute dist_schedule(static, 1)` over [lo, hi): iteration c goes
// to team (c - lo) mod num_teams (Fig. 1's outer loop).  The body
// is the team's sequential code (it may fork parallel regions).
template <class K, class F> __device__ __forceinline__ void distribute_static(int64_t lo, int64_t hi, F &&body) {
    for (int64_t c = lo + team_num<K>(); c < hi; c += num_teams<K>()) body(c);
}

// `for` with a static schedule, chunk 1 (cyclic) -- AMB-2: coalesced.
template <class K, class F> __device__ __forceinline__ void for_static(int64_t lo, int64_t hi, F &&body) {
    const int64_t t = thread_num<K>(), n = num_threads<K>();
    for (int64_t i = lo + t; i < hi; i += n) body(i);
}

// `for schedule(static, chunk)`: chunk k goes to thread k mod num_threads.
template <class K, class F>
__device__ __forceinline__ void for_static_chunk(int64_t lo, int64_t hi, int64_t chunk, F &&body) {
    const int64_t t = thread_num<K>(), n = num_threads<K>();
    for (int64_t c = lo + t * chunk; c < hi; c += n * chunk)
        for (int64_t i = c; i < c + chunk && i < hi; i++) body(i);
}
// `for schedule(dynamic, chunk)`: threads claim chunks from a team counter
// (zeroed by the sequential code before the region).
template <class K, class F>
__device__ __forceinline__ void for_dynamic(int64_t lo, int64_t hi, int64_t chunk, unsigned long long *counter,
                                            F &&body) {
    for (;;) {
        const int64_t c = lo + (int64_t)atomicAdd(counter, (unsigned long long)chunk);
        if (c >= hi) break;
        for (int64_t i = c; i < c + chunk && i < hi; i++) body(i);
    }
}
// `for schedule(guided, chunk)`: chunk = max(chunk, remaining / (2 n)),
// claimed with compare-and-swap on a team counter (zeroed before the region).
template <class K, class F>
__device__ __forceinline__ void for_guided(int64_t lo, int64_t hi, int64_t chunk, unsigned long long *counter,
                                           F &&body) {
    const int64_t n = num_threads<K>();
    unsigned long long cur = *reinterpret_cast<volatile unsigned long long *>(counter);
    for (;;) {
        const int64_t c = lo + (int64_t)cur;
        if (c >= hi) break;
        int64_t sz = (hi - c) / (2 * n);
        if (sz < chunk) sz = chunk;
        const unsigned long long seen = atomicCAS(counter, cur, cur + (unsigned long long)sz);
        if (seen != cur) { cur = seen; continue; }
        for (int64_t i = c; i < c + sz && i < hi; i++) body(i);
        cur = *reinterpret_cast<volatile unsigned long long *>(counter);
    }
}

// `for schedule(dynamic, 32)`: warps claim 32 consecutive iterations at a
// time from a team counter ("dynamically chosen schedule"); the
// counter must be zeroed by the sequential code before the region.
template <class K, class F>
__device__ __forceinline__ void for_dynamic_warp(int64_t lo, int64_t hi, unsigned int *counter, F &&body) {
    const unsigned lane = threadIdx.x & 31u;
    for (;;) {
        unsigned base = 0;
        if (lane == 0) base = atomicAdd(counter, 32u);
        base = __shfl_sync(0xffffffffu, base, 0);
        const int64_t i = lo + (int64_t)base + lane;
        if (lo + (int64_t)base >= hi) break;
        if (i < hi) body(i);
        __syncwarp();
    }
}

// ---------------------------------------------------------------- reductions
// Team reduction of small integer tallies: shared-memory atomics per event,
// one global atomic per counter per team at the end.
__device__ __forceinline__ void tally_flush(const uint32_t *s, int n, unsigned long long *g, int tid, int nthr) {
    for (int k = tid; k < n; k += nthr)
        if (s[k]) atomicAdd(&g[k], (unsigned long long)s[k]);
}

}  // namespace gtr
