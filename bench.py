"""bench.py -- XSBench lookups/s per mode + fork/join ns, % of HBM roofline.

Metric (BASELINE.json): "XSBench lookups/s per mode + fork/join ns; % HBM
roofline at 1/2/4/8 B200".  Workload = config 5, XSBench large: 355 nuclides
x 11,303 gridpoints, 17M lookups per GPU (weak scaling), synthetic seeded
tables (gtr_inputs).  One step = one batch of 17M lookups through libgtr's
headline variant (SPMD-ized + heap-to-stack + folding, thread_limit 256 --
the paper's optimized form of XSBench's `target teams distribute parallel
for`) in XSBench's sorted event mode (sampling pass + sort by material and
grid-index bucket + warp-coherent lookups, all inside the step; `--schedule
bucketed` times the per-chunk bucketed schedule instead, which the line
reports beside the headline either way) plus, for N > 1, the combine of the
18 u64 hash/tallies: fused into the kernel's epilogue over peer memory
(dist.PeerCombine), checked once against an NCCL all-reduce after warm-up
(NCCL is used if they differ).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl gtr|reference] [--schedule sorted|bucketed]
    torchrun --nproc-per-node N bench.py --gpus N ...

Rank 0 prints one JSON line.  `--impl reference` times the oracle (plain C on
the host cores) on a bounded sample of the same workload instead.
"""
import argparse
import json
import os
import subprocess
import sys
import tempfile
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

N_ISO, N_GP, LOOKUPS_PER_GPU = 355, 11303, 17_000_000
METRIC = "XSBench lookups/s per mode + fork/join ns; % HBM roofline at 1/2/4/8 B200"
WORKLOAD = "XSBench large: 355 nuclides x 11,303 gridpoints, 17M lookups per GPU"
BYTES_PER_NUCLIDE = 100     # 4 B index-grid entry + 2 x 48 B gridpoints
FLOPS_PER_NUCLIDE = 28      # fp64 ops of one nuclide visit (c3.2), a division counted once


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=100)   # ~0.5 s timed: several clock samples
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="gtr", choices=["gtr", "reference"])
    ap.add_argument("--no-sweep", action="store_true", help="skip the per-mode / fork-join sweeps")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--schedule", default="sorted", choices=["sorted", "bucketed"],
                    help="headline schedule: XSBench's sorted event mode (sampling pass + sort by (material, "
                         "grid index) + warp-coherent lookups) or the per-chunk bucketed schedule")
    ap.add_argument("--combine", default="auto", choices=["auto", "fused", "nccl"],
                    help="N > 1: combine of the 18 u64 results -- fused into the lookup kernel's epilogue over "
                         "peer memory (auto: if every rank set it up and it matches NCCL once), or NCCL all_reduce")
    return ap.parse_args()


# ---------------------------------------------------------------- helpers
def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured"
    return 6650.0, "fallback"


class Clocks:
    """nvidia-smi sampler for the timed region (B200_PROFILING.md clocks line)."""
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu):
        self.gpu = gpu
        self.f = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)
        self.p = None

    def __enter__(self):
        try:
            self.p = subprocess.Popen(["nvidia-smi", "-i", str(self.gpu), f"--query-gpu={self.Q}",
                                       "--format=csv,noheader,nounits", "-lms", "100"],
                                      stdout=self.f, stderr=subprocess.DEVNULL)
        except OSError:
            self.p = None
        time.sleep(0.3)
        return self

    def __exit__(self, *a):
        if self.p:
            self.p.terminate()
            self.p.wait()

    def summary(self):
        self.f.flush()
        rows = [l.split(", ") for l in open(self.f.name).read().strip().splitlines() if l.count(",") >= 8]
        if not rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unavailable"], "samples": 0}
        sm = np.array([float(r[1]) for r in rows])
        smax = float(rows[0][2])
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[k] for r in rows for k in range(4) if r[5 + k].strip() == "Active"})
        load = sm[sm >= 0.5 * sm.max()] if sm.max() > 0 else sm
        return {"sm_mhz": float(np.median(load)), "sm_max_mhz": smax, "reasons": reasons,
                "samples": len(rows)}


def dist_init():
    import torch
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if ws > 1 or os.environ.get("GTR_BENCH_DIST") == "1":   # GTR_BENCH_DIST: exercise the N>1 path on 1 GPU
        import torch.distributed as dist
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        os.environ.setdefault("MASTER_PORT", "29517")
        os.environ.setdefault("RANK", "0")
        os.environ.setdefault("WORLD_SIZE", str(ws))
        torch.cuda.set_device(local)
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    else:
        torch.cuda.set_device(0)
    return ws, rank, local


def cpu_baseline(tables, first, n, seed):
    """The oracle as it stands, on the host cores, bounded sample."""
    import oracle
    P = oracle.XsProblem(tables)
    cores = os.cpu_count() or 1
    t0 = time.perf_counter()
    out, _ = P.run(first, n, seed, cores)
    dt = time.perf_counter() - t0
    return {"value": n / dt, "unit": "lookups/s", "cores": cores, "kind": "oracle",
            "sample": f"lookups [{first}, {first + n}) of rank 0's range (of {LOOKUPS_PER_GPU}), "
                      f"{cores} pthreads, table build excluded",
            "seconds": dt}, out


def host_info():
    """nproc and the CPU model (lscpu) of the box the oracle baselines ran on."""
    model = None
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        for l in out.splitlines():
            if l.startswith("Model name:"):
                model = l.split(":", 1)[1].strip()
    except (OSError, subprocess.TimeoutExpired):
        pass
    if model is None and os.path.exists("/proc/cpuinfo"):
        for l in open("/proc/cpuinfo"):
            if l.startswith("model name"):
                model = l.split(":", 1)[1].strip()
                break
    return {"nproc": os.cpu_count(), "cpu_model": model}


def oracle_fj(nt, R=20000):
    """Config 2 beside the GPU: the oracle's host team (main + min(thread_limit,
    nproc) pthreads, pthread_barrier fork and join), ns per fork/join."""
    import oracle
    T = max(1, min(nt, os.cpu_count() or 1))
    res = {"threads": T, "regions": R}
    for tag, body, K in (("empty", 0, 1), ("trivial_k4", 1, 4)):
        r, ns = oracle.fj_host_team(T, R, body, K)
        assert r == oracle.fj_team(0, T, R, body, K)
        res[f"{tag}_ns"] = ns
    return res


def oracle_su3(sites=32 ** 4, reps=3):
    """Config 3 beside the GPU: the oracle on nproc threads over the 32^4
    lattice (constant inputs), best of `reps`, ms per iteration."""
    import gtr_inputs.su3 as S
    import oracle
    A, B = S.make_lattice(sites, "constant")
    cores = os.cpu_count() or 1
    best = None
    for _ in range(reps):
        t0 = time.perf_counter()
        Cm = oracle.su3_mat_nn(A, B, cores)
        dt = time.perf_counter() - t0
        best = dt if best is None else min(best, dt)
    ok = bool(np.all(Cm.real == 1.0) and np.all(Cm.imag == 0.0))
    return {"ms_per_iter": best * 1e3, "gb_s": sites * 1152 / best / 1e9, "cores": cores, "kind": "oracle",
            "closed_form_ok": ok, "sample": f"full 32^4 lattice, {cores} pthreads, best of {reps}"}


def oracle_rs(n=100_000):
    """Config 4 beside the GPU: the oracle on nproc threads over a bounded
    sample of the 10M-lookup workload (lookups [0, n)), lookups/s."""
    import gtr_inputs.rs as RS
    import gtr_inputs.xs as X
    import oracle
    P = oracle.RsProblem(RS.make_tables())
    cores = os.cpu_count() or 1
    t0 = time.perf_counter()
    out, _, _ = P.run(0, n, X.SEED_L, cores)
    dt = time.perf_counter() - t0
    return {"lookups_per_s": n / dt, "cores": cores, "kind": "oracle",
            "sample": f"lookups [0, {n}) of the 10M workload, {cores} pthreads, table build excluded"}, out


def xs_small_config(G, torch, ctx, stream):
    """Config 1 (XS small: 68 nuclides x 11,303, 1e5 lookups): the GPU's SPMD
    and NATIVE lookups/s beside the oracle's full run on 1 core and on nproc
    threads (table build excluded), results compared."""
    import gtr_inputs.xs as X
    import oracle
    from paper_conf_cgo_hubercgtddcd22_b200.problems import XsDevice
    t = X.make_tables(68, N_GP)
    n = 100_000
    xs = XsDevice(ctx, t)
    out = torch.zeros(18, dtype=torch.uint64, device="cuda")
    res = {"workload": "XSBench small: 68 nuclides x 11,303 gridpoints, 100,000 lookups"}
    P = oracle.XsProblem(t)
    cores = os.cpu_count() or 1
    t0 = time.perf_counter()
    o1, _ = P.run(0, n, X.SEED_L, 1)
    d1 = time.perf_counter() - t0
    t0 = time.perf_counter()
    P.run(0, n, X.SEED_L, cores)
    dn = time.perf_counter() - t0
    for name, c in (("spmd", G.cfg(G.SPMD, G.PL_STACK, 1, 256)), ("native_plain", G.cfg(G.NATIVE, G.PL_STACK, 1, 256)),
                    ("csm", G.cfg(G.CSM, G.PL_STACK, 1, 256)), ("generic", G.cfg(G.GENERIC, G.PL_STACK, 1, 256))):
        def f():
            out.zero_()
            G.gtr_xs_lookup(ctx, c, xs.tables, 0, n, X.SEED_L, out, None, stream)
        ms = _time(torch, stream, f, 5)
        res[name] = {"lookups_per_s": n / (ms * 1e-3), "ms": ms,
                     "same_result_as_oracle": bool(np.array_equal(out.cpu().numpy(), o1))}
    # the sorted event mode at this size (sort + presorted lookups in one call)
    ws = torch.empty(G.gtr_xs_sorted_workspace_bytes(n), dtype=torch.uint8, device="cuda")
    c = G.cfg(G.SPMD, G.PL_STACK, 1, 256)

    def fs():
        out.zero_()
        G.gtr_xs_lookup_sorted(ctx, c, xs.tables, 0, n, X.SEED_L, out, ws, None, stream)
    ms = _time(torch, stream, fs, 5)
    res["spmd_sorted"] = {"lookups_per_s": n / (ms * 1e-3), "ms": ms,
                          "same_result_as_oracle": bool(np.array_equal(out.cpu().numpy(), o1))}
    del ws
    res["cpu_oracle_1core"] = {"lookups_per_s": n / d1, "cores": 1, "kind": "oracle", "sample": "full run"}
    res["cpu_oracle_nproc"] = {"lookups_per_s": n / dn, "cores": cores, "kind": "oracle", "sample": "full run"}
    del xs
    torch.cuda.empty_cache()
    return res


# ---------------------------------------------------------------- reference arm
def run_reference(a):
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    import gtr_inputs.xs as X
    import oracle
    t = X.make_tables(N_ISO, N_GP)
    P = oracle.XsProblem(t)
    cores = os.cpu_count() or 1
    sample = 400_000
    for w in range(a.warmup):
        P.run(w * sample, sample, X.SEED_L, cores)
    t0 = time.perf_counter()
    for s in range(a.steps):
        P.run(s * sample, sample, X.SEED_L, cores)
    dt = (time.perf_counter() - t0) / a.steps
    v = sample / dt
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": "lookups/s", "n_gpus": a.gpus,
            "steps": a.steps, "warmup": a.warmup, "ms_per_step": dt * 1e3, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": WORKLOAD, "variant": "C oracle (oracle/xs.c), -O2 -ffp-contract=off",
                       "sample_per_step": sample},
            "cpu_baseline": {"value": v, "unit": "lookups/s", "cores": cores, "kind": "oracle",
                             "sample": f"{sample} lookups per step of the 17M-lookup workload, {cores} pthreads"},
            "e2e": {"value": v, "unit": "lookups/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ---------------------------------------------------------------- gtr arm
def run_gtr(a):
    import torch
    import gtr_inputs.xs as X
    from paper_conf_cgo_hubercgtddcd22_b200 import gtr as G
    from paper_conf_cgo_hubercgtddcd22_b200.problems import XsDevice

    ws, rank, local = dist_init()
    dist = None
    import torch.distributed as _d
    if _d.is_initialized():
        dist = _d
    dev = torch.device("cuda", local)
    stream = torch.cuda.current_stream()
    pool = torch.zeros(64 << 20, dtype=torch.uint8, device=dev)
    ctx = G.gtr_ctx_create(local, pool.data_ptr(), pool.numel())

    t_setup = time.perf_counter()
    tables = X.make_tables(N_ISO, N_GP)
    xs = XsDevice(ctx, tables, device=dev)
    torch.cuda.synchronize()
    t_setup = time.perf_counter() - t_setup
    from paper_conf_cgo_hubercgtddcd22_b200.dist import shard_range, combine_results, max_over_ranks
    first, n = shard_range(rank, ws, LOOKUPS_PER_GPU)
    seed = X.SEED_L
    head = G.cfg(G.SPMD, G.PL_STACK, 1, 256)
    out = torch.zeros(18, dtype=torch.uint64, device=dev)
    num_nucs = tables["num_nucs"].astype(np.int64)
    sorted_ = a.schedule == "sorted"
    wsp = torch.empty(G.gtr_xs_sorted_workspace_bytes(n), dtype=torch.uint8, device=dev) if sorted_ else None

    def launch(ptrs, kev=None):
        """One step's launches: (sort, then) the lookups into `out` or, with
        peer pointers, into every rank's buffer (fused combine)."""
        if kev is not None:
            kev[0].record(stream)
        if sorted_:
            G.gtr_xs_sort_lookups(ctx, xs.tables, first, n, seed, wsp, stream)
        if kev is not None:
            kev[1].record(stream)
        if sorted_ and ptrs is not None:
            G.gtr_xs_lookup_presorted_peers(ctx, head, xs.tables, first, n, ptrs, wsp, stream)
        elif sorted_:
            G.gtr_xs_lookup_presorted(ctx, head, xs.tables, first, n, out, wsp, None, stream)
        elif ptrs is not None:
            G.gtr_xs_lookup_peers(ctx, head, xs.tables, first, n, seed, ptrs, stream)
        else:
            G.gtr_xs_lookup(ctx, head, xs.tables, first, n, seed, out, None, stream)
        if kev is not None:
            kev[2].record(stream)

    # N > 1: the 18-u64 combine is fused into the lookup kernel's epilogue
    # (teams add into every rank's buffer over NVLink peer memory, then one
    # device barrier with a timeout; dist.PeerCombine) when every rank could
    # set it up and its first result equals an NCCL all_reduce; otherwise --
    # or with --combine nccl -- NCCL all_reduce.  All ranks decide together.
    pc, combine, combine_check, nranks = None, "none (1 GPU)", None, ws
    if dist is not None:
        from paper_conf_cgo_hubercgtddcd22_b200.dist import PeerCombine
        pc, why = PeerCombine.create_all_or_none(dev, want=a.combine in ("auto", "fused"))
        if pc is not None:
            nranks = pc.nranks
            combine = "fused: team epilogue adds into every rank's buffer over NVLink peer memory + device barrier"
        else:
            combine = f"nccl: all_reduce(SUM) of 18 u64 ({why})" if a.combine != "nccl" else \
                "nccl: all_reduce(SUM) of 18 u64 (--combine nccl)"

    def step():
        nonlocal out
        if pc is not None:
            launch(pc.ptrs())
            out = pc.finish()
            return
        out.zero_()
        launch(None)
        if dist is not None:
            combine_results(out)

    for _ in range(a.warmup):
        step()
    G.gtr_ctx_check(ctx, stream)
    if dist is not None:
        # both combines on the same step, compared (also at N = 1 with
        # GTR_BENCH_DIST=1): the fused result against the NCCL all-reduce of
        # this rank's own lookups; all ranks switch to NCCL together if any differs
        loc = torch.zeros(18, dtype=torch.uint64, device=dev)
        if sorted_:
            G.gtr_xs_lookup_sorted(ctx, head, xs.tables, first, n, seed, loc, wsp, None, stream)
        else:
            G.gtr_xs_lookup(ctx, head, xs.tables, first, n, seed, loc, None, stream)
        combine_results(loc)
        nccl_res = loc.cpu().numpy()
        fused_res = out.cpu().numpy() if pc is not None else None
        same = fused_res is None or bool(np.array_equal(fused_res, nccl_res))
        ok = torch.tensor([1 if same else 0], dtype=torch.int64, device=dev)
        dist.all_reduce(ok, op=dist.ReduceOp.MIN)
        combine_check = {"nccl_hash": int(nccl_res[0]),
                         "fused_hash": int(fused_res[0]) if fused_res is not None else None,
                         "identical_all_ranks": bool(int(ok[0]) == 1) if fused_res is not None else None}
        if pc is not None and int(ok[0]) != 1:
            pc = None
            combine = "nccl: all_reduce(SUM) of 18 u64 (the fused peer-memory combine differed from NCCL)"
            step()

    # timed region: K steps, barrier + sync on both sides, CUDA events on the
    # launching stream; per-launch kernel events for the roofline
    kev = [tuple(torch.cuda.Event(enable_timing=True) for _ in range(3)) for _ in range(a.steps)]
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with Clocks(local) as clk:
        if dist is not None:
            dist.barrier()
        torch.cuda.synchronize()
        e0.record(stream)
        for s in range(a.steps):
            if pc is not None:
                launch(pc.ptrs(), kev[s])
                out = pc.finish()
                continue
            out.zero_()
            launch(None, kev[s])
            if dist is not None:
                combine_results(out)
        e1.record(stream)
        torch.cuda.synchronize()
        if dist is not None:
            dist.barrier()
    G.gtr_ctx_check(ctx, stream)
    ms = e0.elapsed_time(e1) / a.steps
    k_ms = float(np.mean([b.elapsed_time(c) for _, b, c in kev]))        # the lookup kernel
    sort_ms = float(np.mean([a0.elapsed_time(b) for a0, b, _ in kev]))   # sampling pass + sort
    res = out.cpu().numpy().astype(np.uint64)
    t_ms = torch.tensor([ms, k_ms, sort_ms], dtype=torch.float64, device=dev)
    if dist is not None:
        max_over_ranks(t_ms)
    ms, k_ms, sort_ms = float(t_ms[0]), float(t_ms[1]), float(t_ms[2])
    value = ws * n / (ms * 1e-3)

    # algorithmic work of one step (this rank): the material tallies of all
    # ranks are in `res`; per nuclide visit 100 B and 28 fp64
    # flops (c3.2: f = (hi.e - E) / (hi.e - lo.e) 3, five channels x 3, five
    # x (mul, add) into macro; a division counted as one flop)
    mat_tally = res[1:13].astype(np.int64)
    visits = float((mat_tally * num_nucs).sum()) / ws
    alg_bytes = visits * BYTES_PER_NUCLIDE
    hbm, peak_kind = peaks()
    import glob

    def ncu_traffic(pattern, kname):
        """dram read+write bytes per launch of `kname` from the latest `ncu --set full` capture"""
        profs = sorted(glob.glob(os.path.join(ROOT, "profiles", pattern)))
        if profs:
            ks = [k for k in json.load(open(profs[-1]))["kernels"] if kname in k["kernel"]]
            if ks:
                return ks[0]["dram_bytes_per_launch"], os.path.relpath(profs[-1], ROOT)
        return None, None
    hbm_src = f"{peak_kind} MEASURED_PEAKS.json hbm_gbs" if peak_kind == "measured" \
        else "fallback B200_PROFILING.md 6.65 TB/s"
    if sorted_:
        # the sorted lookups share each gridpoint pair across a warp: DRAM
        # traffic is a few GB per launch, far below the 100 B per visit the
        # gather model counts, and the kernel's busiest unit is the fp64 pipe
        fp64 = fp64_peak(G, torch, ctx, stream)
        fp64_src = ("measured: gtr_fp64_probe (independent DFMA chains, 2 flops each); nominal 148 SM x 64 fp64 "
                    "lanes x 2 x 1.965 GHz = 37.2 TFLOP/s")
        flops = visits * FLOPS_PER_NUCLIDE
        achieved = flops / (k_ms * 1e-3) / 1e12
        traffic, traffic_src = ncu_traffic("r*_xs_sorted_ncu.json", "kernel_rt_sorted<Cfg<3, 3, 1, 256")
        pipes = None           # hardware utilisation of the same kernel from the committed capture
        profs = sorted(glob.glob(os.path.join(ROOT, "profiles", "r*_xs_sorted_ncu.json")))
        if profs:
            ks = [k for k in json.load(open(profs[-1]))["kernels"] if "kernel_rt_sorted<Cfg<3, 3, 1, 256" in k["kernel"]]
            if ks:
                pipes = {"fp64_pipe_active_pct": ks[0].get("sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active"),
                         "issue_active_pct": ks[0].get("smsp__issue_active.avg.pct_of_peak_sustained_active"),
                         "warp_instructions": ks[0].get("smsp__inst_executed.sum"),
                         "source": os.path.relpath(profs[-1], ROOT)}
        roofline = {"bound": "alu", "achieved": achieved, "peak": fp64, "unit": "TFLOP/s",
                    "frac": achieved / fp64, "traffic": traffic, "traffic_source": traffic_src,
                    "kernel": "kernel_rt_sorted<SPMD, heap-to-stack, fold, 256> (the lookups in sorted order)",
                    "kernel_ms": k_ms, "sort_ms": sort_ms, "alg_flops_per_launch": flops, "ncu": pipes,
                    "peak_source": fp64_src,
                    "gather_model": {"alg_bytes_per_launch": alg_bytes, "unit": "GB/s",
                                     "achieved_kernel": alg_bytes / (k_ms * 1e-3) / 1e9,
                                     "achieved_step": alg_bytes / (ms * 1e-3) / 1e9, "hbm_peak": hbm,
                                     "note": "SURVEY 8(d)'s 100 B per nuclide visit over the lookup kernel / "
                                             "the whole step (sort included): above the HBM peak because a warp "
                                             "reads each shared gridpoint pair once, not once per lookup"}}
    else:
        achieved = alg_bytes / (k_ms * 1e-3) / 1e9
        traffic, traffic_src = ncu_traffic("r*_xs_headline_ncu.json", "Cfg<3, 3, 1, 256")
        roofline = {"bound": "hbm", "achieved": achieved, "peak": hbm, "unit": "GB/s",
                    "frac": achieved / hbm, "traffic": traffic, "traffic_source": traffic_src,
                    "kernel_ms": k_ms, "alg_bytes_per_launch": alg_bytes, "peak_source": hbm_src}

    extra = {}
    if not a.no_sweep:      # 180 GB HBM: the XS tables stay resident
        extra["sharded"] = sharded_apps(G, torch, ctx, rank, ws, dist, stream, dev)
    if rank == 0:
        # the other schedule of the same step, outside the timed region: the
        # bucketed kernel's HBM roofline (the gather model of SURVEY 8(d))
        if sorted_:
            def fb():
                out.zero_()
                G.gtr_xs_lookup(ctx, head, xs.tables, first, n, seed, out, None, stream)
            bms = _time(torch, stream, fb, 5)
            btr, bsrc = ncu_traffic("r*_xs_headline_ncu.json", "Cfg<3, 3, 1, 256")
            extra["bucketed_schedule"] = {
                "lookups_per_s": n / (bms * 1e-3), "ms": bms, "same_result": bool(np.array_equal(out.cpu().numpy(), res))
                if ws == 1 else None,
                "roofline": {"bound": "hbm", "achieved": alg_bytes / (bms * 1e-3) / 1e9, "peak": hbm, "unit": "GB/s",
                             "frac": alg_bytes / (bms * 1e-3) / 1e9 / hbm, "traffic": btr, "traffic_source": bsrc,
                             "peak_source": hbm_src}}
    if rank == 0 and not a.no_sweep:
        extra.update(sweeps(G, torch, ctx, xs, first, seed, stream, cpu=(ws == 1 and not a.no_cpu_baseline)))

    # e2e through the public host-buffer entry point (H2D request, D2H results)
    h_out = torch.zeros(18, dtype=torch.uint64).pin_memory()
    req = G.gtr_xs_request(first, n, seed)

    def e2e_call():
        if sorted_:
            G.gtr_xs_lookup_sorted_host(ctx, head, xs.tables, req, h_out, wsp, stream)
        else:
            G.gtr_xs_lookup_host(ctx, head, xs.tables, req, h_out, stream)
    e2e_call()
    if dist is not None:
        dist.barrier()
    t0 = time.perf_counter()
    for _ in range(a.steps):
        e2e_call()
    e2e_s = (time.perf_counter() - t0) / a.steps
    t_e = torch.tensor([e2e_s], dtype=torch.float64, device=dev)
    if dist is not None:
        max_over_ranks(t_e)
    e2e_s = float(t_e[0])

    cpu = None
    parity = None
    if rank == 0 and ws == 1 and not a.no_cpu_baseline:
        m = 2_000_000
        cpu, o_out = cpu_baseline(tables, first, m, seed)
        chk = torch.zeros(18, dtype=torch.uint64, device=dev)
        if sorted_:
            G.gtr_xs_lookup_sorted(ctx, head, xs.tables, first, m, seed, chk, wsp, None, stream)
        else:
            G.gtr_xs_lookup(ctx, head, xs.tables, first, m, seed, chk, None, stream)
        parity = bool(np.array_equal(chk.cpu().numpy(), o_out))
        cpu.pop("seconds")

    if rank == 0:
        variant = ("SPMD + heap-to-stack + folding, thread_limit 256; sorted event mode: sampling pass + sort by "
                   "(material, grid index) + warp-coherent lookups, all inside the timed step") if sorted_ else \
            "SPMD + heap-to-stack + folding, thread_limit 256; per-chunk (material, energy) bucketed schedule"
        line = {
            "metric": METRIC, "value": value, "unit": "lookups/s", "n_gpus": ws, "steps": a.steps,
            "warmup": a.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": WORKLOAD, "variant": variant, "schedule": a.schedule,
                       "lookups_per_gpu": n, "parallelism": f"dp{ws}: lookups sharded over {ws} GPU(s)",
                       "combine": combine, "nranks": nranks, "combine_check": combine_check,
                       "l2": "no flush: inputs 5.9 GB per GPU >> 126 MB L2 (index grid 5.7 GB)",
                       "table_setup_s": round(t_setup, 2)},
            "hash": int(res[0]), "hash_mod_999983": int(res[0] % 999983),
            "roofline": roofline,
            "cpu_baseline": cpu, "parity_vs_oracle_2M_sample": parity,
            "e2e": {"value": ws * n / e2e_s, "unit": "lookups/s",
                    "h2d_bytes_per_step": 24, "d2h_bytes_per_step": 144,
                    "note": ("gtr_xs_lookup_sorted_host" if sorted_ else "gtr_xs_lookup_host") +
                            ": pinned host request -> device, lookups, 18 u64 -> pinned host, "
                            "stream sync; tables resident (uploaded once, table_setup_s)"},
            # our kernels per step: sampling, 2 scan, scatter, lookups (sorted; a GTR_XS_SORT_RANK=1 build
            # adds the rank pass); the lookups (bucketed)
            "gpu_launches": a.steps * (5 if sorted_ else 1),
            "clocks": clk.summary(),
            "host": host_info(),
        }
        line.update(extra)
        print(json.dumps(line), flush=True)
    G.gtr_ctx_destroy(ctx)
    if dist is not None:
        dist.destroy_process_group()


def _time(torch, stream, fn, reps):
    fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(stream)
    for _ in range(reps):
        fn()
    b.record(stream)
    torch.cuda.synchronize()
    return a.elapsed_time(b) / reps


def sweeps(G, torch, ctx, xs, first, seed, stream, cpu=True):
    """Per-mode lookups/s (same 17M lookups), the paper's variant ladder, and
    fork/join ns per mode -- each checked for identical results.  With `cpu`,
    the oracle timed on the host cores beside every config (BASELINE.md
    CPU-baseline plan)."""
    n = LOOKUPS_PER_GPU
    out = torch.zeros(18, dtype=torch.uint64, device="cuda")
    modes = {}
    ref = None
    variants = []
    for sched, tag in ((0, ""), (G.F_PLAIN, "_plain")):
        for name, m in (("spmd", G.SPMD), ("csm", G.CSM), ("cascade", G.GENERIC_CASCADE),
                        ("generic", G.GENERIC)):
            variants.append((name + tag, G.cfg(m, G.PL_STACK, 1, 256, flags=sched)))
            if not tag:     # generic modes run thread_limit + 32 threads: 128 fits more teams/SM
                variants.append((name + "_t128", G.cfg(m, G.PL_STACK, 1, 128, flags=sched)))
    variants.insert(0, ("native_plain", G.cfg(G.NATIVE, G.PL_STACK, 1, 256)))
    # the CUDA watermark of the bucketed schedule (plain CUDA, no runtime)
    variants.insert(1, ("native_bucketed", G.cfg(G.NATIVE, G.PL_STACK, 1, 256, flags=G.F_NATIVE_BUCKETED)))
    for name, c in variants:
        def f():
            out.zero_()
            G.gtr_xs_lookup(ctx, c, xs.tables, first, n, seed, out, None, stream)
        ms = _time(torch, stream, f, 3)
        r = out.cpu().numpy()
        ref = r if ref is None else ref
        info = G.gtr_query_variant(G.K_XS, c)
        modes[name] = {"lookups_per_s": n / (ms * 1e-3), "ms": ms, "regs": info["regs"],
                       "static_smem": info["static_smem"], "dyn_smem": info["dyn_smem"],
                       "teams_per_sm": info["teams_per_sm"], "same_result": bool(np.array_equal(r, ref))}
    # the paper's "OpenMP as a fraction of CUDA" (its V100: XS 71%,
    # RS 98%): each runtime mode against the CUDA kernel of the same schedule
    rate = {k: v["lookups_per_s"] for k, v in modes.items()}
    modes["fraction_of_cuda"] = {
        "bucketed_schedule": {m: rate[m] / rate["native_bucketed"] for m in ("spmd", "csm", "cascade", "generic")},
        "paper_plain_schedule": {m: rate[m + "_plain"] / rate["native_plain"]
                                 for m in ("spmd", "csm", "cascade", "generic")},
        "paper_v100": {"xsbench_llvm_dev_vs_cuda": 0.71}}
    # XSBench's other acceleration structures, same lookups
    grids = {}
    import gtr_inputs.xs as X
    from paper_conf_cgo_hubercgtddcd22_b200.problems import XsDevice
    tables = X.make_tables(N_ISO, N_GP)
    for gname, gt in (("nuclide_grid", G.XS_NUCLIDE), ("hash_grid", G.XS_HASH)):
        xg = XsDevice(ctx, tables, grid_type=gt, hash_bins=10000)
        for mname, c in (("spmd", G.cfg(G.SPMD, G.PL_STACK, 1, 256)),
                         ("native_plain", G.cfg(G.NATIVE, G.PL_STACK, 1, 256))):
            def f():
                out.zero_()
                G.gtr_xs_lookup(ctx, c, xg.tables, first, n, seed, out, None, stream)
            ms = _time(torch, stream, f, 2)
            grids[f"{gname}_{mname}"] = {"lookups_per_s": n / (ms * 1e-3), "ms": ms,
                                         "table_bytes": xg.nbytes(),
                                         "same_result": bool(np.array_equal(out.cpu().numpy(), ref))}
        del xg
    grids["unionized_spmd"] = {"lookups_per_s": modes["spmd"]["lookups_per_s"], "table_bytes": xs.nbytes()}
    # XSBench's history-based mode and sorted event-based variant (SURVEY NEXT
    # f2): same lookups, same results; the sorted step includes its sampling
    # pass and counting sort
    f2 = {}
    ws = torch.empty(G.gtr_xs_sorted_workspace_bytes(n), dtype=torch.uint8, device="cuda")
    for name, c, sorted_ in [("spmd_history", G.cfg(G.SPMD, G.PL_STACK, 1, 256, flags=G.F_HISTORY), False),
                             ("native_history", G.cfg(G.NATIVE, G.PL_STACK, 1, 256, flags=G.F_HISTORY), False),
                             ("spmd_sorted", G.cfg(G.SPMD, G.PL_STACK, 1, 256), True),
                             ("csm_sorted", G.cfg(G.CSM, G.PL_STACK, 1, 256), True),
                             ("cascade_sorted", G.cfg(G.GENERIC_CASCADE, G.PL_STACK, 1, 256), True),
                             ("generic_sorted", G.cfg(G.GENERIC, G.PL_STACK, 1, 256), True),
                             ("native_sorted", G.cfg(G.NATIVE, G.PL_STACK, 1, 256), True),
                             # the CUDA watermark of the sorted schedule: the same warp-coherent
                             # loops as a plain CUDA kernel (no runtime)
                             ("native_coherent_sorted",
                              G.cfg(G.NATIVE, G.PL_STACK, 1, 256, flags=G.F_NATIVE_BUCKETED), True)]:
        def f():
            out.zero_()
            if sorted_:
                G.gtr_xs_lookup_sorted(ctx, c, xs.tables, first, n, seed, out, ws, None, stream)
            else:
                G.gtr_xs_lookup(ctx, c, xs.tables, first, n, seed, out, None, stream)
        ms = _time(torch, stream, f, 3)
        f2[name] = {"lookups_per_s": n / (ms * 1e-3), "ms": ms,
                    "same_result": bool(np.array_equal(out.cpu().numpy(), ref))}
    del ws
    f2["fraction_of_cuda_sorted"] = {m: f2[m + "_sorted"]["lookups_per_s"] / f2["native_coherent_sorted"]["lookups_per_s"]
                                     for m in ("spmd", "csm", "cascade", "generic")}
    # the paper's ladder (Fig. 11a) on SPMD: globalized at runtime -> h2s2 -> +fold
    ladder = {}
    for name, c in [("llvm12_coalesced", G.cfg(G.SPMD, G.PL_COALESCED, 0, 256)),
                    ("runtime_globalized", G.cfg(G.SPMD, G.PL_RUNTIME, 0, 256)),
                    ("global_heap", G.cfg(G.SPMD, G.PL_GLOBAL, 0, 256)),
                    ("heap_to_shared", G.cfg(G.SPMD, G.PL_SHARED_STATIC, 0, 256)),
                    ("heap_to_stack", G.cfg(G.SPMD, G.PL_STACK, 0, 256)),
                    ("heap_to_stack_fold", G.cfg(G.SPMD, G.PL_STACK, 1, 256))]:
        def f():
            out.zero_()
            G.gtr_xs_lookup(ctx, c, xs.tables, first, n, seed, out, None, stream)
        G.gtr_ctx_fallback_high_water(ctx, reset=True, stream=stream)
        ms = _time(torch, stream, f, 2)
        info = G.gtr_query_variant(G.K_XS, c)
        ladder[name] = {"lookups_per_s": n / (ms * 1e-3), "ms": ms,
                        "same_result": bool(np.array_equal(out.cpu().numpy(), ref)),
                        "regs": info["regs"], "static_smem": info["static_smem"], "dyn_smem": info["dyn_smem"],
                        "fallback_bytes_per_thread": G.gtr_ctx_fallback_high_water(ctx, reset=True, stream=stream)}
    G.gtr_ctx_check(ctx, stream)
    # fork/join ns: 148 teams (one per SM), 20,000 trivial regions, K = 4
    fj = {}
    R, teams = 20000, 148
    fo = torch.zeros(teams, dtype=torch.uint64, device="cuda")
    for nt in (128, 256):
        row = {}
        fl = G.cfg(thread_limit=nt, num_teams=teams)
        row["barrier_floor_ns"] = _time(torch, stream, lambda: G.gtr_barrier_floor(ctx, fl, R, fo, stream), 2) \
            * 1e6 / R
        # region args in static shared memory (heap-to-shared) for every mode;
        # spmd_stack privatizes them (heap-to-stack: no guard barrier,
        # P:677-681).  "empty": one empty region forked R times (the runtime's
        # own cost); "trivial_k4": 4 distinct regions with a trivial body.
        for name, m, pl in [("generic", G.GENERIC, G.PL_SHARED_STATIC),
                            ("cascade", G.GENERIC_CASCADE, G.PL_SHARED_STATIC),
                            ("csm", G.CSM, G.PL_SHARED_STATIC), ("spmd", G.SPMD, G.PL_SHARED_STATIC),
                            ("spmd_stack", G.SPMD, G.PL_STACK),
                            ("generic_runtime_nofold", G.GENERIC, G.PL_RUNTIME)]:
            c = G.cfg(m, pl, 0 if name.endswith("nofold") else 1, nt, num_teams=teams)
            for tag, body, K in (("empty", 0, 1), ("trivial_k4", 1, 4)):
                ms = _time(torch, stream, lambda: G.gtr_forkjoin(ctx, c, R, body, K, fo, stream), 2)
                row[f"{name}_{tag}_ns"] = ms * 1e6 / R
            row[name + "_regs"] = G.gtr_query_variant(G.K_FORKJOIN, c)["regs"]
        # broadcast body (a guarded side effect producing a value): 2-barrier
        # broadcast vs the double-buffered 1-barrier form
        for name, flags in [("spmd_bcast_2bar", 0), ("spmd_bcast_1bar", G.F_BCAST_1BAR)]:
            c = G.cfg(G.SPMD, G.PL_STACK, 1, nt, num_teams=teams, flags=flags)
            ms = _time(torch, stream, lambda: G.gtr_forkjoin(ctx, c, R, 2, 1, fo, stream), 2)
            row[name + "_ns"] = ms * 1e6 / R
        c = G.cfg(G.GENERIC, G.PL_STACK, 1, nt, num_teams=teams)
        row["generic_bcast_ns"] = _time(torch, stream, lambda: G.gtr_forkjoin(ctx, c, R, 2, 1, fo, stream), 2) \
            * 1e6 / R
        if cpu:
            row["cpu_oracle_host_team"] = oracle_fj(nt)
        fj[f"thread_limit_{nt}"] = row
    G.gtr_ctx_check(ctx, stream)
    res = {"modes": modes, "grid_types": grids, "history_and_sorted": f2, "ladder_spmd": ladder, "forkjoin": fj,
           "su3": su3_sweep(G, torch, ctx, stream), "rsbench": rs_sweep(G, torch, ctx, stream, cpu=cpu)}
    if cpu:
        res["su3"]["cpu_oracle"] = oracle_su3()
        res["xs_small"] = xs_small_config(G, torch, ctx, stream)
    return res


def su3_sweep(G, torch, ctx, stream):
    """Config 3: SU(3) mat_nn on a 32^4 lattice, fp64; ms per iteration and
    algorithmic GB/s (1152 B per site: read A 576 + write C 576, B cached)."""
    import gtr_inputs.su3 as S
    from paper_conf_cgo_hubercgtddcd22_b200.problems import su3_device
    sites = 32 ** 4
    A, B = S.make_lattice(sites, "constant")
    dA, dB = su3_device(A, B)
    dC = torch.empty_like(dA)
    res = {"workload": "32^4 lattice, 4 links/site, complex fp64, constant inputs (C == 1 exactly)"}
    for name, c in [("native", G.cfg(G.NATIVE, G.PL_STACK, 1, 256)),
                    ("spmd", G.cfg(G.SPMD, G.PL_STACK, 1, 64)),
                    ("csm", G.cfg(G.CSM, G.PL_STACK, 1, 64)),
                    ("cascade", G.cfg(G.GENERIC_CASCADE, G.PL_STACK, 1, 64)),
                    ("generic", G.cfg(G.GENERIC, G.PL_STACK, 1, 64)),
                    ("generic_runtime_globalized", G.cfg(G.GENERIC, G.PL_RUNTIME, 0, 64)),
                    ("generic_llvm12_coalesced", G.cfg(G.GENERIC, G.PL_COALESCED, 0, 64)),
                    ("csm_shared_fold", G.cfg(G.CSM, G.PL_SHARED_STATIC, 1, 64)),
                    # GTR_F_TMA: sequential code streams 16-site tiles with bulk async copies
                    ("native_tma", G.cfg(G.NATIVE, G.PL_STACK, 1, 256, flags=G.F_TMA)),
                    ("spmd_tma", G.cfg(G.SPMD, G.PL_STACK, 1, 64, flags=G.F_TMA)),
                    ("csm_tma", G.cfg(G.CSM, G.PL_STACK, 1, 128, flags=G.F_TMA)),
                    ("generic_tma", G.cfg(G.GENERIC, G.PL_STACK, 1, 128, flags=G.F_TMA))]:
        ms = _time(torch, stream, lambda: G.gtr_su3_mat_nn(ctx, c, dA, dB, dC, sites, 1, stream), 3)
        ok = bool(torch.all(dC.view(-1, 2)[:, 0] == 1.0).item()) and bool(torch.all(dC.view(-1, 2)[:, 1] == 0.0).item())
        res[name] = {"ms_per_iter": ms, "gb_s": sites * 1152 / (ms * 1e-3) / 1e9,
                     "hbm_frac": sites * 1152 / (ms * 1e-3) / 1e9 / peaks()[0],
                     "regs": G.gtr_query_variant(G.K_SU3, c)["regs"], "closed_form_ok": ok}
    G.gtr_ctx_check(ctx, stream)
    del dA, dC
    # Fig. 11c analogue: speed-up over the LLVM 12 configuration (generic mode,
    # coalesced globalization, no folding) of each step of the paper's ladder
    base = res["generic_llvm12_coalesced"]["ms_per_iter"]
    res["paper_ladder_speedup_vs_llvm12"] = {
        "opts_disabled_simplified_globalization": base / res["generic_runtime_globalized"]["ms_per_iter"],
        "h2s2_rtcspec_csm": base / res["csm_shared_fold"]["ms_per_iter"],
        "h2s2_rtcspec_spmdization": base / res["spmd"]["ms_per_iter"],
        "cuda_native": base / res["native"]["ms_per_iter"]}
    return res


def fp64_peak(G, torch, ctx, stream):
    """Measured fp64 FMA ceiling (gtr_fp64_probe), TFLOP/s."""
    scratch = torch.zeros(1, dtype=torch.uint64, device="cuda")
    fl = G.gtr_fp64_probe(ctx, 4096, scratch, stream)
    ms = _time(torch, stream, lambda: G.gtr_fp64_probe(ctx, 4096, scratch, stream), 5)
    return fl / (ms * 1e-3) / 1e12


def rs_roofline(G, torch, ctx, stream, first, n, ms):
    """`bound: alu` roofline of the RS lookup kernel: algorithmic flops of the
    timed lookups (profiles/rs_work.json, written by tools/rs_work.py from the
    oracle's work counter) per second vs the measured fp64 FMA ceiling."""
    p = os.path.join(ROOT, "profiles", "rs_work.json")
    if not os.path.exists(p):
        return None
    w = json.load(open(p))
    if (w["first"], w["n"]) != (first, n):
        return None
    peak = fp64_peak(G, torch, ctx, stream)
    ach = w["flops"] / (ms * 1e-3) / 1e12
    return {"bound": "alu", "achieved": ach, "peak": peak, "unit": "TFLOP/s", "frac": ach / peak,
            "traffic": None, "flops_per_launch": w["flops"], "transcendentals_per_launch": w["transcendentals"],
            "peak_source": "measured: gtr_fp64_probe (independent DFMA chains, 2 flops each); nominal "
                           "148 SM x 64 fp64 lanes x 2 x 1.965 GHz = 37.2 TFLOP/s",
            "flops_source": "profiles/rs_work.json (oracle work counter, tools/rs_work.py)"}


def sharded_apps(G, torch, ctx, rank, ws, dist, stream, dev):
    """RSBench lookups and SU3 sites sharded over the ranks
    (weak scaling), timed on the device, max over ranks.  RS: 10M lookups per
    GPU + the same NCCL all-reduce of the 18 u64 results as XS.  SU3: 32^4
    sites per GPU (A, C sharded, B replicated), no collective on the data path;
    the closed form (C == 1 exactly) is checked on every rank."""
    import gtr_inputs.rs as RS
    import gtr_inputs.su3 as S
    import gtr_inputs.xs as X
    from paper_conf_cgo_hubercgtddcd22_b200.problems import RsDevice, su3_device
    from paper_conf_cgo_hubercgtddcd22_b200.dist import shard_range, site_shard, combine_results, max_over_ranks
    res = {}
    n_rs = 10_000_000
    first, n = shard_range(rank, ws, n_rs)
    rsd = RsDevice(RS.make_tables(), device=dev)
    out = torch.zeros(18, dtype=torch.uint64, device=dev)
    c = G.cfg(G.SPMD, G.PL_STACK, 1, 128)

    def rs_step():
        out.zero_()
        G.gtr_rs_lookup(ctx, c, rsd.tables, first, n, X.SEED_L, out, None, stream)

    ms = _time(torch, stream, rs_step, 2)
    t = torch.tensor([ms], dtype=torch.float64, device=dev)
    if dist is not None:
        combine_results(out)
        max_over_ranks(t)
    ms = float(t[0])
    r = out.cpu().numpy()
    res["rsbench"] = {"workload": f"{n_rs} lookups per GPU (global ids [r*{n_rs}, (r+1)*{n_rs})), "
                                  "SPMD + heap-to-stack + folding, thread_limit 128",
                      "n_gpus": ws, "lookups_per_s": ws * n / (ms * 1e-3), "ms_max_over_ranks": ms,
                      "hash": int(r[0]), "collective": "NCCL all_reduce(SUM) of 18 u64" if ws > 1 else None}
    del rsd
    sites = 32 ** 4
    f0, m = site_shard(rank, ws, sites)
    A, B = S.make_lattice(m, "constant", first_site=f0)
    dA, dB = su3_device(A, B, device=dev)
    del A
    dC = torch.empty_like(dA)
    for name, cc in (("native", G.cfg(G.NATIVE, G.PL_STACK, 1, 256)), ("spmd", G.cfg(G.SPMD, G.PL_STACK, 1, 64)),
                     ("native_tma", G.cfg(G.NATIVE, G.PL_STACK, 1, 256, flags=G.F_TMA)),
                     ("spmd_tma", G.cfg(G.SPMD, G.PL_STACK, 1, 64, flags=G.F_TMA))):
        ms = _time(torch, stream, lambda: G.gtr_su3_mat_nn(ctx, cc, dA, dB, dC, m, 1, stream), 3)
        ok = bool(torch.all(dC.view(-1, 2)[:, 0] == 1.0).item()) and bool(torch.all(dC.view(-1, 2)[:, 1] == 0.0).item())
        t = torch.tensor([ms, 0.0 if ok else 1.0], dtype=torch.float64, device=dev)
        if dist is not None:
            max_over_ranks(t)
        ms = float(t[0])
        res[f"su3_{name}"] = {"workload": "32^4 sites per GPU, constant inputs", "n_gpus": ws,
                              "ms_per_iter_max_over_ranks": ms, "sites_per_s": ws * m / (ms * 1e-3),
                              "gb_s_aggregate": ws * m * 1152 / (ms * 1e-3) / 1e9,
                              "closed_form_ok_all_ranks": float(t[1]) == 0.0}
    del dA, dC
    G.gtr_ctx_check(ctx, stream)
    torch.cuda.empty_cache()
    return res


def rs_sweep(G, torch, ctx, stream, n=10_000_000, cpu=True):
    """Config 4: RSBench multipole lookups (355 nuclides, 10M lookups),
    lookups/s per mode (+ the oracle on the host cores, bounded sample)."""
    import gtr_inputs.rs as RS
    import gtr_inputs.xs as X
    from paper_conf_cgo_hubercgtddcd22_b200.problems import RsDevice
    dev = RsDevice(RS.make_tables())
    out = torch.zeros(18, dtype=torch.uint64, device="cuda")
    res = {"workload": f"355 nuclides, ~1000 poles / 100 windows each, {n} lookups"}
    ref = None
    for name, c in [("native_plain", G.cfg(G.NATIVE, G.PL_STACK, 1, 128)),
                    ("native_bucketed", G.cfg(G.NATIVE, G.PL_STACK, 1, 128, flags=G.F_NATIVE_BUCKETED)),
                    ("spmd", G.cfg(G.SPMD, G.PL_STACK, 1, 128)),
                    ("spmd_plain", G.cfg(G.SPMD, G.PL_STACK, 1, 128, flags=G.F_PLAIN)),
                    ("csm", G.cfg(G.CSM, G.PL_STACK, 1, 128)),
                    ("generic", G.cfg(G.GENERIC, G.PL_STACK, 1, 128)),
                    ("generic_plain", G.cfg(G.GENERIC, G.PL_STACK, 1, 128, flags=G.F_PLAIN)),
                    ("spmd_runtime_globalized", G.cfg(G.SPMD, G.PL_RUNTIME, 0, 128)),
                    ("spmd_global_heap", G.cfg(G.SPMD, G.PL_GLOBAL, 0, 128))]:
        def f():
            out.zero_()
            G.gtr_rs_lookup(ctx, c, dev.tables, 0, n, X.SEED_L, out, None, stream)
        G.gtr_ctx_fallback_high_water(ctx, reset=True, stream=stream)
        ms = _time(torch, stream, f, 1)
        r = out.cpu().numpy()
        ref = r if ref is None else ref
        res[name] = {"lookups_per_s": n / (ms * 1e-3), "ms": ms, "regs": G.gtr_query_variant(G.K_RS, c)["regs"],
                     "same_result": bool(np.array_equal(r, ref)),
                     "fallback_bytes_per_thread": G.gtr_ctx_fallback_high_water(ctx, reset=True, stream=stream)}
    G.gtr_ctx_check(ctx, stream)
    rate = {k: v["lookups_per_s"] for k, v in res.items() if isinstance(v, dict)}
    res["fraction_of_cuda"] = {
        "bucketed_schedule": {m: rate[m] / rate["native_bucketed"] for m in ("spmd", "csm", "generic")},
        "paper_plain_schedule": {m: rate[m + "_plain"] / rate["native_plain"] for m in ("spmd", "generic")},
        "paper_v100": {"rsbench_llvm_dev_vs_cuda": 0.98}}
    res["roofline_spmd"] = rs_roofline(G, torch, ctx, stream, 0, n, res["spmd"]["ms"])
    if cpu:
        orc, o_out = oracle_rs()
        m = 100_000
        out.zero_()
        G.gtr_rs_lookup(ctx, G.cfg(G.SPMD, G.PL_STACK, 1, 128), dev.tables, 0, m, X.SEED_L, out, None, stream)
        orc["same_result_as_gpu"] = bool(np.array_equal(out.cpu().numpy(), o_out))
        res["cpu_oracle"] = orc
    return res


if __name__ == "__main__":
    a = parse()
    if a.impl == "reference":
        run_reference(a)
    else:
        run_gtr(a)
