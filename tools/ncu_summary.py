"""Summarise ncu captures into profiles/ (run here, on the CPU box).

    python tools/ncu_summary.py full   <report.ncu-rep> <out.json>   # --set full capture
    python tools/ncu_summary.py launch <launches.csv>  <out.json>    # gpu__time_duration list
"""
import csv
import io
import json
import subprocess
import sys

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_sector_hit_rate.pct",
        "lts__t_sectors_srcunit_tex_op_read.sum", "l1tex__t_sector_hit_rate.pct",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
        "launch__occupancy_limit_registers", "launch__occupancy_limit_shared_mem",
        "smsp__thread_inst_executed_per_inst_executed.ratio", "smsp__inst_executed.sum",
        "lts__throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "launch__grid_size", "launch__block_size",
        # L1 data pipe (one wavefront per 128-byte line a warp instruction touches)
        "l1tex__data_pipe_lsu_wavefronts.sum", "l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "l1tex__data_pipe_lsu_wavefronts_mem_lgds.sum",
        "l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum", "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum",
        "l1tex__t_requests_pipe_lsu_mem_global_op_ldgsts.sum", "l1tex__t_sectors_pipe_lsu_mem_global_op_ldgsts.sum",
        "l1tex__throughput.avg.pct_of_peak_sustained_elapsed", "l1tex__lsu_writeback_active.avg.pct_of_peak_sustained_elapsed",
        "lts__t_sectors.sum", "lts__t_requests.sum",
        "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "smsp__average_warp_latency_issue_stalled_long_scoreboard.ratio",
        "smsp__average_warp_latency_issue_stalled_barrier.ratio",
        "smsp__average_warp_latency_issue_stalled_lg_throttle.ratio",
        "smsp__average_warp_latency_issue_stalled_mio_throttle.ratio",
        "smsp__average_warp_latency_issue_stalled_short_scoreboard.ratio",
        "smsp__average_warp_latency_issue_stalled_wait.ratio",
        "smsp__average_warp_latency_issue_stalled_math_pipe_throttle.ratio",
        "smsp__average_warp_latency_issue_stalled_membar.ratio",
        "smsp__average_warp_latency_issue_stalled_long_scoreboard.pct",
        "smsp__warp_issue_stalled_long_scoreboard_per_warp_active.pct",
        "smsp__warp_issue_stalled_lg_throttle_per_warp_active.pct",
        "smsp__warp_issue_stalled_mio_throttle_per_warp_active.pct",
        "smsp__warp_issue_stalled_barrier_per_warp_active.pct",
        "smsp__warp_issue_stalled_short_scoreboard_per_warp_active.pct",
        "smsp__warp_issue_stalled_wait_per_warp_active.pct",
        "smsp__warp_issue_stalled_math_pipe_throttle_per_warp_active.pct",
        "smsp__warp_issue_stalled_no_instruction_per_warp_active.pct",
        "smsp__warp_issue_stalled_selected_per_warp_active.pct",
        "smsp__warp_issue_stalled_not_selected_per_warp_active.pct",
        "smsp__warp_issue_stalled_dispatch_stall_per_warp_active.pct",
        "smsp__warp_issue_stalled_drain_per_warp_active.pct",
        "smsp__warp_issue_stalled_sleeping_per_warp_active.pct",
        "smsp__warp_issue_stalled_branch_resolving_per_warp_active.pct",
        "smsp__warp_issue_stalled_imc_miss_per_warp_active.pct",
        "smsp__warp_issue_stalled_membar_per_warp_active.pct",
        "smsp__inst_executed_pipe_fp64.sum", "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active"]
SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12, "ns": 1e-9, "us": 1e-6, "ms": 1e-3, "s": 1,
         "nsecond": 1e-9, "usecond": 1e-6, "msecond": 1e-3, "second": 1}


def full(rep, out):
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr, units = rows[0], rows[1]
    kernels = []
    for row in rows[2:]:
        k = {"kernel": row[hdr.index("Kernel Name")]}
        for key in KEYS:
            if key in hdr:
                i = hdr.index(key)
                v = row[i].replace(",", "")
                try:
                    v = float(v) * SCALE.get(units[i], 1)
                except ValueError:
                    pass
                k[key] = v
        if "dram__bytes_read.sum" in k:
            k["dram_bytes_per_launch"] = k["dram__bytes_read.sum"] + k.get("dram__bytes_write.sum", 0.0)
        kernels.append(k)
    json.dump({"source": rep, "units": "bytes / seconds / percent as named", "kernels": kernels},
              open(out, "w"), indent=1)
    return kernels


def launches(path, out):
    txt = open(path).read()
    lines = [l for l in txt.splitlines() if l.startswith('"')]
    rows = list(csv.reader(io.StringIO("\n".join(lines))))
    hdr = rows[0]
    ki, vi, ui = hdr.index("Kernel Name"), hdr.index("Metric Value"), hdr.index("Metric Unit")
    per = {}
    order = []
    for r in rows[1:]:
        name = r[ki].split("(")[0]
        t = float(r[vi].replace(",", "")) * SCALE.get(r[ui], 1)
        if name not in per:
            per[name] = []
            order.append(name)
        per[name].append(t)
    total = sum(sum(v) for v in per.values())
    summ = [{"kernel": n, "launches": len(per[n]), "total_s": sum(per[n]), "mean_s": sum(per[n]) / len(per[n]),
             "share": sum(per[n]) / total} for n in order]
    json.dump({"source": path, "total_s": total, "kernels": summ}, open(out, "w"), indent=1)
    return summ


if __name__ == "__main__":
    mode, src, dst = sys.argv[1:4]
    res = full(src, dst) if mode == "full" else launches(src, dst)
    for k in res:
        print(json.dumps(k)[:300])
