"""Summarise ncu --set full reports (.ncu-rep) into profiles/ncu_<name>.txt + profiles/ncu_summary.json.

usage: python tools/ncu_summary.py KERNEL_ID REPORT.ncu-rep [ROUND]
"""
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
KEYS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
    "dram__throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
    "sm__warps_active.avg.pct_of_peak_sustained_active", "sm__maximum_warps_per_active_cycle_pct",
    "launch__registers_per_thread", "launch__occupancy_limit_registers", "launch__occupancy_limit_shared_mem",
    "launch__occupancy_limit_warps", "launch__occupancy_limit_blocks", "launch__shared_mem_per_block_dynamic",
    "launch__shared_mem_config_size", "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
    "sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active",
    "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active",
    "sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active",
    "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
    "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum",
    "l1tex__data_pipe_lsu_wavefronts_mem_shared.avg.pct_of_peak_sustained_elapsed",
    "l1tex__t_bytes_pipe_lsu_mem_local_op_ld.sum", "l1tex__t_bytes_pipe_lsu_mem_local_op_st.sum",
    "smsp__average_warp_latency_issue_stalled_long_scoreboard", "smsp__inst_executed.sum",
    "sm__cycles_elapsed.avg.per_second", "smsp__issue_active.avg.pct_of_peak_sustained_active",
    "smsp__average_warps_issue_stalled_short_scoreboard_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_barrier_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_mio_throttle_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_math_pipe_throttle_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_lg_throttle_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_wait_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_not_selected_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_selected_per_issue_active.ratio",
]


def main():
    kid, rep = sys.argv[1], sys.argv[2]
    rnd = sys.argv[3] if len(sys.argv) > 3 else "r02"
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units, data = rows[0], rows[1], rows[2:]
    res = []
    for r in data:
        d = dict(zip(hdr, r))
        ent = {"kernel": d.get("Kernel Name"), "id": d.get("ID")}
        for k in KEYS:
            for h in hdr:
                if h == k:
                    ent[k] = d[h] + " " + units[hdr.index(h)]
        res.append(ent)
    txt = os.path.join(ROOT, "profiles", f"ncu_{rnd}_{kid}.txt")
    with open(txt, "w") as f:
        for e in res:
            for k, v in e.items():
                f.write(f"{k}: {v}\n")
            f.write("\n")
    summ = os.path.join(ROOT, "profiles", "ncu_summary.json")
    js = json.load(open(summ)) if os.path.exists(summ) else {}
    e = res[-1]

    def nbytes(k):
        try:
            v, u = e[k].split()[0].replace(",", ""), e[k].split()[-1]
            return float(v) * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "KB": 1e3, "MB": 1e6,
                               "GB": 1e9}.get(u, 1)
        except Exception:
            return None
    rd, wr = nbytes("dram__bytes_read.sum"), nbytes("dram__bytes_write.sum")
    js[kid] = {"round": rnd, "report": os.path.basename(rep),
               "dram_bytes_per_launch": (rd + wr) if rd is not None and wr is not None else None,
               "metrics": e}
    with open(summ, "w") as f:
        json.dump(js, f, indent=1)
    print(open(txt).read())


if __name__ == "__main__":
    main()
