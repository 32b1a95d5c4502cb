"""Per-level ncu evidence (SURVEY 8(d) "ncu evidence per level"): profile one launch of every
occupancy level of a kernel with a small metric set and write a table to profiles/.

On the GPU box:   python tools/ncu_levels.py run KERNEL W H [THREADS] [BATCH]   -> gpurun_out/levels_KERNEL.csv
Here:             python tools/ncu_levels.py summarise KERNEL ROUND     -> profiles/ncu_levels_ROUND_KERNEL.txt
"""
import csv
import os
import subprocess
import sys

METRICS = [
    "gpu__time_duration.sum",
    "launch__registers_per_thread",
    "launch__occupancy_limit_registers",
    "launch__occupancy_limit_shared_mem",
    "sm__maximum_warps_per_active_cycle_pct",
    "sm__warps_active.avg.pct_of_peak_sustained_active",
    "l1tex__t_bytes_pipe_lsu_mem_local_op_ld.sum",
    "l1tex__t_bytes_pipe_lsu_mem_local_op_st.sum",
    "dram__bytes_read.sum",
    "dram__bytes_write.sum",
    "smsp__issue_active.avg.pct_of_peak_sustained_active",
    "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
    "smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio",
    "launch__shared_mem_config_size",
    "launch__shared_mem_per_block_dynamic",
]
SHORT = ["us", "regs", "lim_reg", "lim_smem", "occ_theo%", "occ_ach%", "local_ld_MB", "local_st_MB", "dram_rd_MB",
         "dram_wr_MB", "issue%", "fma%", "long_sb", "cfg_KB", "dyn_KB"]
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def run(kernel, W, H, threads="0", batch="1"):
    out = os.path.join(ROOT, "gpurun_out", f"levels_{kernel}.csv")
    cmd = ["ncu", "--clock-control", "none", "--nvtx", "--nvtx-include", "measure/", "--csv", "--metrics", ",".join(METRICS), "-k", "regex:orion_",
           "--log-file", out, sys.executable, os.path.join(ROOT, "tools", "ncu_one.py"), kernel, "all", W, H, threads, "1", batch]
    subprocess.run(cmd, check=True)


def summarise(kernel, rnd):
    path = os.path.join(ROOT, "gpurun_out", f"levels_{kernel}.csv")
    rows = [r for r in csv.reader(l for l in open(path) if l.startswith('"'))]
    hdr, data = rows[0], rows[1:]
    iid, iname, ival, iunit = hdr.index("ID"), hdr.index("Metric Name"), hdr.index("Metric Value"), hdr.index("Metric Unit")
    ik, ig = hdr.index("Kernel Name"), hdr.index("Grid Size")
    per, names = {}, {}
    for r in data:
        if "_gen_" in r[ik] or "_stats" in r[ik]:     # the input generator / SRAD statistics
            continue
        if r[ig].replace(" ", "").endswith(",1,1)") and int(r[ig].strip("()").split(",")[0]) % 4736 == 0:
            continue                                  # residency-probe launches of the build (148 x 32 CTAs)
        per.setdefault(int(r[iid]), {})[r[iname]] = (r[ival], r[iunit])
        names[int(r[iid])] = r[ik]

    def val(m, name):
        v, unit = m.get(name, ("nan", ""))
        unit = unit.split("/")[0]
        x = float(v.replace(",", ""))
        scale = {"byte": 1e-6, "Kbyte": 1e-3, "Mbyte": 1.0, "Gbyte": 1e3, "nsecond": 1e-3, "ns": 1e-3,
                 "usecond": 1.0, "us": 1.0, "msecond": 1e3, "ms": 1e3}.get(unit, 1.0)
        kb = name.startswith("launch__shared_mem")      # reported in KB, not MB
        return x * scale * (1e3 if kb else 1.0)

    lines = [f"# ncu per-level evidence: {kernel} = {names[min(per)]} (one launch per level in level order, "
             f"MIN_CARVEOUT realisation, --clock-control none; times are cold, single-launch)",
             "level " + " ".join(f"{s:>11s}" for s in SHORT)]
    for lvl, k in enumerate(sorted(per)):
        lines.append(f"{lvl:5d} " + " ".join(f"{val(per[k], m):11.2f}" for m in METRICS))
    dst = os.path.join(ROOT, "profiles", f"ncu_levels_{rnd}_{kernel}.txt")
    open(dst, "w").write("\n".join(lines) + "\n")
    print("\n".join(lines))


if __name__ == "__main__":
    if sys.argv[1] == "run":
        run(*sys.argv[2:])
    else:
        summarise(sys.argv[2], sys.argv[3])
