"""Print the key fields of bench JSON lines (tools/show_bench.py FILE...)."""
import json
import sys

for fn in sys.argv[1:]:
    for line in open(fn):
        line = line.strip()
        if not line.startswith("{"):
            continue
        d = json.loads(line)
        sw = d.get("sweep", {})
        print(fn, d.get("config", {}).get("workload"), "value=%.1f %s ms/step=%.4f" % (d["value"], d["unit"],
              d["ms_per_step"]))
        if "roofline" in d:
            r = d["roofline"]
            print("  roofline", r["bound"], "achieved=%.3g peak=%.3g frac=%.3f traffic=%s" % (
                r["achieved"], r["peak"], r["frac"], r.get("traffic")))
        if "tuner" in d:
            print("  tuner", d["tuner"], "regret=%.4f vs_maxocc=%.4f vs_nvcc=%.4f" % (
                d["regret"], d["vs_maxocc"], d["vs_nvcc_default"]))
            print("  sweep", [(l["k"], l["reg_cap"], l["regs"], l["pad"], l.get("carveout_kb"), l["spill_st"], l["ms"])
                              for l in sw["levels"]])
        if d.get("carveout_axis"):
            ca = d["carveout_axis"]
            print("  carveout axis", ca["realise"], [(l["k"], l["carveout_kb"], l["pad"], l["ms"]) for l in ca["levels"]])
        for k in ("cpu_baseline", "e2e", "clocks", "gpu_launches"):
            if k in d:
                print("  ", k, d[k])
