"""Merge the r02 ncu --set full captures (raw CSV pages) into profiles/traffic.json (DRAM bytes
read + written per launch, per workload and kernel class) and a readable summary."""
import glob, json, os, sys
sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), ".."))
import ncu_summary

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
dirs = sys.argv[1:] or ["gpurun_out/r02full/full", "gpurun_out/r02full2/full"]
caps = {}
for d in dirs:                                  # later directories win (re-captures)
    for p in sorted(glob.glob(os.path.join(ROOT, d, "*.csv"))):
        rows = ncu_summary.one(p)
        if rows:
            caps[os.path.basename(p)[:-4]] = rows[0]
traffic = {}
lines = ["# r02 ncu --set full --clock-control none, one launch per (workload, class); cold cache "
         "(ncu flushes before each replay pass); MB = 1e6 bytes, time in us",
         "%-18s %-48s %9s %9s %9s %9s %9s %9s %6s" % ("capture", "kernel", "time", "dram_rd", "dram_wr",
                                                      "dram_%", "tensor_%", "sm_%", "regs")]
for cap in sorted(caps):
    d = caps[cap]
    wl, cls = cap.split("_", 1)
    kern = d["kernel"].split("::")[-1].split("(")[0]
    b = (d.get("dram_rd", 0) + d.get("dram_wr", 0)) * 1e6
    t = traffic.setdefault(wl, {"kernels": {}})
    t[cls] = b
    t["kernels"][cls] = kern
    lines.append("%-18s %-48s %9.2f %9.2f %9.2f %9.2f %9.2f %9.2f %6d" % (
        cap, kern[:48], d.get("time", 0), d.get("dram_rd", 0), d.get("dram_wr", 0), d.get("dram_%", 0),
        d.get("tensor_%", 0), d.get("sm_%", 0), d.get("regs", 0)))
for wl in traffic:
    traffic[wl]["note"] = ("round r02 (scripts/r02/profile_full.sh): dram__bytes_read.sum + dram__bytes_write.sum "
                           "per launch from one ncu --set full --clock-control none capture per kernel class; "
                           "writes still resident in the 126 MB L2 when the kernel ends are not counted, so "
                           "the write side is a lower bound")
json.dump(traffic, open(os.path.join(ROOT, "profiles", "traffic.json"), "w"), indent=1, sort_keys=True)
summary = os.environ.get("SUMMARY", os.path.join("profiles", "r02", "r02full_ncu_summary.txt"))
open(os.path.join(ROOT, summary), "w").write("\n".join(lines) + "\n")
print("\n".join(lines))
