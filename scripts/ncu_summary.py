"""Summarise ncu --set full reports (one kernel each) into a table for profiles/."""
import csv, glob, io, json, subprocess, sys

KEYS = [("gpu__time_duration.sum", "time"), ("sm__cycles_elapsed.avg.per_second", "sm_clk"),
        ("dram__bytes_read.sum", "dram_rd"), ("dram__bytes_write.sum", "dram_wr"),
        ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "dram_%"),
        ("sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed", "tensor_%"),
        ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm_%"),
        ("lts__t_bytes.sum", "l2_bytes"),
        ("sm__warps_active.avg.pct_of_peak_sustained_active", "occ_%"),
        ("launch__registers_per_thread", "regs"), ("launch__grid_size", "grid")]
SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "nsecond": 1e-3, "usecond": 1,
         "msecond": 1e3, "us": 1, "ns": 1e-3}


def one(path):
    if path.endswith(".csv"):           # raw page exported on the GPU box
        out = open(path).read()
    else:
        out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True,
                             text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    if len(rows) < 3 or "Kernel Name" not in rows[0]:
        return []
    hdr, units = rows[0], rows[1]
    res = []
    for r in rows[2:]:
        d = {"kernel": r[hdr.index("Kernel Name")][:60]}
        for k, name in KEYS:
            if k not in hdr:
                continue
            i = hdr.index(k)
            try:
                v = float(r[i].replace(",", ""))
            except ValueError:
                continue
            u = units[i]
            if "byte" in u:
                v = v * SCALE.get(u, 1) / 1e6   # MB
            elif "second" in u:
                v = v * SCALE.get(u, 1)         # us
            d[name] = v
        res.append(d)
    return res


if __name__ == "__main__":
    allr = []
    paths = sorted(glob.glob(sys.argv[1] + "/*.ncu-rep")) + sorted(glob.glob(sys.argv[1] + "/*.csv"))
    for p in paths:
        for d in one(p):
            d["capture"] = p.split("/")[-1].replace(".ncu-rep", "").replace(".csv", "")
            allr.append(d)
    print("# ncu --set full --clock-control none (cold cache, kernel replayed): bytes in MB, time in us")
    cols = ["time", "sm_clk", "dram_rd", "dram_wr", "dram_%", "tensor_%", "sm_%", "occ_%", "regs", "grid"]
    print("%-62s " % "kernel" + " ".join("%9s" % c for c in cols))
    for d in allr:
        print("%-62s " % (d["capture"][:16] + " " + d["kernel"].split("::")[-1][:45]) + " ".join("%9.2f" % d.get(c, float("nan")) for c in cols))
    json.dump(allr, open(sys.argv[2], "w"), indent=1) if len(sys.argv) > 2 else None
