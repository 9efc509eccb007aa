"""Summarise ncu reports into profiles/: per-kernel duration, DRAM bytes, registers,
occupancy, FP64-pipe and issue utilisation, top stall reasons; launch-list shares."""
import collections, csv, io, json, subprocess, sys

def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    r = list(csv.reader(io.StringIO(out)))
    return r[0], r[1], r[2:]

KEYS = {"gpu__time_duration.sum": "duration", "dram__bytes_read.sum": "dram_read", "dram__bytes_write.sum": "dram_write",
        "launch__registers_per_thread": "regs", "sm__warps_active.avg.pct_of_peak_sustained_active": "achieved_occupancy_pct",
        "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active": "fp64_pipe_pct",
        "sm__issue_active.avg.pct_of_peak_sustained_elapsed": "issue_active_pct",
        "smsp__inst_executed.sum": "warp_inst", "dram__throughput.avg.pct_of_peak_sustained_elapsed": "dram_pct",
        "launch__grid_size": "grid", "launch__block_size": "block"}
SCALE = {"ms": 1e-3, "us": 1e-6, "ns": 1e-9, "s": 1.0, "msecond": 1e-3, "usecond": 1e-6, "nsecond": 1e-9,
         "byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "KB": 1e3, "MB": 1e6, "GB": 1e9}

def summarise(reps):
    ks = {}
    for rep in reps:
        h, u, rows = raw(rep)
        for r in rows:
            name = r[h.index("Kernel Name")]
            short = name.split("(")[0].replace("void ", "").replace("crocco::", "")
            d = {}
            for k, v in KEYS.items():
                if k in h:
                    j = h.index(k)
                    try:
                        val = float(r[j].replace(",", ""))
                    except ValueError:
                        continue
                    val *= SCALE.get(u[j], 1.0)
                    d[v] = val
            stalls = []
            for j, w in enumerate(h):
                if w.startswith("smsp__average_warps_issue_stalled_") and w.endswith("_per_issue_active.ratio"):
                    try:
                        stalls.append((float(r[j]), w[len("smsp__average_warps_issue_stalled_"):-len("_per_issue_active.ratio")]))
                    except ValueError:
                        pass
            d["top_stalls"] = [f"{n}={v:.2f}" for v, n in sorted(stalls, reverse=True)[:4]]
            if "dram_read" in d:
                d["dram_bytes_per_launch"] = d["dram_read"] + d.get("dram_write", 0)
            ks[short] = d
    return ks

def launches(csvpath):
    rows = list(csv.reader(open(csvpath)))
    start = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
    h = rows[start]
    iN, iV, iU = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
    agg = collections.defaultdict(list)
    for r in rows[start + 1:]:
        if len(r) > iV:
            agg[r[iN].split("(")[0].replace("void ", "")].append(float(r[iV].replace(",", "")) * SCALE.get(r[iU], 1e-9))
    tot = sum(sum(v) for v in agg.values())
    return {k: {"n": len(v), "avg_ms": 1e3 * sum(v) / len(v), "share": sum(v) / tot}
            for k, v in sorted(agg.items(), key=lambda kv: -sum(kv[1]))}

if __name__ == "__main__":
    out, lcsv, reps = sys.argv[1], sys.argv[2], sys.argv[3:]
    js = {"kernels": summarise(reps), "launch_list": launches(lcsv)}
    json.dump(js, open(out, "w"), indent=1)
    for k, v in js["kernels"].items():
        print(k, {kk: (round(vv, 4) if isinstance(vv, float) else vv) for kk, vv in v.items()})
