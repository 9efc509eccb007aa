"""Regenerate the two tables of profiles/r02_ncu.md from profiles/ncu_summary.json."""
import json, sys

def main(md="profiles/r02_ncu.md", summ="profiles/ncu_summary.json", tag=None):
    d = json.load(open(summ))
    ll = {k.replace("crocco::", ""): v for k, v in d["launch_list"].items()
          if k.startswith(("crocco::k_sweep_s", "crocco::k_visc_tiled", "crocco::k_fill_gather"))}
    tot = sum(v["n"] * v["avg_ms"] for v in ll.values())
    rows = ["| kernel | launches | avg ms | share of step kernels |", "|---|---|---|---|"]
    for k, v in sorted(ll.items(), key=lambda kv: -kv[1]["avg_ms"]):
        rows.append(f"| `{k}` | {v['n']} | {v['avg_ms']:.3f} | {v['n'] * v['avg_ms'] / tot:.3f} |")
    t2 = ["| kernel | ms | regs | occupancy % | FP64 pipe % | issue active % | DRAM GB / launch | top stalls (per issue) |",
          "|---|---|---|---|---|---|---|---|"]
    for k, v in d["kernels"].items():
        t2.append(f"| `{k}` | {v['duration'] * 1e3:.3f} | {v['regs']:.0f} | {v['achieved_occupancy_pct']:.1f} | "
                  f"{v['fp64_pipe_pct']:.1f} | {v['issue_active_pct']:.1f} | {v['dram_bytes_per_launch'] / 1e9:.2f} | "
                  f"{', '.join(v['top_stalls'])} |")
    src = open(md).read()
    a = src.index("| kernel | launches"); b = src.index("## Full capture")
    c = src.index("| kernel | ms |"); e = src.index("Final capture of round 2")
    new = src[:a] + "\n".join(rows) + "\n\n" + src[b:c] + "\n".join(t2) + "\n\n" + src[e:]
    if tag:
        import re
        new = re.sub(r"Final capture of round 2 \([^)]*\)", f"Final capture of round 2 ({tag})", new, count=1)
    open(md, "w").write(new)

if __name__ == "__main__":
    main(tag=sys.argv[1] if len(sys.argv) > 1 else None)
