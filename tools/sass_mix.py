"""Aggregate an `ncu --page source --csv --print-source sass` dump by opcode:
thread instructions executed per unit of work, and stall samples."""
import csv, collections, sys
path, units = sys.argv[1], float(sys.argv[2])
rows = list(csv.reader(open(path)))
h = rows[1]
iS, iT, iW = h.index("Source"), h.index("Predicated-On Thread Instructions Executed"), h.index("Warp Stall Sampling (All Samples)")
cnt = collections.Counter(); st = collections.Counter(); tot = 0; stt = 0
for r in rows[2:]:
    if len(r) <= iT: continue
    toks = r[iS].strip().split()
    if not toks: continue
    op = toks[1] if toks[0].startswith("@") and len(toks) > 1 else toks[0]
    base = op.split(".")[0]
    try:
        v = float(r[iT] or 0)
    except ValueError:
        continue
    cnt[base] += v; tot += v
    s = float(r[iW] or 0); st[base] += s; stt += s
print(f"total thread instr / unit: {tot/units:.1f}")
for k, v in cnt.most_common(25):
    print(f"  {k:10s} {v/units:9.1f}   stall-samples {st[k]/max(stt,1)*100:5.1f}%")
fl = (cnt["DADD"] + cnt["DMUL"] + 2 * cnt["DFMA"]) / units
dp = sum(cnt[k] for k in ("DADD", "DMUL", "DFMA", "DSETP", "DMNMX")) / units
print(f"FP64 flops/unit (DADD+DMUL+2*DFMA): {fl:.1f};  DP-pipe instr/unit: {dp:.1f}")
