"""Top CUDA source lines by warp-stall samples, per kernel, from an ncu report (source page, cuda,sass view).
usage: python scripts/ncu_hot_src.py rep.ncu-rep [top]

The cuda,sass view lists, per file and function, each CUDA line with its aggregated metrics followed
by its SASS; only the aggregated CUDA-line rows are used.  Stall reasons of each line are printed as
the largest per-reason columns."""
import collections
import csv
import subprocess
import sys

rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 25
txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
per = collections.defaultdict(list)        # function -> [(samples, file:line, source, reasons)]
fpath, func, hdr = "", "", None
for r in csv.reader(txt.splitlines()):
    if not r:
        continue
    if r[0] == "File Path":
        fpath = r[1].split("/")[-1]
        continue
    if r[0] == "Function Name":
        func = r[1]
        continue
    if r[0] == "Line No":
        hdr = r
        continue
    if hdr is None or not r[0] or r[0] == "":
        continue
    try:
        smp = float(r[4])
    except (ValueError, IndexError):
        continue
    reasons = []
    for i, h in enumerate(hdr):
        if h.startswith("stall_") or "Stall Sampling (" in h and h not in ("Warp Stall Sampling (All Samples)",
                                                                            "Warp Stall Sampling (Not-issued Samples)"):
            try:
                v = float(r[i])
            except (ValueError, IndexError):
                continue
            if v > 0.15 * smp and v > 0:
                reasons.append("%s=%d" % (h.replace("stall_", ""), v))
    per[func].append((smp, "%s:%s" % (fpath, r[0]), r[1], reasons))

for func, lines in per.items():
    tot = sum(x[0] for x in lines)
    print("== %s  samples %d" % (func[:120], tot))
    for smp, loc, src, reasons in sorted(lines, key=lambda x: -x[0])[:top]:
        print("  %6d %5.1f%%  %-22s %-70s %s" % (smp, 100 * smp / max(tot, 1), loc, src.strip()[:70], " ".join(reasons[:3])))
