"""Per-opcode executed-instruction mix from an ncu report's SASS source page.
usage: python scripts/sass_mix.py rep.ncu-rep [elements]"""
import csv, io, subprocess, sys, collections
rep = sys.argv[1]
elems = float(sys.argv[2]) if len(sys.argv) > 2 else 4608 * 65536
raw = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
lines = raw.splitlines()
rows = list(csv.reader(io.StringIO("\n".join(lines[1:]))))
h = rows[0]
ie, src, smp = h.index("Instructions Executed"), h.index("Source"), h.index("Warp Stall Sampling (All Samples)")
mix, stall = collections.Counter(), collections.Counter()
tot = 0
for r in rows[1:]:
    try:
        n = int(r[ie]); s = int(r[smp])
    except Exception:
        continue
    op = r[src].strip().split()[0] if r[src].strip() else "?"
    if op.startswith("@"):
        op = r[src].strip().split()[1]
    op = op.split(".")[0]
    mix[op] += n; stall[op] += s; tot += n
print("total warp-instr %.0f  = %.1f thread-instr/element" % (tot, tot * 32 / elems))
for op, n in mix.most_common(25):
    print("  %-12s %6.2f /elem  stall-samples %d" % (op, n * 32 / elems, stall[op]))
