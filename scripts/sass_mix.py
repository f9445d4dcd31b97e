"""Per-opcode executed-instruction mix of ONE launch of each kernel in an ncu report (SASS source page).

usage: python scripts/sass_mix.py rep.ncu-rep [elements_per_launch]

The source page holds one block per profiled launch.  Only the first launch of every kernel name is
counted, and the counts are divided by the elements ONE launch transforms (default: config 3, 4608
rows x 2^16).  The round-1 version summed every launch in the report over one launch's elements and
so over-stated the per-element counts by the number of launches (4x in profiles/r01/s3/sass_v8_final.txt).
"""
import collections
import csv
import subprocess
import sys

rep = sys.argv[1]
elems = float(sys.argv[2]) if len(sys.argv) > 2 else 4608 * 65536
raw = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
blocks, cur = [], None
for r in csv.reader(raw.splitlines()):
    if r and r[0] == "Kernel Name":
        cur = [r[1], None, []]
        blocks.append(cur)
        continue
    if r and r[0] == "Address" and cur is not None:
        cur[1] = r
        continue
    if cur is not None and cur[1] and r:
        cur[2].append(r)

seen = set()
for name, hdr, data in blocks:
    if name in seen or hdr is None:
        continue
    seen.add(name)
    ie, src = hdr.index("Instructions Executed"), hdr.index("Source")
    smp = hdr.index("Warp Stall Sampling (All Samples)")
    mix, stall = collections.Counter(), collections.Counter()
    tot = 0
    for r in data:
        try:
            n = int(r[ie])
            s = int(float(r[smp] or 0))
        except (ValueError, IndexError):
            continue
        toks = r[src].strip().split()
        if not toks:
            continue
        op = toks[1] if toks[0].startswith("@") and len(toks) > 1 else toks[0]
        op = op.split(".")[0]
        mix[op] += n
        stall[op] += s
        tot += n
    print("== %s (one launch, %.0f elements)" % (name, elems))
    print("total warp-instr %.0f  = %.1f thread-instr/element" % (tot, tot * 32 / elems))
    for op, n in mix.most_common(25):
        print("  %-12s %6.2f /elem  stall-samples %d" % (op, n * 32 / elems, stall[op]))
