"""Top stall sites of each kernel in an ncu report (source page, SASS view)."""
import csv, subprocess, sys

rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 20
txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(txt.splitlines()))
ks, cur = [], None
for r in rows:
    if r and r[0] == "Kernel Name":
        cur = [r[1], None, []]; ks.append(cur); continue
    if r and r[0] == "Address":
        cur[1] = r; continue
    if cur and cur[1] and r:
        cur[2].append(r)
cols = ["stall_barrier", "stall_long_sb", "stall_mio", "stall_membar", "stall_lg", "stall_wait",
        "stall_math", "stall_short_sb", "stall_branch_resolving"]
seen = set()
for name, hdr, data in ks:
    if name in seen:
        continue
    seen.add(name)
    ix = {h: i for i, h in enumerate(hdr)}
    allc = ix["Warp Stall Sampling (All Samples)"]
    tot = sum(float(d[allc] or 0) for d in data)
    print("==", name, "samples", int(tot))
    print("  ", {c[6:]: int(sum(float(d[ix[c]] or 0) for d in data)) for c in cols if c in ix})
    for d in sorted(data, key=lambda d: -float(d[allc] or 0))[:top]:
        print("  ", d[0][-5:], d[1][:58].ljust(58), d[allc],
              " ".join("%s=%s" % (c[6:], d[ix[c]]) for c in cols if c in ix and float(d[ix[c]] or 0) > 0.1 * float(d[allc] or 1)))
