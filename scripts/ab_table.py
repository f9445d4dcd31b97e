"""Summarise gpu_ab.sh outputs: python scripts/ab_table.py TAG"""
import glob, json, sys, collections
tag = sys.argv[1]
res = collections.defaultdict(list)
for f in sorted(glob.glob("gpurun_out/ab_%s_*.json" % tag)):
    key = "_".join(f.split("/")[-1][:-5].split("_")[2:-1])
    try:
        d = json.load(open(f))
        res[key].append((d["value"], d["fwd_ms"], d["inv_ms"], d["clocks"]["sm_mhz"]))
    except Exception as e:
        res[key].append(("ERR", open(f[:-5] + ".err").read()[-200:]))
for k, v in res.items():
    print("%-14s" % k, "  ".join("%.0f (%.3f/%.3f @%s)" % x if x[0] != "ERR" else "ERR %s" % x[1] for x in v))
