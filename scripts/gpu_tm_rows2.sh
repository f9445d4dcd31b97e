#!/bin/bash
# tm vs v8 at N = 2^14 / 2^15 over row counts (L = 36): point_time.py with WD_NTT_KERNEL forced
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
for ln in 15 14; do
for nct in 2 3 4 8 16 32 64 128; do
  for k in v8 tm; do
    echo -n "logN=$ln L=36 rows=$((72 * nct)) kern=$k: "; WD_NTT_KERNEL=$k timeout 120 python scripts/point_time.py $ln 36 $nct 20 2>&1 | tail -1
  done
done
done
