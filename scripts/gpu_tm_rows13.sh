#!/bin/bash
# tm vs v8 at N = 2^13 over row counts (L = 36): point_time.py with WD_NTT_KERNEL forced
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
for nct in 2 4 8 9 16 32 64 128; do
  for k in v8 tm; do
    echo -n "logN=13 L=36 rows=$((72 * nct)) kern=$k: "; WD_NTT_KERNEL=$k timeout 120 python scripts/point_time.py 13 36 $nct 20 2>&1 | tail -1
  done
done
