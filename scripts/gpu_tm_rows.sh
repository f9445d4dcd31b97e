#!/bin/bash
# tm vs v8 (AUTO's choice) at N = 2^16 over row counts around the 2 x SM threshold: point_time.py with
# L = 2 (rows = 4 x ciphertexts) and L = 36
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
for nct in 37 38 74 75 111 148 296 576 1152; do
  for k in v8 tm; do
    echo -n "L=2 rows=$((4 * nct)) kern=$k: "; WD_NTT_KERNEL=$k timeout 120 python scripts/point_time.py 16 2 $nct 20 2>&1 | tail -1
  done
done
for nct in 2 4 8 16 32 64 128; do
  for k in v8 tm; do
    echo -n "L=36 rows=$((72 * nct)) kern=$k: "; WD_NTT_KERNEL=$k timeout 120 python scripts/point_time.py 16 36 $nct 20 2>&1 | tail -1
  done
done
