#!/bin/bash
# point timings (scripts/point_time.py, config 3 by default) of library variants x kernel choices:
# gpu_ab_kern.sh "lib1 lib2" "v8 tm" REPEATS [LOGN L NCT]
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
LIBS=$1; KERNS=$2; REP=${3:-2}; LOGN=${4:-16}; L=${5:-36}; NCT=${6:-64}
D=paper_conf_hpca_fanzzfzdtksy25_b200
cp $D/libwdntt.so /tmp/libwdntt_orig.so
for r in $(seq 1 $REP); do
for v in $LIBS; do
  cp $D/libwdntt_$v.so $D/libwdntt.so
  for k in $KERNS; do
    echo -n "lib=$v kern=$k: "; WD_NTT_KERNEL=$k timeout 120 python scripts/point_time.py $LOGN $L $NCT 20 2>&1 | tail -1
  done
done; done
cp /tmp/libwdntt_orig.so $D/libwdntt.so
