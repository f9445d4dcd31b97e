#!/bin/bash
# tm kernels under the -DWD_TM_DEBUG build (scripts/build_variant.py tmdbg -DWD_TM_DEBUG): TMEM addresses,
# row indices and mbarrier waits checked on the device (trap on violation), over the tm parity tests
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
D=paper_conf_hpca_fanzzfzdtksy25_b200
cp $D/libwdntt.so /tmp/libwdntt_orig.so
cp $D/libwdntt_tmdbg.so $D/libwdntt.so
timeout 1500 python -m pytest tests/test_gpu_parity.py -q -k "tm_kernel or tail_split or boundaries or config3" -p no:cacheprovider 2>&1 | tail -3
cp /tmp/libwdntt_orig.so $D/libwdntt.so
