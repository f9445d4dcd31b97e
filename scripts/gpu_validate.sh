#!/bin/bash
# full GPU validation: build, the -m gpu suite, smoke; logs under gpurun_out/val_<tag>*
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
TAG=${1:-v}
mkdir -p gpurun_out
timeout 2400 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/val_${TAG}_pytest.txt 2>&1; echo "pytest rc=$?"
tail -5 gpurun_out/val_${TAG}_pytest.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/val_${TAG}_smoke.txt 2>&1; echo "smoke rc=$?"
tail -3 gpurun_out/val_${TAG}_smoke.txt
