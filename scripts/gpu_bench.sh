#!/bin/bash
# One GPU call: build, then bench lines.  usage: gpurun -- bash scripts/gpu_bench.sh TAG "ARGS1" "ARGS2" ...
# each ARGS is passed to bench.py; outputs gpurun_out/TAG_<i>.json / .err
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
TAG=$1; shift
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1 || { tail -30 gpurun_out/${TAG}_build.log; exit 1; }
i=0
for a in "$@"; do
  i=$((i+1))
  echo "== $a" > gpurun_out/${TAG}_$i.err
  timeout 900 python bench.py $a > gpurun_out/${TAG}_$i.json 2>> gpurun_out/${TAG}_$i.err
  echo "rc=$? $a"; tail -c 600 gpurun_out/${TAG}_$i.json
done
