#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
TAG=$1; shift
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1 || { tail -30 gpurun_out/${TAG}_build.log; exit 1; }
timeout 1500 python tools/band_sweep.py "$@" > gpurun_out/${TAG}.jsonl 2> gpurun_out/${TAG}.err
echo "rc=$?"; cat gpurun_out/${TAG}.jsonl | cut -c1-400
