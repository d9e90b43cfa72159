#!/bin/bash
# ncu --set full of one band_kernel launch and one per-level sweep_kernel launch (level 0)
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
TAG=$1; shift
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1 || exit 1
python tools/band_sweep.py --config C3 --k 64 --cache /tmp/c3.phast --reps 1 --grid flags=16 > /dev/null 2>&1   # build + cache the hierarchy
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:band_kernel -c 1 -o gpurun_out/${TAG}_band \
   python tools/band_sweep.py --config C3 --k 64 --cache /tmp/c3.phast --reps 1 --grid "$@" > gpurun_out/${TAG}_band.log 2>&1
echo "band rc=$?"; tail -3 gpurun_out/${TAG}_band.log
