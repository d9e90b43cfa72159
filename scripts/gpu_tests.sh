#!/bin/bash
# One GPU call: build, GPU tests (fast set, then the full-size @slow cases), smoke.
# usage: gpurun -- bash scripts/gpu_tests.sh [pytest -k expr]
set -x
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/gpu.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
if [ -n "$1" ]; then K=(-k "$1"); else K=(); fi
timeout 2400 python -m pytest tests -m "gpu and not slow" -x -q "${K[@]}" > gpurun_out/pytest_gpu.log 2>&1; echo "fast rc=$?" >> gpurun_out/pytest_gpu.log
tail -5 gpurun_out/pytest_gpu.log
if [ -z "$1" ]; then
  timeout 2400 python -m pytest tests -m "gpu and slow" -x -q > gpurun_out/pytest_slow.log 2>&1; echo "slow rc=$?" >> gpurun_out/pytest_slow.log
  tail -5 gpurun_out/pytest_slow.log
fi
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
tail -4 gpurun_out/smoke.log
