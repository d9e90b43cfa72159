#!/bin/bash
# One GPU call: the full GPU test set + smoke (scripts/gpu_tests.sh), then the headline bench line.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
bash scripts/gpu_tests.sh
timeout 900 python bench.py --config C3 --k 64 > gpurun_out/val_c3k64.json 2> gpurun_out/val_c3k64.err; echo "bench rc=$?"
tail -c 1500 gpurun_out/val_c3k64.json
