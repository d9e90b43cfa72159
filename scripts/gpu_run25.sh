set -x
mkdir -p gpurun_out
export PHAST_VERBOSE=1
timeout 900 python -m pytest tests -x -q -m gpu 2>&1 | tail -3
B="python bench.py --e2e-steps 0 --no-cpu-baseline --cache /tmp/c3b.phast"
for ab in 2 3 4; do PHAST_ARC_BATCH=$ab timeout 400 $B > gpurun_out/r25_ab$ab.json 2>/dev/null; cat gpurun_out/r25_ab$ab.json; done
for k in 16 32; do for ab in 2 3; do PHAST_ARC_BATCH=$ab timeout 400 $B --k $k > gpurun_out/r25_k${k}_ab$ab.json 2>/dev/null; cat gpurun_out/r25_k${k}_ab$ab.json; done; done
