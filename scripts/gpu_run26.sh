set -x
mkdir -p gpurun_out
export PHAST_VERBOSE=1
timeout 600 python -m pytest tests/test_gpu.py -x -q -k "sweep_modes and levels" 2>&1 | tail -3
B="python bench.py --e2e-steps 0 --no-cpu-baseline --cache /tmp/c3b.phast"
for ab in 8 2; do PHAST_ARC_BATCH=$ab timeout 400 $B > gpurun_out/r26_ab$ab.json 2>/dev/null; cat gpurun_out/r26_ab$ab.json; done
for k in 16 32; do PHAST_ARC_BATCH=8 timeout 400 $B --k $k > gpurun_out/r26_k${k}_ab8.json 2>/dev/null; cat gpurun_out/r26_k${k}_ab8.json; done
PHAST_ARC_BATCH=8 timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r26_launches_ab8.csv python bench.py --cache /tmp/c3b.phast --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
