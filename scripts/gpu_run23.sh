set -x
mkdir -p gpurun_out
export PHAST_VERBOSE=1
timeout 600 python -m pytest tests/test_gpu.py -x -q -k "sweep_modes" 2>&1 | tail -3
B="python bench.py --e2e-steps 0 --no-cpu-baseline --cache /tmp/c3b.phast"
for t in 0 2000 20000 70000; do PHAST_TOP_THRESH=$t timeout 400 $B > gpurun_out/r23_t$t.json 2>/dev/null; cat gpurun_out/r23_t$t.json; done
PHAST_TOP_CTAS=6 PHAST_TOP_THRESH=20000 timeout 400 $B > gpurun_out/r23_t20000_c6.json 2>/dev/null; cat gpurun_out/r23_t20000_c6.json
PHAST_TOP_CTAS=2 PHAST_TOP_THRESH=20000 timeout 400 $B > gpurun_out/r23_t20000_c2.json 2>/dev/null; cat gpurun_out/r23_t20000_c2.json
PHAST_TOP_THRESH=20000 timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r23_launches_t20000.csv python bench.py --cache /tmp/c3b.phast --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
