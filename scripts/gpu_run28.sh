set -x
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu.py -x -q -k "sweep_modes and levels or c1_all or every_k" 2>&1 | tail -3
B="python bench.py --e2e-steps 0 --no-cpu-baseline --cache /tmp/c3b.phast"
timeout 400 $B > gpurun_out/r28_ab2.json 2>/dev/null; cat gpurun_out/r28_ab2.json
PHAST_ARC_BATCH=8 timeout 400 $B > gpurun_out/r28_ab8.json 2>/dev/null; cat gpurun_out/r28_ab8.json
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r28_launches.csv python bench.py --cache /tmp/c3b.phast --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:sweep_kernel -s 246 -c 2 -o gpurun_out/r28_levels python bench.py --cache /tmp/c3b.phast --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline > gpurun_out/r28_ncu.log 2>&1
tail -3 gpurun_out/r28_ncu.log
