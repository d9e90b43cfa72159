set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r32_build.log 2>&1 || echo BUILD FAILED
timeout 1200 python -m pytest tests -x -q -m gpu 2>&1 | tail -5
B="python bench.py --e2e-steps 0 --no-cpu-baseline"
timeout 600 $B --cache /tmp/c3_r32.phast > gpurun_out/r32_c3.json 2>gpurun_out/r32_c3.err; cat gpurun_out/r32_c3.json; tail -2 gpurun_out/r32_c3.err
for cut in 2 3 4; do for lag in 1 2; do
PHAST_BOTTOM_SEG=1 PHAST_DIAG_CUT=$cut PHAST_DIAG_LAG=$lag timeout 600 $B --layout diagonal --delta 65536 --cache /tmp/c3d_${cut}_${lag}.phast > gpurun_out/r32_diag_${cut}_${lag}.json 2>gpurun_out/r32_diag_${cut}_${lag}.err; echo cut=$cut lag=$lag; python -c "import json;d=json.load(open('gpurun_out/r32_diag_${cut}_${lag}.json'));print(d['roofline']['sweep_ms'], d['roofline']['frac'])"; tail -1 gpurun_out/r32_diag_${cut}_${lag}.err
done; done
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r32_launches.csv $B --cache /tmp/c3_r32.phast --steps 1 --warmup 3 > /dev/null 2>&1
python tools/launches.py gpurun_out/r32_launches.csv > gpurun_out/r32_launches.txt 2>&1; head -30 gpurun_out/r32_launches.txt
