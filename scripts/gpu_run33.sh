set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r33_build.log 2>&1 || echo BUILD FAILED
timeout 900 python -m pytest tests -x -q -m gpu -k "top or c1 or every_k or edge or diameter or parents" 2>&1 | tail -3
B="python bench.py --e2e-steps 0 --no-cpu-baseline"
timeout 600 $B --cache /tmp/c3_r33.phast > gpurun_out/r33_c3.json 2>gpurun_out/r33_c3.err; cat gpurun_out/r33_c3.json; tail -2 gpurun_out/r33_c3.err
PHAST_TOP=0 timeout 600 $B --cache /tmp/c3_r33.phast > gpurun_out/r33_c3_notop.json 2>&1; tail -1 gpurun_out/r33_c3_notop.json
PHAST_VERBOSE=1 timeout 600 $B --config C1 --k 1 --steps 50 > gpurun_out/r33_c1.json 2>gpurun_out/r33_c1.err; cat gpurun_out/r33_c1.json; grep -i "top plan" gpurun_out/r33_c1.err
PHAST_TOP=0 timeout 600 $B --config C1 --k 1 --steps 50 > gpurun_out/r33_c1_notop.json 2>&1; tail -1 gpurun_out/r33_c1_notop.json
PHAST_VERBOSE=1 timeout 600 $B --config C2 --k 16 --steps 50 > gpurun_out/r33_c2.json 2>gpurun_out/r33_c2.err; cat gpurun_out/r33_c2.json; grep -i "top plan" gpurun_out/r33_c2.err
PHAST_TOP=0 timeout 600 $B --config C2 --k 16 --steps 50 > gpurun_out/r33_c2_notop.json 2>&1; tail -1 gpurun_out/r33_c2_notop.json
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r33_launches_c1.csv $B --config C1 --k 1 --steps 1 --warmup 3 > /dev/null 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r33_launches.csv $B --cache /tmp/c3_r33.phast --steps 1 --warmup 3 > /dev/null 2>&1
python tools/launches.py gpurun_out/r33_launches.csv v > gpurun_out/r33_launches.txt 2>&1; head -3 gpurun_out/r33_launches.txt
python tools/launches.py gpurun_out/r33_launches_c1.csv v > gpurun_out/r33_launches_c1.txt 2>&1; tail -12 gpurun_out/r33_launches_c1.txt
