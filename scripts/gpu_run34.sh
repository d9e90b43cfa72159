set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r34_build.log 2>&1 || echo BUILD FAILED
timeout 1500 python -m pytest tests -x -q -m gpu 2>&1 | tail -4
B="python bench.py --e2e-steps 0 --no-cpu-baseline"
PHAST_VERBOSE=1 timeout 600 $B --config C1 --k 1 --steps 50 > gpurun_out/r34_c1.json 2>gpurun_out/r34_c1.err; cat gpurun_out/r34_c1.json; grep -i "plan" gpurun_out/r34_c1.err
PHAST_VERBOSE=1 timeout 600 $B --config C2 --k 16 --steps 50 > gpurun_out/r34_c2.json 2>gpurun_out/r34_c2.err; cat gpurun_out/r34_c2.json; grep -i "plan" gpurun_out/r34_c2.err
PHAST_VERBOSE=1 timeout 600 $B --cache /tmp/c3_r34.phast > gpurun_out/r34_c3.json 2>gpurun_out/r34_c3.err; cat gpurun_out/r34_c3.json; grep -i "plan" gpurun_out/r34_c3.err
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r34_launches_c1.csv $B --config C1 --k 1 --steps 1 --warmup 3 > /dev/null 2>&1
python tools/launches.py gpurun_out/r34_launches_c1.csv v > gpurun_out/r34_launches_c1.txt 2>&1; tail -5 gpurun_out/r34_launches_c1.txt
