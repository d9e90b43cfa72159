set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r35_build.log 2>&1 || echo BUILD FAILED
timeout 1500 python -m pytest tests -x -q -m gpu 2>&1 | tail -4
B="python bench.py --e2e-steps 0 --no-cpu-baseline"
for cfg in "C1 --k 1" "C1 --k 4" "C2 --k 16" "C2D --k 16"; do
n=$(echo $cfg | tr -d ' -')
PHAST_VERBOSE=1 timeout 600 $B --config $cfg --steps 50 > gpurun_out/r35_$n.json 2>gpurun_out/r35_$n.err; echo $n; python -c "import json;d=json.load(open('gpurun_out/r35_$n.json'));r=d['roofline'];print(d['value'],d['config']['us_per_tree'],r['sweep_ms'],r['upward_ms'],d['config']['levels'])"; grep -i "plan" gpurun_out/r35_$n.err
done
timeout 600 $B --cache /tmp/c3_r35.phast > gpurun_out/r35_c3.json 2>gpurun_out/r35_c3.err; cat gpurun_out/r35_c3.json
PHAST_ARC_BATCH=2 timeout 600 $B --cache /tmp/c3_r35.phast > gpurun_out/r35_c3_ab2.json 2>&1; tail -1 gpurun_out/r35_c3_ab2.json
for k in 16 32; do timeout 600 $B --cache /tmp/c3_r35.phast --k $k > gpurun_out/r35_c3_k$k.json 2>&1; tail -1 gpurun_out/r35_c3_k$k.json; done
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r35_launches.csv $B --cache /tmp/c3_r35.phast --steps 1 --warmup 3 > /dev/null 2>&1
python tools/launches.py gpurun_out/r35_launches.csv v > gpurun_out/r35_launches.txt 2>&1; head -3 gpurun_out/r35_launches.txt; tail -8 gpurun_out/r35_launches.txt
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r35_launches_c1.csv $B --config C1 --k 1 --steps 1 --warmup 3 > /dev/null 2>&1
python tools/launches.py gpurun_out/r35_launches_c1.csv v > gpurun_out/r35_launches_c1.txt 2>&1; tail -3 gpurun_out/r35_launches_c1.txt
