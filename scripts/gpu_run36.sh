set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r36_build.log 2>&1 || echo BUILD FAILED
B="python bench.py --e2e-steps 0 --no-cpu-baseline"
for cfg in "C1 --k 1" "C1 --k 4" "C2 --k 16" "C2D --k 16"; do
n=$(echo $cfg | tr -d ' -')
timeout 600 $B --config $cfg --steps 50 > gpurun_out/r36_$n.json 2>gpurun_out/r36_$n.err; echo $n; python -c "import json;d=json.load(open('gpurun_out/r36_$n.json'));r=d['roofline'];print(d['value'],d['config']['us_per_tree'],r['sweep_ms'],r['upward_ms'],d['config']['levels'])"
done
timeout 600 ncu --set full --import-source on --clock-control none -k regex:sweep_top_kernel -s 3 -c 1 -o gpurun_out/r36_top_c1 $B --config C1 --k 1 --steps 1 --warmup 3 > gpurun_out/r36_ncu_c1.log 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r36_launches_c2.csv $B --config C2 --k 16 --steps 1 --warmup 3 > /dev/null 2>&1
python tools/launches.py gpurun_out/r36_launches_c2.csv v > gpurun_out/r36_launches_c2.txt 2>&1; tail -22 gpurun_out/r36_launches_c2.txt
timeout 1500 python -m pytest tests -x -q -m gpu 2>&1 | tail -4
