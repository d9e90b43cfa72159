set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r44_build.log 2>&1 || echo BUILD FAILED
timeout 900 python -m pytest tests -x -q -m gpu -k "sweep_modes and levels" 2>&1 | tail -3
B="python bench.py --e2e-steps 0 --no-cpu-baseline"
show() { python -c "import json,sys;d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]);r=d['roofline'];print(sys.argv[1], round(d['value'],1), 'step', round(d['ms_per_step'],4), 'sweep', round(r['sweep_ms'],4), 'up', round(r['upward_ms'],4), 'frac', round(r['frac'],3), d['config'].get('us_per_tree'))" $1; }
for k in 64 16 32; do
timeout 600 $B --cache /tmp/c3_r44.phast --k $k > gpurun_out/r44_c3_k$k.json 2>/dev/null; show gpurun_out/r44_c3_k$k.json
PHAST_ARC_BATCH=17 timeout 600 $B --cache /tmp/c3_r44.phast --k $k > gpurun_out/r44_c3_k${k}_ellp.json 2>/dev/null; show gpurun_out/r44_c3_k${k}_ellp.json
done
timeout 600 $B --config C2 --k 16 --steps 50 > gpurun_out/r44_c2.json 2>/dev/null; show gpurun_out/r44_c2.json
PHAST_ARC_BATCH=17 timeout 600 $B --config C2 --k 16 --steps 50 > gpurun_out/r44_c2_ellp.json 2>/dev/null; show gpurun_out/r44_c2_ellp.json
timeout 300 ncu --cache-control none --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r44_launches_ellp.csv env PHAST_ARC_BATCH=17 $B --cache /tmp/c3_r44.phast --steps 1 --warmup 3 > /dev/null 2>&1
python tools/launches.py gpurun_out/r44_launches_ellp.csv v > gpurun_out/r44_launches_ellp.txt 2>&1; head -3 gpurun_out/r44_launches_ellp.txt; tail -10 gpurun_out/r44_launches_ellp.txt
