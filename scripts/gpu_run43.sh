set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r43_build.log 2>&1 || echo BUILD FAILED
timeout 900 python -m pytest tests -x -q -m gpu -k "top or fused or upward or distance or edge or every_k or c2" 2>&1 | tail -3
B="python bench.py --e2e-steps 0 --no-cpu-baseline"
show() { python -c "import json,sys;d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]);r=d['roofline'];print(sys.argv[1], round(d['value'],1), 'step', round(d['ms_per_step'],4), 'sweep', round(r['sweep_ms'],4), 'up', round(r['upward_ms'],4), 'frac', round(r['frac'],3), d['config'].get('us_per_tree'))" $1; }
for cfg in "C2 --k 16" "C2D --k 16" "C2 --k 64"; do
n=$(echo $cfg | tr -d ' -')
PHAST_VERBOSE=1 timeout 600 $B --config $cfg --steps 50 > gpurun_out/r43_$n.json 2>gpurun_out/r43_$n.err; show gpurun_out/r43_$n.json; grep plan gpurun_out/r43_$n.err
PHAST_UP_HYBRID=0 timeout 600 $B --config $cfg --steps 50 > gpurun_out/r43_${n}_nohy.json 2>/dev/null; show gpurun_out/r43_${n}_nohy.json
done
timeout 600 $B --cache /tmp/c3_r43.phast > gpurun_out/r43_c3.json 2>/dev/null; show gpurun_out/r43_c3.json
PHAST_UP_HYBRID=0 timeout 600 $B --cache /tmp/c3_r43.phast > gpurun_out/r43_c3_nohy.json 2>/dev/null; show gpurun_out/r43_c3_nohy.json
timeout 600 $B --cache /tmp/c3_r43.phast --k 16 > gpurun_out/r43_c3_k16.json 2>/dev/null; show gpurun_out/r43_c3_k16.json
PHAST_UP_HYBRID=0 timeout 600 $B --cache /tmp/c3_r43.phast --k 16 > gpurun_out/r43_c3_k16_nohy.json 2>/dev/null; show gpurun_out/r43_c3_k16_nohy.json
timeout 900 ncu --set full --import-source on --clock-control none --kernel-name-base demangled -k "regex:sweep_kernel<\(int\)64, \(bool\)0, \(bool\)1, \(bool\)1" -s 2 -c 1 -o gpurun_out/r43_level0 $B --cache /tmp/c3_r43.phast --steps 1 --warmup 3 > gpurun_out/r43_ncu.log 2>&1; tail -2 gpurun_out/r43_ncu.log
