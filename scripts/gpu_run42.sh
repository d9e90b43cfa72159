set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r42_build.log 2>&1 || echo BUILD FAILED
timeout 900 python -m pytest tests -x -q -m gpu -k "top or fused or c1 or distance or edge or every_k" 2>&1 | tail -3
B="python bench.py --e2e-steps 0 --no-cpu-baseline"
show() { python -c "import json,sys;d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]);r=d['roofline'];print(sys.argv[1], round(d['value'],1), 'step', round(d['ms_per_step'],4), 'sweep', round(r['sweep_ms'],4), 'frac', round(r['frac'],3), d['config'].get('us_per_tree'))" $1; }
PHAST_VERBOSE=1 timeout 600 $B --cache /tmp/c3_r42.phast > gpurun_out/r42_c3.json 2>gpurun_out/r42_c3.err; show gpurun_out/r42_c3.json; grep plan gpurun_out/r42_c3.err
for p in 2 4 16; do PHAST_CL_PASSES=$p timeout 600 $B --cache /tmp/c3_r42.phast > gpurun_out/r42_c3_p$p.json 2>/dev/null; show gpurun_out/r42_c3_p$p.json; done
PHAST_CL_SIZE=8 timeout 600 $B --cache /tmp/c3_r42.phast > gpurun_out/r42_c3_cl8.json 2>/dev/null; show gpurun_out/r42_c3_cl8.json
PHAST_CL_SIZE=0 timeout 600 $B --cache /tmp/c3_r42.phast > gpurun_out/r42_c3_cl0.json 2>/dev/null; show gpurun_out/r42_c3_cl0.json
for k in 16 32; do timeout 600 $B --cache /tmp/c3_r42.phast --k $k > gpurun_out/r42_c3_k$k.json 2>/dev/null; show gpurun_out/r42_c3_k$k.json; done
for cfg in "C1 --k 1" "C2 --k 16" "C2D --k 16"; do
n=$(echo $cfg | tr -d ' -')
PHAST_VERBOSE=1 timeout 600 $B --config $cfg --steps 50 > gpurun_out/r42_$n.json 2>gpurun_out/r42_$n.err; show gpurun_out/r42_$n.json; grep plan gpurun_out/r42_$n.err
PHAST_CL_SIZE=0 timeout 600 $B --config $cfg --steps 50 > gpurun_out/r42_${n}_cl0.json 2>/dev/null; show gpurun_out/r42_${n}_cl0.json
done
