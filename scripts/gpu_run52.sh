set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r52_build.log 2>&1 || echo BUILD FAILED
B="python bench.py --e2e-steps 0 --no-cpu-baseline"
show() { python -c "import json,sys;d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]);r=d['roofline'];print(sys.argv[1], round(d['value'],1), 'step', round(d['ms_per_step'],4), 'sweep', round(r['sweep_ms'],4), 'up', round(r['upward_ms'],4), 'frac', round(r['frac'],3), d['config'].get('us_per_tree'))" $1; }
for cfg in "C1 --k 1" "C1 --k 4" "C2 --k 16" "C2D --k 16"; do
n=$(echo $cfg | tr -d ' -')
for t in 1 0; do PHAST_TOP_TMA=$t timeout 600 $B --config $cfg --steps 50 > gpurun_out/r52_${n}_t$t.json 2>/dev/null; show gpurun_out/r52_${n}_t$t.json; done
done
for sk in 0 2; do PHAST_TOP_SKIP=$sk PHAST_TOP_DEBUG=gpurun_out/r52_top_c1_s$sk.bin timeout 600 $B --config C1 --k 1 --steps 3 --warmup 3 > /dev/null 2>&1; done
timeout 600 $B --cache /tmp/c3_r52.phast > gpurun_out/r52_c3.json 2>/dev/null; show gpurun_out/r52_c3.json
timeout 900 python -m pytest tests -x -q -m gpu -k "top or fused or hub or c1_all or edge_case or distance_metric_deep" 2>&1 | tail -2
