set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r37_build.log 2>&1 || echo BUILD FAILED
B="python bench.py --e2e-steps 0 --no-cpu-baseline"
for cfg in "C1 --k 1" "C1 --k 4" "C2 --k 16" "C2D --k 16"; do
n=$(echo $cfg | tr -d ' -')
timeout 600 $B --config $cfg --steps 50 > gpurun_out/r37_$n.json 2>gpurun_out/r37_$n.err; echo $n; python -c "import json;d=json.load(open('gpurun_out/r37_$n.json'));r=d['roofline'];print(d['value'],d['config']['us_per_tree'],r['sweep_ms'],r['upward_ms'],d['config']['levels'])"
done
timeout 900 python -m pytest tests -x -q -m gpu -k "top or fused or c1 or distance or edge" 2>&1 | tail -3
