set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r38_build.log 2>&1 || echo BUILD FAILED
B="python bench.py --e2e-steps 0 --no-cpu-baseline"
for st in 2 4 8 24; do
PHAST_TOP_STAGES=$st timeout 600 $B --config C1 --k 1 --steps 30 > gpurun_out/r38_st$st.json 2>/dev/null; echo stages=$st; python -c "import json;d=json.load(open('gpurun_out/r38_st$st.json'));print(d['config']['us_per_tree'])"
done
timeout 600 ncu --set full --warp-sampling-interval 0 --import-source on --clock-control none -k regex:sweep_top_kernel -s 3 -c 1 -o gpurun_out/r38_top_c1 $B --config C1 --k 1 --steps 1 --warmup 3 > gpurun_out/r38_ncu_c1.log 2>&1
