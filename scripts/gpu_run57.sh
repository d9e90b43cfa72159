set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r57_build.log 2>&1 || echo BUILD FAILED
timeout 900 python -m pytest tests -x -q -m gpu -k "betweenness or reach" 2>&1 | tail -15
for c in C1 C2; do
  cnt=1024; k=64; [ $c = C2 ] && cnt=256 && k=16
  timeout 600 python bench_betweenness.py --config $c --count $cnt --k $k > gpurun_out/r57_bc_$c.json 2>gpurun_out/r57_bc_$c.err; cat gpurun_out/r57_bc_$c.json; tail -3 gpurun_out/r57_bc_$c.err
  timeout 600 python bench_betweenness.py --reach --config $c --count $cnt --k $k > gpurun_out/r57_reach_$c.json 2>gpurun_out/r57_reach_$c.err; cat gpurun_out/r57_reach_$c.json; tail -3 gpurun_out/r57_reach_$c.err
done
