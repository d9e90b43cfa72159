set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r60_build.log 2>&1 || echo BUILD FAILED
timeout 600 python -m pytest tests -x -q -m gpu -k "betweenness or reach or centrality" 2>&1 | tail -5
for c in C1 C2; do
  cnt=1024; k=64; [ $c = C2 ] && cnt=256 && k=16
  timeout 600 python bench_betweenness.py --config $c --count $cnt --k $k > gpurun_out/r60_bc_$c.json 2>gpurun_out/r60_bc_$c.err; cat gpurun_out/r60_bc_$c.json; tail -3 gpurun_out/r60_bc_$c.err
  timeout 600 python bench_betweenness.py --reach --config $c --count $cnt --k $k > gpurun_out/r60_reach_$c.json 2>gpurun_out/r60_reach_$c.err; cat gpurun_out/r60_reach_$c.json; tail -3 gpurun_out/r60_reach_$c.err
done
timeout 300 python bench_betweenness.py --config C2 --count 256 --k 64 --check 0 > gpurun_out/r60_bc_C2_k64.json 2>&1; cat gpurun_out/r60_bc_C2_k64.json
timeout 300 python bench_betweenness.py --reach --config C2 --count 256 --k 64 --check 0 > gpurun_out/r60_reach_C2_k64.json 2>&1; cat gpurun_out/r60_reach_C2_k64.json
python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" 2>&1 | tail -1
