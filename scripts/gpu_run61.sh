set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r61_build.log 2>&1 || echo BUILD FAILED
timeout 600 python -m pytest tests -x -q -m gpu -k "betweenness or reach or centrality or library" 2>&1 | tail -3
timeout 300 python bench_betweenness.py --config C2 --count 256 --k 64 --check 0 > gpurun_out/r61_bc_C2_k64.json 2>&1; cat gpurun_out/r61_bc_C2_k64.json
timeout 300 python bench_betweenness.py --reach --config C2 --count 256 --k 64 --check 0 > gpurun_out/r61_reach_C2_k64.json 2>&1; cat gpurun_out/r61_reach_C2_k64.json
python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" 2>&1 | tail -1
