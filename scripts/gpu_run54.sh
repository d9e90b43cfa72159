set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r54_build.log 2>&1 || echo BUILD FAILED
timeout 1800 python -m pytest tests -x -q -m gpu --durations=6 2>&1 | tail -10
python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" 2>&1 | tail -1
timeout 900 python bench.py > gpurun_out/r54_c3.json 2>gpurun_out/r54_c3.err; cat gpurun_out/r54_c3.json
timeout 900 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/r54_ref.json 2>gpurun_out/r54_ref.err; cat gpurun_out/r54_ref.json
