set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r45_build.log 2>&1 || echo BUILD FAILED
timeout 1800 python -m pytest tests -x -q -m gpu --durations=8 2>&1 | tail -14
python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" 2>&1 | tail -1
timeout 900 python bench.py > gpurun_out/r45_c3.json 2>gpurun_out/r45_c3.err; cat gpurun_out/r45_c3.json
timeout 1200 python bench.py --config C4 --steps 128 --e2e-steps 1 --no-cpu-baseline > gpurun_out/r45_c4.json 2>gpurun_out/r45_c4.err; cat gpurun_out/r45_c4.json
