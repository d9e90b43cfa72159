set -x
mkdir -p gpurun_out
(cd paper_conf_ipps_dellinggnw11_b200/csrc && make -B -j16 > /dev/null 2>&1) || echo BUILD FAILED
timeout 900 python -m pytest tests -x -q -m gpu 2>&1 | tail -3
timeout 500 python bench.py --cache /tmp/c3p.phast --parents --e2e-steps 0 --no-cpu-baseline > gpurun_out/r30_c3p.json 2>gpurun_out/r30_c3p.err; cat gpurun_out/r30_c3p.json; tail -2 gpurun_out/r30_c3p.err
for k in 1 4 16; do timeout 300 python bench.py --k $k --cache /tmp/c3p.phast --e2e-steps 0 --no-cpu-baseline > gpurun_out/r30_k$k.json 2>/dev/null; cat gpurun_out/r30_k$k.json; done
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
