#!/bin/bash
# Round-2 measurement set (one GPU): the GPU tests and smoke (scripts/gpu_tests.sh), every
# config's bench line, C4 strong scaling, C5 diameter, centrality, parents, and one ncu
# --set full of the dominant launch.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
T=${1:-fin}
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${T}_build.log 2>&1 || exit 1
[ -n "$2" ] && bash scripts/gpu_tests.sh
run() { n=$1; shift; timeout 1200 python bench.py "$@" > gpurun_out/${T}_$n.json 2> gpurun_out/${T}_$n.err; echo "$n rc=$?"; }
run c3k64 --config C3 --k 64 --cache /tmp/C3.phast --parents
run c3k32 --config C3 --k 32 --cache /tmp/C3.phast --no-cpu-baseline
run c3k16 --config C3 --k 16 --cache /tmp/C3.phast --no-cpu-baseline
run c3ref --impl reference --config C3 --steps 3 --warmup 1
run c4 --config C4 --k 64 --total-sources 8192 --cache /tmp/C4.phast --no-cpu-baseline
run c2 --config C2 --k 16
run c2steady --config C2 --k 16 --steady --no-cpu-baseline
run c2d --config C2D --k 16 --no-cpu-baseline
run c1 --config C1 --k 1 --inflight 1
timeout 1200 python bench_diameter.py --config C5 > gpurun_out/${T}_c5.json 2> gpurun_out/${T}_c5.err; echo "c5 rc=$?"
timeout 900 python bench_betweenness.py > gpurun_out/${T}_bc.json 2> gpurun_out/${T}_bc.err; echo "bc rc=$?"
timeout 900 python bench_betweenness.py --reach > gpurun_out/${T}_reach.json 2> gpurun_out/${T}_reach.err; echo "reach rc=$?"
# the dominant launch: the bottom band (levels 0-4 at C3 k=64), the last band launch of the 3rd query
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sweep_band_kernel -s 26 -c 1 -o gpurun_out/${T}_ncu_band0 \
   python bench.py --config C3 --k 64 --cache /tmp/C3.phast --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-probes \
   > gpurun_out/${T}_ncu.log 2>&1; echo "ncu rc=$?"
