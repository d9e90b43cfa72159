#!/bin/bash
# Band-launch check: GPU tests of the schedules, then C3 lines (bands vs levels-bfs, unit sizes).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
T=${1:-bd}
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${T}_build.log 2>&1 || { tail -30 gpurun_out/${T}_build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu.py -x -q -k "schedule or every_k or repeated or diameter" > gpurun_out/${T}_pytest.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/${T}_pytest.log
b() { n=$1; shift; timeout 600 python bench.py --no-cpu-baseline --e2e-steps 0 "$@" > gpurun_out/${T}_$n.json 2> gpurun_out/${T}_$n.err; echo "$n rc=$?"; python - gpurun_out/${T}_$n.json <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); r=d["roofline"]
    print(f"   value {d['value']:.0f} sweep_ms {r['sweep_ms']:.3f} frac {r['frac']:.3f} sched {d['config'].get('schedule')}")
except Exception as e: print("   parse error", e)
PY
}
b c3k64 --config C3 --k 64 --cache /tmp/C3b.phast
b c3k64_u64 --config C3 --k 64 --cache /tmp/C3b.phast --band-unit 64 --no-probes
b c3k64_u256 --config C3 --k 64 --cache /tmp/C3b.phast --band-unit 256 --no-probes
b c3k64_u512 --config C3 --k 64 --cache /tmp/C3b.phast --band-unit 512 --no-probes
b c3k32 --config C3 --k 32 --cache /tmp/C3b.phast --no-probes
b c3k16 --config C3 --k 16 --cache /tmp/C3b.phast --no-probes
b c3k64_nob --config C3 --k 64 --cache /tmp/C3b.phast --query-flags 64 --no-probes
b c2 --config C2 --k 16 --no-probes
