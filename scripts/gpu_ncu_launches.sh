#!/bin/bash
# Warm-L2 ncu launch lists (time + DRAM bytes per launch) of the bench's default path.
# usage: gpurun -- bash scripts/gpu_ncu_launches.sh TAG C3:64 C3:32 ...
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
TAG=$1; shift
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1 || exit 1
for ck in "$@"; do
  C=${ck%%:*}; K=${ck##*:}
  timeout 1500 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --cache-control none \
     --clock-control none --csv --log-file gpurun_out/${TAG}_${C}_k${K}.csv \
     python bench.py --config $C --k $K --steps 2 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-probes \
       --cache /tmp/${C}.phast > gpurun_out/${TAG}_${C}_k${K}.log 2>&1
  echo "$C k=$K rc=$?"
  python tools/launches.py gpurun_out/${TAG}_${C}_k${K}.csv | tail -2
done
