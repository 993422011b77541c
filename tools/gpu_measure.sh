#!/bin/bash
# GPU-box measurement script (run through gpurun from the repo root).
#   bash tools/gpu_measure.sh TAG STAGE [STAGE ...]
# Stages:
#   smoke     __graft_entry__ build + smoke
#   tests     pytest -m gpu
#   bench     bench.py default line (C4) + the other configs (short)
#   ref       bench.py --impl reference (default workload)
#   launches  ncu launch list (gpu__time_duration) of the default bench command
#   full_C4   ncu --set full of the C4 loop launch
#   full_C5   ncu --set full of both C5 loop launches
#   full_C2   ncu --set full of the C2 loop launch
# Outputs: gpurun_out/TAG_* (summaries go to profiles/ afterwards).
TAG=$1; shift
O=gpurun_out
mkdir -p $O
for S in "$@"; do
case $S in
smoke)
  python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/${TAG}_smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $O/${TAG}_smoke.log ;;
tests)
  timeout 2400 python -m pytest tests -m gpu -q -x > $O/${TAG}_pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 $O/${TAG}_pytest_gpu.log ;;
bench)
  timeout 1200 python bench.py --steps 5 --warmup 3 > $O/${TAG}_bench_C4.json 2> $O/${TAG}_bench_C4.err; echo "C4 rc=$?"
  for W in C2 C1 C3; do timeout 600 python bench.py --workload $W > $O/${TAG}_bench_$W.json 2> $O/${TAG}_bench_$W.err; echo "$W rc=$?"; done
  timeout 900 python bench.py --workload C5 --steps 5 > $O/${TAG}_bench_C5.json 2> $O/${TAG}_bench_C5.err; echo "C5 rc=$?" ;;
bench4)
  timeout 1200 python bench.py --steps 3 --warmup 3 > $O/${TAG}_bench_C4.json 2> $O/${TAG}_bench_C4.err; echo "C4 rc=$?"; tail -c 600 $O/${TAG}_bench_C4.json ;;
ref)
  timeout 900 python bench.py --impl reference --steps 3 --warmup 3 > $O/${TAG}_bench_reference_C4.json 2> $O/${TAG}_ref.err; echo "ref rc=$?" ;;
launches)
  timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/${TAG}_launches_C4.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline > $O/${TAG}_ncu_bench.log 2>&1; echo "launches rc=$?" ;;
full_C4)
  timeout 3000 ncu --set full --import-source on --clock-control none -k regex:"dts_(cta|warp)_kernel" -s 3 -c 1 -o $O/${TAG}_full_C4 python bench.py --steps 1 --warmup 3 --no-cpu-baseline > $O/${TAG}_ncu_full_C4.log 2>&1; echo "full C4 rc=$?" ;;
full_C5)
  timeout 1500 ncu --set full --import-source on --clock-control none -k regex:"dts_(cta|warp)_kernel" -s 6 -c 2 -o $O/${TAG}_full_C5 python bench.py --workload C5 --steps 1 --warmup 3 --no-cpu-baseline > $O/${TAG}_ncu_full_C5.log 2>&1; echo "full C5 rc=$?" ;;
full_C2)
  timeout 900 ncu --set full --import-source on --clock-control none -k regex:"dts_(cta|warp)_kernel" -s 3 -c 1 -o $O/${TAG}_full_C2 python bench.py --workload C2 --steps 1 --warmup 3 --no-cpu-baseline > $O/${TAG}_ncu_full_C2.log 2>&1; echo "full C2 rc=$?" ;;
esac
done
ls $O | grep "^$TAG" | head -50
