TAG=${1:-r01m}
O=gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/${TAG}_smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $O/${TAG}_smoke.log
timeout 1500 python -m pytest tests -m gpu -x -q > $O/${TAG}_pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 $O/${TAG}_pytest_gpu.log
timeout 600 python bench.py > $O/${TAG}_bench_C2.json 2> $O/${TAG}_bench_C2.err; echo "C2 rc=$?"; cat $O/${TAG}_bench_C2.json
timeout 900 python bench.py --workload C5 --steps 5 > $O/${TAG}_bench_C5.json 2> $O/${TAG}_bench_C5.err; echo "C5 rc=$?"
timeout 600 python bench.py --workload C3 > $O/${TAG}_bench_C3.json 2> $O/${TAG}_bench_C3.err; echo "C3 rc=$?"
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > $O/${TAG}_bench_reference_C2.json 2> $O/${TAG}_ref.err; echo "ref rc=$?"
