# State-mode A/B + full GPU parity.  usage (on the GPU box): bash tools/gpu/ab.sh TAG
TAG=${1:-ab}
O=gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/${TAG}_smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $O/${TAG}_smoke.log
timeout 1500 python -m pytest tests -m gpu -x -q > $O/${TAG}_pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -4 $O/${TAG}_pytest_gpu.log
timeout 900 python tools/ab_state.py c2 c3 c5long c4 2>&1 | tee $O/${TAG}_ab.txt
DTS_PROFILE=1 timeout 900 python tools/ab_state.py c2 c3 c5long 2>&1 | tee $O/${TAG}_ab_prof.txt
timeout 900 compute-sanitizer --tool memcheck python tools/san_sweep.py > $O/${TAG}_san.log 2>&1; echo "san rc=$?"; tail -5 $O/${TAG}_san.log
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:dts_cta_kernel -c 6 --csv python bench.py --workload C5 --steps 1 --warmup 3 --no-cpu-baseline > $O/${TAG}_ncu_c5_lite.log 2>&1; echo "ncu lite C5 rc=$?"; tail -4 $O/${TAG}_ncu_c5_lite.log
timeout 900 ncu --set full --clock-control none -k regex:dts_cta_kernel -s 3 -c 1 -o $O/${TAG}_full_C5 python bench.py --workload C5 --steps 1 --warmup 3 --no-cpu-baseline > $O/${TAG}_ncu_full_C5.log 2>&1; echo "full C5 rc=$?"; tail -4 $O/${TAG}_ncu_full_C5.log
