TAG=${1:-c4}
O=gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/${TAG}_smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $O/${TAG}_smoke.log
timeout 1500 python -m pytest tests -m gpu -x -q > $O/${TAG}_pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 $O/${TAG}_pytest_gpu.log
timeout 600 python tools/c4_ab.py 2>&1 | tee $O/${TAG}_c4ab.txt
DTS_PROFILE=1 timeout 600 python tools/c4_ab.py 2>&1 | tee $O/${TAG}_c4ab_prof.txt
timeout 600 python tools/ab_state.py c2 c3 c5long 2>&1 | tee $O/${TAG}_ab.txt
