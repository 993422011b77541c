TAG=${1:-trk}
O=gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/${TAG}_smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $O/${TAG}_smoke.log
for L in tools/oldlib_0b842ed.so paper_conf_ipps_gonthiermt22_b200/lib/libdts.so; do timeout 300 python tools/lib_ab.py $L 5 2>&1 | tail -1; done
timeout 600 python tools/c4_block.py 2>&1 | grep "block 512"
DTS_TRACK=1 timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "verify or shapes or lru or w1 or opti" > $O/${TAG}_track_pytest.log 2>&1; echo "forced-track pytest rc=$?"; tail -2 $O/${TAG}_track_pytest.log
timeout 1500 python -m pytest tests -m gpu -x -q > $O/${TAG}_pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 $O/${TAG}_pytest_gpu.log
