TAG=${1:-fx}
O=gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/${TAG}_smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $O/${TAG}_smoke.log
for B in 128 64 256; do DTS_BLOCK=$B timeout 300 python tools/san_c5.py 25 > $O/${TAG}_rep$B.log 2>&1; echo "C5 rep block $B x25 rc=$?"; tail -1 $O/${TAG}_rep$B.log; done
timeout 300 python tools/san_c5.py 25 > $O/${TAG}_rep_auto.log 2>&1; echo "C5 rep auto(split) x25 rc=$?"; tail -1 $O/${TAG}_rep_auto.log
DTS_BLOCK=128 timeout 900 compute-sanitizer --tool synccheck --print-limit 20 python tools/san_c5.py 1 16 > $O/${TAG}_sync.log 2>&1; echo "synccheck128 rc=$?"; grep -v "^=========     " $O/${TAG}_sync.log | tail -3
timeout 900 compute-sanitizer --tool synccheck --print-limit 20 python tools/san_c5.py 1 8 > $O/${TAG}_sync2.log 2>&1; echo "synccheck auto rc=$?"; grep -v "^=========     " $O/${TAG}_sync2.log | tail -3
timeout 1500 python -m pytest tests -m gpu -x -q > $O/${TAG}_pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 $O/${TAG}_pytest_gpu.log
timeout 600 python tools/ab_state.py c2 c3 c5long 2>&1 | tee $O/${TAG}_ab.txt
DTS_PROFILE=1 timeout 600 python tools/ab_state.py c4 2>&1 | tee $O/${TAG}_ab_c4prof.txt
