O=gpurun_out
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
for r in 1 2; do
for L in tools/oldlib_75692b6.so tools/oldlib_1d7b8ac.so tools/var_noce_nodefer.so paper_conf_ipps_gonthiermt22_b200/lib/libdts.so; do
  timeout 300 python tools/lib_ab.py $L 9 2>&1 | tail -1
done; done
timeout 1500 python -m pytest tests -m gpu -x -q > $O/ab3_pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 $O/ab3_pytest_gpu.log
timeout 300 python tools/san_c5.py 10 > $O/ab3_rep.log 2>&1; echo "C5 rep x10 rc=$?"; tail -1 $O/ab3_rep.log
DTS_BLOCK=128 timeout 300 python tools/san_c5.py 10 > $O/ab3_rep128.log 2>&1; echo "C5 rep128 x10 rc=$?"; tail -1 $O/ab3_rep128.log
