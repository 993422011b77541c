O=gpurun_out
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
for r in 1 2; do
for L in tools/var_base.so tools/var_nob.so; do
  timeout 300 python tools/lib_ab.py $L 9 2>&1 | tail -1
done; done
timeout 1500 python -m pytest tests -m gpu -x -q > $O/ab5_pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $O/ab5_pytest.log
timeout 300 python tools/san_c5.py 6 > $O/ab5_rep.log 2>&1; echo "C5 rep x6 rc=$?"; tail -1 $O/ab5_rep.log
DTS_BLOCK=128 timeout 900 compute-sanitizer --tool synccheck --print-limit 10 python tools/san_c5.py 1 16 > $O/ab5_sync.log 2>&1; echo "synccheck rc=$?"; grep -v "^=========     " $O/ab5_sync.log | tail -2
