O=gpurun_out
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "compact or packed or verify or shapes or sweep or config2" > $O/dbg_pytest.log 2>&1; echo "pytest rc=$?"; tail -3 $O/dbg_pytest.log
for B in 128 256; do DTS_BLOCK=$B timeout 300 python tools/san_c5.py 8 > $O/dbg_rep_$B.log 2>&1; echo "rep block $B rc=$?"; tail -2 $O/dbg_rep_$B.log; done
DTS_BLOCK=128 timeout 1200 compute-sanitizer --tool memcheck --print-limit 20 python tools/san_c5.py 3 > $O/dbg_san128.log 2>&1; echo "san rc=$?"; grep -v "^=========     " $O/dbg_san128.log | head -40
