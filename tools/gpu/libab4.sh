O=gpurun_out
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
for r in 1 2; do
for L in tools/var_base.so tools/var_split.so; do
  timeout 300 python tools/lib_ab.py $L 9 2>&1 | tail -1
done; done
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "packed or verify or long_rows or shapes" > $O/ab4_pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $O/ab4_pytest.log
