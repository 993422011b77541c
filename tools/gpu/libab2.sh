O=gpurun_out
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
for r in 1 2; do
for L in tools/oldlib_1d7b8ac.so tools/var_noce.so tools/var_nodefer.so tools/var_noce_nodefer.so paper_conf_ipps_gonthiermt22_b200/lib/libdts.so; do
  timeout 300 python tools/lib_ab.py $L 9 2>&1 | tail -1
done; done
