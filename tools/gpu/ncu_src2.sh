python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 ncu --section SourceCounters --section WarpStateStats --import-source on --clock-control none -k regex:dts_cta_kernel -s 1 -c 1 -o gpurun_out/c2n100b python tools/one_instance.py C2 19 > gpurun_out/ncu_src.log 2>&1
echo "ncu rc=$?"
ncu -i gpurun_out/c2n100b.ncu-rep --page source --csv --print-source sass > gpurun_out/c2n100b_sass.csv 2>&1
ls -la gpurun_out/c2n100b*
