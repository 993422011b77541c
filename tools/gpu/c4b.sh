O=gpurun_out
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 900 python tools/c4_block.py 2>&1 | tee $O/c4_block.txt
