set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"
tail -3 gpurun_out/pytest_gpu.log
timeout 300 python bench.py > gpurun_out/bench_C2.json 2> gpurun_out/bench_C2.err; echo "bench rc=$?"
cat gpurun_out/bench_C2.json
timeout 300 python tools/prof_phases.py > gpurun_out/phases.txt 2>&1
timeout 600 python tools/prof_phases.py big > gpurun_out/phases_big.txt 2>&1
cat gpurun_out/phases.txt gpurun_out/phases_big.txt
