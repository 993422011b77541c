#!/bin/bash
# Round-3 ncu captures (run through gpurun from the repo root); summaries go to
# profiles/ via tools/ncu_summary.py afterwards.
O=gpurun_out
M=dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_bytes.sum,sm__throughput.avg.pct_of_peak_sustained_elapsed,sm__warps_active.avg.pct_of_peak_sustained_active,launch__grid_size,launch__block_size,launch__registers_per_thread
timeout 900 ncu --metrics $M --clock-control none -k regex:dts_cta_kernel -s 3 -c 1 -o $O/r03i_c4_dram python bench.py --steps 1 --warmup 3 --no-cpu-baseline > $O/r03i_c4_dram.log 2>&1; echo "c4 dram rc=$?"
timeout 600 ncu --metrics $M --clock-control none -k regex:dts_warp_kernel -s 3 -c 1 -o $O/r03i_c5_dram python bench.py --workload C5 --steps 1 --warmup 3 --no-cpu-baseline > $O/r03i_c5_dram.log 2>&1; echo "c5 dram rc=$?"
timeout 900 ncu --set full --import-source on --clock-control none -k regex:dts_warp_kernel -s 3 -c 1 -o $O/r03i_full_C5 python bench.py --workload C5 --steps 1 --warmup 3 --no-cpu-baseline > $O/r03i_full_C5.log 2>&1; echo "full C5 rc=$?"
timeout 600 ncu --set full --import-source on --clock-control none -k regex:dts_warp_kernel -s 3 -c 1 -o $O/r03i_full_C2 python bench.py --workload C2 --steps 1 --warmup 3 --no-cpu-baseline > $O/r03i_full_C2.log 2>&1; echo "full C2 rc=$?"
for c in C4b C4a; do timeout 900 ncu --set full --import-source on --clock-control none -k regex:dts_cta_kernel -c 1 -o $O/r03i_full_${c}_prefix python tools/ncu_prefix.py $c 20000 > $O/r03i_full_${c}.log 2>&1; echo "full $c rc=$?"; done
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/r03i_launches_C4.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline > $O/r03i_ncu_bench.log 2>&1; echo "launches rc=$?"
ls -la $O | grep r03i
