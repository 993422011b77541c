for T in 10 1000000 3 40; do echo "== DTS_POP_BATCH_MIN=$T"; DTS_POP_BATCH_MIN=$T python tools/prof_fine.py 2>&1 | grep -A1 "2d_N100\|3d"; done
