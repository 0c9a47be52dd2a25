#!/bin/bash
# Check build of the warp-coherent sorted lookups (GTR_XS_CO_CHECK=1): every
# nuclide visit compares the pair it interpolates with its own index-table
# entry and traps otherwise.  Builds exp/libgtr_chk.so (CSM + SPMD, thread
# limit 256) and runs the sorted-mode GPU tests and the 17M-lookup XS-large
# sorted run with it.  Usage (on a GPU box): bash tools/xs_co_check.sh
set -e
[ -f exp/libgtr_chk.so ] || python tools/xs_exp_lib.py chk 256 -DGTR_XS_CO_CHECK=1
export GTR_LIB=$PWD/exp/libgtr_chk.so
python -m pytest tests/test_gpu_xs.py -q -p no:cacheprovider -k "sorted or sort_then or duplicate" 2>&1 | tail -1
python tools/xs_launch.py spmd_sorted csm_sorted --time --reps 1
