#!/bin/bash
# ncu --set full of the evict_first pass (launch 301, as r05's capture) and of an early panel launch
O=gpurun_out; mkdir -p $O; T=${1:-r12}
timeout 600 ncu --set full --clock-control none --import-source on -k regex:pass_tc -s 301 -c 1 \
  -o $O/full_pass_$T -f python tools/prof_run.py > $O/ncu_full_pass_$T.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:panel_chol -s 40 -c 1 \
  -o $O/full_panel_$T -f python tools/prof_run.py > $O/ncu_full_panel_$T.log 2>&1
python tools/ncu_summary.py $O/full_pass_$T.ncu-rep > $O/ncu_full_pass_$T.txt 2>&1
python tools/ncu_summary.py $O/full_panel_$T.ncu-rep > $O/ncu_full_panel_$T.txt 2>&1
echo done
