#!/bin/bash
# r12: CholeskyQR panel phase trace inside the config-4 reduction vs standalone
O=gpurun_out; mkdir -p $O; T=${1:-r12}
python -c "import __graft_entry__ as g; g.build()" > $O/build_$T.log 2>&1
timeout 600 python tools/panel_chain_trace.py > $O/panel_chain_trace_$T.txt 2>&1
echo done
