#!/bin/bash
# SURVEY §8(f) f3/f4 on B200: nb sweep at n=32768 b=32 FP16 (nb = b = 32 is the non-lazy ZY-style
# per-panel rank-2b update, P:203 / Fig. 6, 10), and the panel ablation (SBR_PANEL=tsqr: the paper's
# TSQR panel only, Fig. 8/9) at nb = 1024.
O=gpurun_out; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for nb in 32 256 512 1024 2048; do
  st=3; [ $nb = 32 ] && st=1
  timeout 900 python bench.py --nb $nb --steps $st --warmup 1 --no-cpu-baseline --e2e-steps 0 --form-q-steps 0 --profile-steps 1 > $O/sweep_nb$nb.json 2> $O/sweep_nb$nb.err
done
SBR_PANEL=tsqr timeout 900 python bench.py --steps 2 --warmup 1 --no-cpu-baseline --e2e-steps 0 --form-q-steps 0 --profile-steps 1 > $O/sweep_tsqr.json 2> $O/sweep_tsqr.err
SBR_PDL=0 timeout 900 python bench.py --steps 2 --warmup 1 --no-cpu-baseline --e2e-steps 0 --form-q-steps 0 --profile-steps 1 > $O/sweep_nopdl.json 2> $O/sweep_nopdl.err
echo done
