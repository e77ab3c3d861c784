#!/bin/bash
# fp16 pass variants (SBR_PASS_CFG) on the config-4 bench: pass ms per step from the breakdown
O=gpurun_out; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for v in 0 1 2; do
  SBR_PASS_CFG=$v timeout 600 python bench.py --steps 3 --warmup 2 --no-cpu-baseline --e2e-steps 0 --form-q-steps 0 --profile-steps 1 > $O/passcfg_$v.json 2>/dev/null
done
