#!/bin/bash
# timing-only experiment: pass with MMA directions disabled (results invalid), SBR_PASS_EXPER bits
O=gpurun_out; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for v in 0 1 2 3; do
  SBR_PASS_EXPER=$v timeout 600 python bench.py --steps 2 --warmup 1 --no-cpu-baseline --e2e-steps 0 --form-q-steps 0 --profile-steps 1 > $O/pexp_$v.json 2>$O/pexp_$v.err
done
