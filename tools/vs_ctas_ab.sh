#!/bin/bash
# A/B of the wide victim scan's grid size (UM_VS_CTAS) on the state microbench.
mkdir -p gpurun_out/vsab
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/vsab/build.log 2>&1
for c in 0 148 296 444; do
  if [ $c = 0 ]; then unset UM_VS_CTAS; else export UM_VS_CTAS=$c; fi
  timeout 300 python bench.py --state-only > gpurun_out/vsab/state_$c.json 2> gpurun_out/vsab/state_$c.err; echo "ctas=$c rc=$?"
done
unset UM_VS_CTAS
