#!/bin/bash
# A/B of the fused wide victim kernel (UM_VS_FUSED=1): parity subset and state microbench.
O=gpurun_out/fused; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1; echo build rc=$?
UM_VS_FUSED=1 timeout 1500 python -m pytest tests/test_gpu_parity.py -x -q -k "wide or sparse or reserve or state_micro or evict or c3_small or c1 or scenarios or radix or hash" > $O/pyt.log 2>&1; echo pyt rc=$?; tail -3 $O/pyt.log
i=0; for f in 1 0 1 0; do i=$((i+1)); UM_VS_FUSED=$f timeout 300 python bench.py --state-only > $O/state_${i}_$f.json 2> $O/state_${i}_$f.err; echo "state $i fused=$f rc=$?"; done
