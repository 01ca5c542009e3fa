#!/bin/bash
# A/B of k_classify geometry on the GPU box (rebuilds in the box's copy of the repo)
set -u
K=paper_conf_iiswc_zhucvhcr22_b200/csrc
run() {
  python -m paper_conf_iiswc_zhucvhcr22_b200.build --force > /dev/null || return
  for r in 1 2; do timeout 300 python tools/state_micro.py | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read())
print('$1', [(k, round(v['ms_plan']*1000,1)) for k,v in d.items() if k!='stats'])"; done
}
run ipt8_lb5
sed -i 's/constexpr int kClsIPT = 8;/constexpr int kClsIPT = 16;/' $K/um_internal.h
sed -i 's/__launch_bounds__(kStTPB, 5) k_classify(/__launch_bounds__(kStTPB, 4) k_classify(/' $K/um_kernels.cu
run ipt16_lb4
sed -i 's/constexpr int kClsIPT = 16;/constexpr int kClsIPT = 4;/' $K/um_internal.h
sed -i 's/__launch_bounds__(kStTPB, 4) k_classify(/__launch_bounds__(kStTPB, 8) k_classify(/' $K/um_kernels.cu
run ipt4_lb8
