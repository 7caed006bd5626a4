#!/bin/bash
# A/B of the dim_T = 1 LBM push kernels on 256^3 (FP32 / FP64): tools/lbm_ab.sh "ENV=.." ...
for v in "$@"; do
  echo "== $v"; env $v python tools/lbm_quick.py 256 1
done
