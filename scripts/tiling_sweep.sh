#!/bin/bash
# Hot-latency sweep over the contraction tiling knobs (plan.cpp gemm_tiling).
b=${1:-1}; m=${2:-resnet50}
run() { out=$(env "$@" python bench.py --model $m --batch $b --steps 100 --warmup 5 --no-cpu-baseline 2>/dev/null | tail -n1)
  echo "$* : $(echo "$out" | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["hot_ms"], d["hot_l2_warm_ms"], d["cold_ms"])' 2>&1)"; }
run X=0
run PASK_TILE_TARGET=148
run PASK_BN_MIN=32
run PASK_BN_MIN=32 PASK_TILE_TARGET=148
run PASK_BN_MIN=16 PASK_TILE_TARGET=148
run PASK_SPLIT_MINKB=4
run PASK_SPLIT_MINKB=2
run PASK_SPLIT_MAX=16
run PASK_SPLIT_MAX=16 PASK_SPLIT_MINKB=4
run PASK_BN_MIN=32 PASK_SPLIT_MINKB=4
run PASK_BN_MIN=32 PASK_TILE_TARGET=148 PASK_SPLIT_MINKB=4
