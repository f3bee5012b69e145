#!/bin/bash
# Hot-latency sweep over split-K knobs for several models.
run() { m=$1; shift; out=$(env "$@" python bench.py --model $m --steps 100 --warmup 5 --no-cpu-baseline 2>/dev/null | tail -n1)
  echo "$m $* : $(echo "$out" | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["hot_ms"], d["hot_l2_warm_ms"])' 2>&1)"; }
for m in bert_base_fa resnet50 mobilenet_v2; do
run $m X=0
run $m PASK_SPLIT_FILL=1
run $m PASK_SPLIT_FILL=1 PASK_SPLIT_MINKB=4
run $m PASK_SPLIT_MINKB=4
run $m PASK_SPLIT_FILL=1 PASK_TILE_TARGET=148
run $m PASK_BN_MIN=32 PASK_SPLIT_FILL=1
done
