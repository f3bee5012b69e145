#!/bin/bash
# Hot-latency A/B over runtime experiment knobs (bench.py, ResNet-50 b1 unless $1 given).
b=${1:-1}
for st in coal tma; do for pre in 0 1 2; do for one in 0 1; do
  envs=""
  [ $st = tma ] && envs="$envs PASK_TMA_STORE=1"
  [ $pre != 0 ] && envs="$envs PASK_PRE_B=$pre"
  [ $one = 1 ] && envs="$envs PASK_ONE_CTA_PER_SM=1"
  out=$(env $envs python bench.py --batch $b --steps 100 --warmup 5 --no-cpu-baseline 2>/dev/null | tail -n1)
  echo "store=$st pre_b=$pre one_cta=$one : $(echo "$out" | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["hot_ms"], d["hot_l2_warm_ms"], d["cold_ms"])')"
done; done; done
