# hot-path A/B: alternate an experiment switch ($SW) on / off, 3 rounds, one box
P=${P:-h}
python -c "import __graft_entry__ as g; g.build()" || exit 1
for r in 1 2 3; do
  for m in ${MODELS:-resnet50}; do
    timeout 300 python scripts/hot_probe.py $m >> gpurun_out/${P}_hot.log 2>&1
    env $SW timeout 300 python scripts/hot_probe.py $m >> gpurun_out/${P}_hot.log 2>&1
  done
done
grep hot gpurun_out/${P}_hot.log
