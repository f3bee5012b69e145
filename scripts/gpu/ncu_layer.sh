# ncu --set full of one contraction launch of a model (the bench's hot path kernel)
# usage: P=<prefix> K=<kernel regex> SKIP=<launches to skip> B=<batch> bash scripts/gpu/ncu_layer.sh
python -c "import __graft_entry__ as g; g.build()" || exit 1
python scripts/fold_probe.py resnet50 --batch ${B:-128} || exit 1
ncu --kernel-name regex:${K:-pask_conv_igemm_pt} --launch-skip ${SKIP:-2} --launch-count 1 --set full --import-source on \
  --clock-control none -o gpurun_out/${P}_layer -f python scripts/fold_probe.py resnet50 --batch ${B:-128} > gpurun_out/${P}_ncu.log 2>&1
tail -2 gpurun_out/${P}_ncu.log
