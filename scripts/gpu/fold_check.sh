# stem fold (D16): parity + timelines fold on / off + ncu of the layout kernel
P=${P:-s7}
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 900 python -m pytest tests/test_gpu_kernels.py -q -x -k "stem_fold or unfolded or conv_cases or persistent" > gpurun_out/${P}_pytest_fold.log 2>&1; tail -3 gpurun_out/${P}_pytest_fold.log
timeout 1200 python -m pytest tests/test_gpu_models.py tests/test_gpu_modes.py -q -x > gpurun_out/${P}_pytest_models.log 2>&1; tail -3 gpurun_out/${P}_pytest_models.log
for b in 1 128; do
  timeout 300 python scripts/node_timeline.py resnet50 --batch $b --reps 10 > gpurun_out/${P}_tl_r50_b${b}_fold.log 2>&1
  PASK_STEM_FOLD=0 timeout 300 python scripts/node_timeline.py resnet50 --batch $b --reps 10 > gpurun_out/${P}_tl_r50_b${b}_nofold.log 2>&1
done
head -6 gpurun_out/${P}_tl_*.log
ncu --kernel-name pask_mem --launch-skip 0 --launch-count 1 --set full --import-source on --clock-control none \
  -o gpurun_out/${P}_fold_b128 -f python scripts/fold_probe.py resnet50 --batch 128 > gpurun_out/${P}_ncu_b128.log 2>&1
