# stem fold (D16): parity, timelines and fresh-process cold starts with the fold on / off (same box)
P=${P:-f}
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 900 python -m pytest tests/test_gpu_kernels.py -q -x -k "stem_fold or unfolded or conv_cases" > gpurun_out/${P}_pytest_fold.log 2>&1; tail -1 gpurun_out/${P}_pytest_fold.log
for b in 1 128; do timeout 300 python scripts/node_timeline.py resnet50 --batch $b --reps 10 > gpurun_out/${P}_tl_r50_b${b}.log 2>&1; done
head -5 gpurun_out/${P}_tl_*.log
for round in 1 2; do
  timeout 600 python scripts/cold_samples.py --model resnet50 --n 12 --schemes pask_single_function > gpurun_out/${P}_cold_fold_$round.log 2>&1
  PASK_STEM_FOLD=0 timeout 600 python scripts/cold_samples.py --model resnet50 --n 12 --schemes pask_single_function > gpurun_out/${P}_cold_nofold_$round.log 2>&1
done
tail -3 gpurun_out/${P}_cold_*.log
