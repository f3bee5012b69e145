# D18 (resident B for one-N-tile persistent layers): parity + b128 / b16 timelines on / off
P=${P:-b}
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 900 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_models.py tests/test_gpu_modes.py -q -x -k "persistent or stem_fold or batched or batch32" > gpurun_out/${P}_pytest.log 2>&1; tail -1 gpurun_out/${P}_pytest.log
for b in 128 16; do
  timeout 300 python scripts/node_timeline.py resnet50 --batch $b --reps 10 > gpurun_out/${P}_tl_r50_b${b}.log 2>&1
  PASK_NO_B_RES=1 timeout 300 python scripts/node_timeline.py resnet50 --batch $b --reps 10 > gpurun_out/${P}_tl_r50_b${b}_nobres.log 2>&1
done
head -8 gpurun_out/${P}_tl_*.log
