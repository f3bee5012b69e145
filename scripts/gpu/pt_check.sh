# persistent-tile kernel change: parity (bitwise vs one-tile, batched models) + b128 / b16 timelines
P=${P:-p}
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 900 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_models.py tests/test_gpu_modes.py -q -x -k "persistent or stem_fold or batched or batch32" > gpurun_out/${P}_pytest.log 2>&1; tail -1 gpurun_out/${P}_pytest.log
for b in 128 16; do timeout 300 python scripts/node_timeline.py resnet50 --batch $b --reps 10 > gpurun_out/${P}_tl_r50_b${b}.log 2>&1; done
head -1 gpurun_out/${P}_tl_*.log
