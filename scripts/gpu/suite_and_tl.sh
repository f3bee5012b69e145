P=${P:-s}
python -c "import __graft_entry__ as g; g.build()" || exit 1
for b in 1 128; do timeout 300 python scripts/node_timeline.py resnet50 --batch $b --reps 10 > gpurun_out/${P}_tl_r50_b${b}.log 2>&1; done
head -5 gpurun_out/${P}_tl_*.log
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/${P}_pytest_gpu.log 2>&1; tail -3 gpurun_out/${P}_pytest_gpu.log
timeout 300 python __graft_entry__.py smoke > gpurun_out/${P}_smoke.log 2>&1; tail -1 gpurun_out/${P}_smoke.log
