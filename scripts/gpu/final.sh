# final round-end evidence: GPU suite, smoke, default bench, batch 64 / 128 bench lines
P=${P:-final}
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/${P}_pytest_gpu.log 2>&1; tail -2 gpurun_out/${P}_pytest_gpu.log
timeout 300 python __graft_entry__.py smoke > gpurun_out/${P}_smoke.log 2>&1; tail -1 gpurun_out/${P}_smoke.log
timeout 900 python bench.py > gpurun_out/${P}_bench.json 2> gpurun_out/${P}_bench.err
for b in 64 128; do
  timeout 600 python bench.py --batch $b --steps 30 --warmup 5 --no-configs --py-cold-samples 0 --cold-samples 5 \
      --timeline-samples 2 --ablation-samples 0 --no-cpu-baseline > gpurun_out/${P}_bench_batch$b.json 2> gpurun_out/${P}_bench_batch$b.err
done
ls -la gpurun_out | grep ${P}
